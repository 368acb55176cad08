"""Multi-GPU flow through libgsnp on one GPU (the "fake cluster" of §4): the
genome is split into contiguous shards by shard.plan_by_bases; each rank calibrates only the reads
it owns (by start), the counts are summed (the all-reduce), every rank finalizes the same tables,
calls its own sites with the read-length halo, and its records land at the offset the all-gather
of per-rank sizes gives.  The merged output must be byte-identical to one context calling the
whole genome.  Sites are independent, so no other exchange exists."""
from __future__ import annotations

import os
import socket
import tempfile

import numpy as np
import pytest

import synth
from paper_conf_icpp_luzlwfl11_b200 import gsnp, shard

pytestmark = pytest.mark.gpu

GENOME = dict(n_sites=1_500_000, depth=20.0, seed=61, n_frac=0.1, n_lead_frac=0.03, n_blocks=4)


def _genome():
    return synth.generate("C2", **GENOME)


def _rank_ctx(w, s0, s1, **params):
    """A context holding only the reference span rank [s0, s1) needs (halo both sides)."""
    origin, n = int(w["origin"]), len(w["ref"])
    L = int(w["read_len"])
    rs0, rs1 = shard.reference_span(s0, s1, L, origin, n)
    kp = np.asarray(w["known_pos"], np.uint64)
    k0, k1 = np.searchsorted(kp, np.uint64(rs0)), np.searchsorted(kp, np.uint64(rs1))
    return gsnp.Context(w["ref"][rs0 - origin:rs1 - origin], rs0, kp[k0:k1],
                        np.asarray(w["known_prior10"])[k0:k1], **params)


def _single(w):
    origin, n = int(w["origin"]), len(w["ref"])
    with gsnp.Context.from_workload(w) as ctx:
        counts = ctx.calibrate_count(w)
        ctx.calibrate_finalize(counts)
        return counts, ctx.call(w, origin, origin + n)


@pytest.mark.parametrize("world", [2, 4, 8])
def test_virtual_ranks_byte_identical(world):
    w = _genome()
    origin, n = int(w["origin"]), len(w["ref"])
    plan = shard.plan_by_bases(w["pos"], w["len"], n, origin, world)
    assert plan[0][0] == origin and plan[-1][1] == origin + n
    ctxs = [_rank_ctx(w, a, b) for a, b in plan]
    total = np.zeros(64 * 256 * 16, np.uint64)
    for (a, b), ctx in zip(plan, ctxs):                      # calibration: owned reads only
        ra, rb = shard.owned_reads(w["pos"], a, b)
        total += ctx.calibrate_count(shard.take_reads(w, ra, rb))
    recs = []
    for (a, b), ctx in zip(plan, ctxs):
        ctx.calibrate_finalize(total)                        # identical tables on every rank
        ca, cb = shard.call_reads(w["pos"], a, b, int(w["read_len"]))
        recs.append(ctx.call(shard.take_reads(w, ca, cb), a, b))
        ctx.close()
    offs = shard.output_offsets([len(r) for r in recs])
    merged = np.zeros(n, gsnp.RECORD_DTYPE)
    for o, r in zip(offs, recs):
        merged[o:o + len(r)] = r
    counts1, rec1 = _single(w)
    assert np.array_equal(total, counts1)
    assert merged.tobytes() == rec1.tobytes()
    # balance: shards hold similar numbers of aligned bases
    bases = [int(w["off"][shard.owned_reads(w["pos"], a, b)[1]] - w["off"][shard.owned_reads(w["pos"], a, b)[0]])
             for a, b in plan]
    assert max(bases) <= 1.05 * (sum(bases) / world)


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _rank_main(rank, world, port, path):
    """One process per rank, gloo collectives, libgsnp on cuda:0 (one GPU box)."""
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    w = _genome()
    origin, n = int(w["origin"]), len(w["ref"])
    a, b = shard.plan_by_bases(w["pos"], w["len"], n, origin, world)[rank]
    ctx = _rank_ctx(w, a, b, device=0)
    ra, rb = shard.owned_reads(w["pos"], a, b)
    c = ctx.calibrate_count(shard.take_reads(w, ra, rb)).astype(np.int64)
    t = torch.from_numpy(c)
    dist.all_reduce(t)                                       # §8(e) collective 1
    ctx.calibrate_finalize(t.numpy().astype(np.uint64))
    ca, cb = shard.call_reads(w["pos"], a, b, int(w["read_len"]))
    rec = ctx.call(shard.take_reads(w, ca, cb), a, b)
    offs, tot = shard.gather_output_offsets(dist, len(rec), "cpu")   # §8(e) collective 2
    assert tot == n
    out = np.memmap(path, dtype=gsnp.RECORD_DTYPE, mode="r+", shape=(n,))
    out[offs[rank]:offs[rank] + len(rec)] = rec
    out.flush()
    ctx.close()
    dist.barrier()
    dist.destroy_process_group()


def test_two_processes_gloo_byte_identical():
    import torch.multiprocessing as mp
    w = _genome()
    n = len(w["ref"])
    with tempfile.TemporaryDirectory() as d:
        path = os.path.join(d, "records.bin")
        np.memmap(path, dtype=gsnp.RECORD_DTYPE, mode="w+", shape=(n,)).flush()
        mp.start_processes(_rank_main, args=(2, _free_port(), path), nprocs=2, join=True,
                           start_method="spawn")
        merged = np.array(np.memmap(path, dtype=gsnp.RECORD_DTYPE, mode="r", shape=(n,)))
    _, rec1 = _single(w)
    assert merged.tobytes() == rec1.tobytes()
