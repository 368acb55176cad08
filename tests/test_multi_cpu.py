"""Multi-rank host logic on CPU (world_size 2, gloo): shards of one genome generated
independently per rank, calibration counts all-reduced across ranks, records gathered — must
equal the single-process result.  The per-shard arithmetic here is the oracle's; what is under
test is the sharding (ownership, halo, reference span) and the exchange the GPU path uses."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_icpp_luzlwfl11_b200 import shard

GENOME = dict(n_sites=24_000, depth=15.0, seed=31, n_frac=0.05, n_lead_frac=0.01, n_blocks=2,
              dup_rate=0.05)


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _rank_main(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    P = oracle.Params()
    lo, hi = shard.plan_equal(GENOME["n_sites"], 0, world)[rank]
    w = synth.generate("C1", region_lo=lo, region_hi=hi, **GENOME)
    assert w["region"] == (lo, hi)
    # the generated reference covers the calling halo
    rs0, rs1 = shard.reference_span(lo, hi, w["read_len"], 0, GENOME["n_sites"])
    assert int(w["origin"]) <= rs0 and int(w["origin"]) + len(w["ref"]) >= rs1
    ra, rb = shard.owned_reads(w["pos"], lo, hi)
    C = oracle.calib_counts(P, shard.take_reads(w, ra, rb)).astype(np.int64)
    t = torch.from_numpy(C.reshape(-1).copy())
    dist.all_reduce(t)                                   # the only exchange of the path
    p = oracle.p_matrix(P, t.numpy().astype(np.uint64).reshape(64, 256, 4, 4))
    ca, cb = shard.call_reads(w["pos"], lo, hi, w["read_len"])
    rec = oracle.call_window(P, shard.take_reads(w, ca, cb), p, lo, hi)
    # collective 2: per-rank record counts -> global output offsets
    offs, total = shard.gather_output_offsets(dist, len(rec))
    assert total == GENOME["n_sites"] and offs[rank] == lo
    out = [None] * world
    dist.all_gather_object(out, (t.numpy(), rec.tobytes(), offs))
    if rank == 0:
        q.put(out)
    dist.destroy_process_group()


def test_two_rank_shards_equal_single_process():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_rank_main, args=(r, world, port, q)) for r in range(world)]
    for pr in procs:
        pr.start()
    out = q.get(timeout=300)
    for pr in procs:
        pr.join(timeout=60)
        assert pr.exitcode == 0
    # single process, whole genome
    P = oracle.Params()
    w = synth.generate("C1", **GENOME)
    C = oracle.calib_counts(P, w)
    p = oracle.p_matrix(P, C)
    rec = oracle.call_window(P, w, p, 0, GENOME["n_sites"])
    for counts, _, _ in out:
        assert np.array_equal(counts.reshape(64, 256, 4, 4).astype(np.uint64), C)
    # every rank writes its records at its gathered offset of one whole-genome output
    offs = out[0][2]
    assert all(o[2] == offs for o in out)
    merged = bytearray(len(rec.tobytes()))
    for r, (_, b, _) in enumerate(out):
        merged[40 * offs[r]:40 * offs[r] + len(b)] = b
    assert bytes(merged) == rec.tobytes()


def test_output_offsets():
    assert shard.output_offsets([3, 0, 5, 2]) == [0, 3, 3, 8]
    assert shard.output_offsets([]) == []


def test_plan_by_bases_balances_and_covers():
    rng = np.random.default_rng(0)
    pos = np.sort(np.concatenate([rng.integers(0, 1000, 5000), rng.integers(1000, 100_000, 5000)]))
    ln = np.full(len(pos), 100)
    plan = shard.plan_by_bases(pos.astype(np.uint64), ln, 100_000, 0, 4)
    assert plan[0][0] == 0 and plan[-1][1] == 100_000
    assert all(a[1] == b[0] for a, b in zip(plan, plan[1:]))
    owned = [shard.owned_reads(pos.astype(np.uint64), s0, s1) for s0, s1 in plan]
    counts = [rb - ra for ra, rb in owned]
    assert sum(counts) == len(pos)
    assert max(counts) < 1.3 * len(pos) / 4
    # equal-site planning would put half the reads on the first shard
    eq = [shard.owned_reads(pos.astype(np.uint64), *s) for s in shard.plan_equal(100_000, 0, 4)]
    assert eq[0][1] - eq[0][0] > 0.5 * len(pos)


def test_call_halo_contains_every_covering_read():
    w = synth.generate("C1", n_sites=5000, depth=12.0, seed=3)
    for s0, s1 in shard.plan_equal(5000, 0, 3):
        ra, rb = shard.call_reads(w["pos"], s0, s1, 100)
        p = w["pos"].astype(np.int64)
        cover = (p + w["len"].astype(np.int64) > s0) & (p < s1)
        idx = np.nonzero(cover)[0]
        assert idx.min() >= ra and idx.max() < rb
