"""GPU decode of the packed read format (reading R21, gsnp_unpack_reads / k_unpack): streams
written by the ORACLE's encoder (oracle/pack.py) decode to the original read arrays exactly, from
host (pinned and pageable) and device memory (aligned and not); the C2-sized stream written by the
library decodes to the C2 input; and calls on decoded reads give the same records."""
from __future__ import annotations

import numpy as np
import pytest

import synth
from oracle import pack as opk
from paper_conf_icpp_luzlwfl11_b200 import gsnp
from tests.test_pack_host import _edge

pytestmark = pytest.mark.gpu

KEYS = ("pos", "len", "off", "bases", "quals", "strand", "hits")


def _same(got, w):
    import torch
    n = len(w["pos"])
    ln = np.asarray(w["len"], np.int64)
    off = np.asarray(w["off"], np.int64)
    g = {k: v.cpu().numpy() for k, v in got.items()}
    assert np.array_equal(g["pos"], np.asarray(w["pos"], np.uint64))
    assert np.array_equal(g["len"], ln.astype(np.uint16))
    assert np.array_equal(g["strand"], np.asarray(w["strand"], np.uint8))
    assert np.array_equal(g["hits"], np.asarray(w["hits"], np.uint16))
    want_off = np.zeros(n + 1, np.uint64)
    want_off[1:] = np.cumsum(ln).astype(np.uint64)
    assert np.array_equal(g["off"], want_off)
    contiguous = np.array_equal(off - off[0], want_off.astype(np.int64))
    for k in ("bases", "quals"):
        src = np.asarray(w[k])[off[0]:off[-1]] if contiguous else \
            np.concatenate([np.asarray(w[k])[off[r]:off[r] + ln[r]] for r in range(n)])
        assert np.array_equal(g[k][:int(want_off[-1])], src), k
    del torch


@pytest.mark.parametrize("block_reads", [1, 37, 1024, 4096])
def test_oracle_stream_decodes_exactly(block_reads):
    import torch
    for w in (_edge(), synth.generate("C1", n_sites=40_000, depth=15.0, seed=23)):
        buf = np.frombuffer(opk.pack(w, block_reads), np.uint8)
        with gsnp.Context.from_workload(w) as ctx:
            _same(ctx.unpack_reads(buf), w)                                    # pageable host
            _same(ctx.unpack_reads(torch.from_numpy(buf.copy()).pin_memory()), w)   # pinned host
            _same(ctx.unpack_reads(torch.from_numpy(buf.copy()).cuda()), w)          # device
            odd = torch.zeros(len(buf) + 3, dtype=torch.uint8, device="cuda")
            odd[3:] = torch.from_numpy(buf.copy()).cuda()
            _same(ctx.unpack_reads(odd[3:]), w)                                 # unaligned device
            torch.cuda.synchronize()


def test_c2_stream_roundtrip_and_same_records():
    import torch
    w = synth.generate("C2")
    buf = gsnp.pack_reads(w, 1024)
    raw = sum(np.asarray(w[k]).nbytes for k in KEYS)
    assert len(buf) * 4 < raw                                   # > 4x smaller on the wire
    lo, hi = w["region"]
    with gsnp.Context.from_workload(w, stream=torch.cuda.current_stream()) as ctx:
        dev = ctx.unpack_reads(torch.from_numpy(buf).pin_memory())
        torch.cuda.synchronize()
        _same(dev, w)
        ctx.calibrate(dev)
        a = torch.empty(40 * 2_000_000, dtype=torch.uint8, device="cuda")
        ctx.call(dev, lo + 20_000_000, lo + 22_000_000, a)
        orig = {k: torch.from_numpy(np.ascontiguousarray(w[k])).cuda() for k in KEYS}
        ctx.calibrate(orig)
        b = torch.empty_like(a)
        ctx.call(orig, lo + 20_000_000, lo + 22_000_000, b)
        torch.cuda.synchronize()
        assert torch.equal(a, b)


def test_bad_stream_is_an_error():
    import torch
    w = _edge()
    good = gsnp.pack_reads(w)
    bad = good.copy()
    bad[0] ^= 1                                          # magic
    out = {k: torch.zeros(8, dtype=torch.uint64, device="cuda") for k in KEYS}
    with gsnp.Context.from_workload(w) as ctx:
        for stream, n in ((bad, len(bad)), (good, 100)):  # bad magic; truncated stream
            st = gsnp.lib().gsnp_unpack_reads(ctx.h, gsnp._ptr(stream), n,
                                             *[gsnp._ptr(out[k]) for k in KEYS])
            assert st == -1
        dev = ctx.unpack_reads(good)                      # the context is still usable
        assert int(dev["off"][-1]) == gsnp.packed_sizes(good)[1]


@pytest.mark.parametrize("block_reads", [5, 1024])
def test_reference_relative_stream_decodes_exactly(block_reads):
    """Version 2 streams (bases predicted from the context's reference, mismatches listed):
    written by the oracle, decoded on the GPU against the context's device reference."""
    import torch
    w = synth.generate("C1", n_sites=40_000, depth=15.0, seed=29)
    w = dict(w, ref=np.asarray(w["ref"]).copy())
    w["ref"][9000:9200] = 4                            # reads over an N stretch
    buf = np.frombuffer(opk.pack(w, block_reads, ref=w["ref"], origin=int(w["origin"])), np.uint8)
    with gsnp.Context.from_workload(w) as ctx:
        _same(ctx.unpack_reads(buf), w)
        _same(ctx.unpack_reads(torch.from_numpy(buf.copy()).cuda()), w)
        torch.cuda.synchronize()


def test_c2_reference_relative_roundtrip():
    import torch
    w = synth.generate("C2")
    lo = int(w["origin"])
    buf = gsnp.pack_reads(w, 1024, ref=w["ref"], origin=lo)
    assert len(buf) < 0.35 * len(w["bases"])              # < 0.35 B per base on the wire
    with gsnp.Context.from_workload(w, stream=torch.cuda.current_stream()) as ctx:
        dev = ctx.unpack_reads(torch.from_numpy(buf).pin_memory())
        torch.cuda.synchronize()
        _same(dev, w)
