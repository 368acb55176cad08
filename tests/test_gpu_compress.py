"""GPU parity of the §V-B output compression (format R17): the CUDA path
(gsnp_compress / gsnp_call_compressed through the C ABI) against the CPU oracle's encoder
(oracle/compress.c) on the same seeded record tables — the word streams must be identical, and the
oracle's separate decoder must give the records back."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import synth
from paper_conf_icpp_luzlwfl11_b200 import gsnp
from tests._records import records

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def ctx():
    ref = np.zeros(1000, np.uint8)
    with gsnp.Context(ref) as c:
        yield c


def _check(ctx, r, B, device):
    import torch
    want = oracle.compress(r, B)
    if device:
        rd = torch.from_numpy(r.view(np.uint8).copy()).cuda()
        out = torch.zeros(len(want) + 7, dtype=torch.int32, device="cuda")
        _, nw = ctx.compress(rd, B, out)
        got = out[:nw].cpu().numpy().view(np.uint32)
    else:
        got, nw = ctx.compress(r, B)
    assert nw == len(want)
    if not np.array_equal(got, want):
        bad = np.flatnonzero(got != want)
        raise AssertionError(f"{len(bad)} words differ, first at {bad[:8].tolist()}: "
                             f"gpu {got[bad[:8]].tolist()} oracle {want[bad[:8]].tolist()}")
    assert oracle.decompress(got, len(r)).tobytes() == r.tobytes()


@pytest.mark.parametrize("kind,n,B", [
    ("call", 100_000, 65536), ("call", 4097, 1024), ("runs", 70_001, 8192),
    ("random", 20_000, 8192), ("random", 33, 16), ("const", 5000, 4096), ("call", 1, 65536),
    ("call", 17, 16), ("call", 2047, 2048), ("call", 2049, 2048), ("call", 6145, 3000),
    ("random", 9000, 9000), ("call", 300_000, 1 << 20), ("runs", 50_000, 1),
])
@pytest.mark.parametrize("device", [False, True])
def test_compress_matches_oracle(ctx, kind, n, B, device):
    _check(ctx, records(n, seed=n % 101, kind=kind), B, device)


def test_compress_adversarial_values(ctx):
    """0xFFFFFFFF values inside dictionaries, exactly 4096 and 4097 distinct run values, every
    site an exception, all-N planes."""
    n = 12_000
    r = records(n, seed=7)
    r["depth"][:4096] = np.arange(4096, dtype=np.uint32) * 3      # 4096 distinct runs ...
    r["depth"][4096:] = 0xFFFFFFFF                                # ... plus the max value
    r["copy_num"] = np.arange(n, dtype=np.uint32).view(np.float32)  # all distinct -> RAW
    r["genotype"] = 3
    r["ref"][::2] = 4
    r["base1"][:] = 4
    _check(ctx, r, 16384, False)
    r["depth"][4096:] = 5                                         # 4097 distinct -> RAW
    _check(ctx, r, 16384, True)
    _check(ctx, r, 4096, True)


def test_capacity_and_query(ctx):
    r = records(5000, seed=1)
    want = oracle.compress(r, 1024)
    out = np.zeros(len(want) - 1, np.uint32)
    with pytest.raises(gsnp.GsnpError) as e:
        ctx.compress(r, 1024, out)
    assert e.value.status == -7 and not out.any()
    nw = gsnp.ctypes.c_uint64(0)
    st = gsnp.lib().gsnp_compress(ctx.h, gsnp._ptr(r), len(r), 1024, None, 0, gsnp.ctypes.byref(nw))
    assert st == -7 and nw.value == len(want)
    with pytest.raises(gsnp.GsnpError):
        ctx.compress(r, 0)
    assert ctx.compress(r[:0], 1024)[1] == 0


def test_call_compressed_matches_oracle_pipeline():
    """gsnp_call_compressed on a C1 workload == oracle.compress(oracle call records)."""
    import torch
    w = synth.generate("C1", n_sites=30_000, depth=10.0, seed=23)
    P = oracle.Params()
    p = oracle.p_matrix(P, oracle.calib_counts(P, w))
    rec_o = oracle.call_window(P, w, p, 0, 30_000)
    for B in (4096, 65536):
        want = oracle.compress(rec_o, B)
        with gsnp.Context.from_workload(w) as c:
            c.calibrate(w)
            out = np.zeros(len(want), np.uint32)
            nw = c.call_compressed(w, 0, 30_000, out, B)
            assert nw == len(want) and np.array_equal(out, want)
            dev = {k: torch.from_numpy(np.ascontiguousarray(w[k])).cuda()
                   for k in ("pos", "len", "off", "bases", "quals", "strand", "hits")}
            outd = torch.zeros(len(want), dtype=torch.int32, device="cuda")
            nw = c.call_compressed(dev, 0, 30_000, outd, B)
            assert nw == len(want)
            assert np.array_equal(outd.cpu().numpy().view(np.uint32), want)
        assert oracle.decompress(want, 30_000).tobytes() == rec_o.tobytes()


@pytest.mark.slow
def test_compress_full_size():
    """A C2-sized table (48 M records, 733 blocks of 65536) through the device path: identical
    to the oracle's stream."""
    import torch
    n = 48_000_000
    r = records(n, seed=11)
    want = oracle.compress(r, 65536)
    with gsnp.Context(np.zeros(16, np.uint8)) as c:
        rd = torch.from_numpy(r.view(np.uint8)).cuda()
        out = torch.zeros(len(want), dtype=torch.int32, device="cuda")
        _, nw = c.compress(rd, 65536, out)
        assert nw == len(want)
        got = out.cpu().numpy().view(np.uint32)
    assert np.array_equal(got, want)
