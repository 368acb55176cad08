"""GPU edge cases of the read input (ABI: len 1..max_read_len, include/gsnp.h): reads of 1-3 bp
on both strands through the calibration histogram (every batch takes the flat or staged path by
its read lengths) and through the caller, and out-of-contract read arrays, which must come back
as statuses from gsnp_calibrate / gsnp_call without touching memory out of bounds."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import synth
from paper_conf_icpp_luzlwfl11_b200 import gsnp
from tests._parity import compare
from tests._util import workload

pytestmark = pytest.mark.gpu

OP = oracle.Params()


def _short_reads(lengths, n_reads, S=3_000, seed=0, dup_every=7):
    """n_reads reads with lengths drawn from `lengths`, both strands, 5% multi-hit, sorted by
    position; every `dup_every`-th read repeats its predecessor's start (pcr > 1)."""
    rng = np.random.default_rng(seed)
    ref = rng.integers(0, 4, S).astype(np.uint8)
    ref[rng.random(S) < 0.01] = 4
    reads = []
    for i in range(n_reads):
        ln = int(rng.choice(lengths))
        p = int(rng.integers(0, S - ln + 1)) if i % dup_every or not reads else reads[-1]["pos"]
        p = min(p, S - ln)
        b = ref[p:p + ln].copy()
        b[b == 4] = 0
        err = rng.random(ln) < 0.05
        b[err] = (b[err] + rng.integers(1, 4, err.sum())) % 4
        b[rng.random(ln) < 0.01] = 4
        reads.append(dict(pos=p, strand=int(rng.integers(2)), hits=1 if rng.random() > 0.05 else 3,
                          bases=b, quals=list(rng.integers(0, 41, ln))))
    kn = [(int(s), [0.8, 0.1, 0.1, 0.1, 1e-3, 1e-3, 1e-3, 1e-3, 1e-3, 1e-3])
          for s in sorted(rng.choice(S, 20, replace=False))]
    return workload(ref, reads, known=kn)


@pytest.mark.parametrize("lengths", [(1,), (2,), (3,), (1, 2, 3)])
def test_short_reads_calibration_and_calls(lengths):
    """1-, 2- and 3-bp reads (uniform batches take the flat word path except at length 1, where
    the read-index multiply-high would wrap; mixed lengths take the staged path)."""
    w = _short_reads(lengths, 40_000, seed=len(lengths) * 10 + lengths[0])
    C = oracle.calib_counts(OP, w)
    assert C.sum() > 0
    p = oracle.p_matrix(OP, C)
    S = len(w["ref"])
    rec_o, dbg = oracle.call_window(OP, w, p, 0, S, debug=True)
    with gsnp.Context.from_workload(w) as ctx:
        counts = ctx.calibrate_count(w)
        assert np.array_equal(counts.reshape(64, 256, 4, 4), C)
        ctx.calibrate_finalize(counts)
        rec_g = ctx.call(w, 0, S)
        dg = ctx.debug_window(w, 0, S)
    compare(w, rec_g, rec_o, dbg["L10"], dbg["post10"], dg["L10"], dg["post10"])


def test_single_one_bp_read_each_strand():
    w = workload("ACGTN", [dict(pos=1, strand=1, bases="C", quals=30),
                           dict(pos=2, strand=0, bases="G", quals=20)])
    C = oracle.calib_counts(OP, w)
    with gsnp.Context.from_workload(w) as ctx:
        counts = ctx.calibrate_count(w)
        assert np.array_equal(counts.reshape(64, 256, 4, 4), C)
        ctx.calibrate_finalize(counts)
        rec_g = ctx.call(w, 0, 5)
    p = oracle.p_matrix(OP, C)
    rec_o, dbg = oracle.call_window(OP, w, p, 0, 5, debug=True)
    compare(w, rec_g, rec_o, dbg["L10"])


def _big():
    return synth.generate("C1", n_sites=60_000, depth=20.0, seed=31)


def _bad_variants(w):
    """Read sets that break the contract in the middle of a large input (inside one
    calibration batch, where the TMA stage windows are sized from the batch's first/last read)."""
    n = len(w["pos"])
    m = n // 2
    out = {}
    v = dict(w)                                    # one interior read moved far back
    v["pos"] = w["pos"].copy()
    v["pos"][m] = 5
    out["interior_unsorted"] = (v, -3)
    v = dict(w)                                    # one interior read moved far forward
    v["pos"] = w["pos"].copy()
    v["pos"][m] = w["pos"][-1] - 50
    out["interior_forward"] = (v, -3)
    v = dict(w)                                    # offsets out of order inside a batch
    v["off"] = w["off"].copy()
    v["off"][m] = w["off"][m - 40]
    out["offsets_backwards"] = (v, -2)
    v = dict(w)                                    # a length beyond max_read_len
    v["len"] = w["len"].copy()
    v["len"][m] = 300
    out["too_long"] = (v, -2)
    v = dict(w)                                    # a read past the reference end
    v["pos"] = w["pos"].copy()
    v["pos"][-1] = len(w["ref"]) - 10
    out["past_end"] = (v, -2)
    return out


@pytest.mark.parametrize("device_arrays", [False, True])
def test_contract_violations_are_statuses_in_calibrate_and_call(device_arrays):
    import torch
    w = _big()
    S = len(w["ref"])
    with gsnp.Context.from_workload(w) as ctx:
        for name, (bad, status) in _bad_variants(w).items():
            src = bad
            if device_arrays:
                src = {k: torch.from_numpy(np.ascontiguousarray(bad[k])).cuda()
                       for k in ("pos", "len", "off", "bases", "quals", "strand", "hits")}
            with pytest.raises(gsnp.GsnpError) as e:
                ctx.calibrate_count(src)
            assert e.value.status == status, (name, e.value.status)
            with pytest.raises(gsnp.GsnpError) as e:
                ctx.calibrate(src)
            assert e.value.status == status, (name, "calibrate", e.value.status)
        ctx.calibrate(w)                           # the context is still usable
        for name, (bad, status) in _bad_variants(w).items():
            with pytest.raises(gsnp.GsnpError) as e:
                ctx.call(bad, 0, S)
            assert e.value.status == status, (name, "call", e.value.status)
        rec = ctx.call(w, 0, S)
    P = OP
    C = oracle.calib_counts(P, w)
    rec_o, dbg = oracle.call_window(P, w, oracle.p_matrix(P, C), 0, S, debug=True)
    compare(w, rec, rec_o, dbg["L10"])


def test_pile_inside_shallow_window():
    """A 1500-read pile inside a long low-depth window: the window is called by the shallow kernel,
    whose warp path must hand the >1024-key sites to the CTA path without overrunning its
    shared-memory key buffer."""
    w0 = synth.generate("C1", n_sites=60_000, depth=5.0, seed=57)
    rng = np.random.default_rng(57)
    ref = w0["ref"]
    reads = []
    for k in range(len(w0["pos"])):
        o = int(w0["off"][k])
        ln = int(w0["len"][k])
        reads.append(dict(pos=int(w0["pos"][k]), strand=int(w0["strand"][k]), hits=int(w0["hits"][k]),
                          bases=w0["bases"][o:o + ln], quals=w0["quals"][o:o + ln]))
    for k in range(1500):
        p = 30_000 + int(rng.integers(0, 4))
        b = ref[p:p + 100].copy()
        b[b == 4] = 0
        reads.append(dict(pos=p, strand=int(rng.integers(2)), bases=b, quals=list(rng.integers(2, 41, 100))))
    w = workload(ref, reads)
    S = len(ref)
    P = OP
    C = oracle.calib_counts(P, w)
    p = oracle.p_matrix(P, C)
    lo, hi = 29_000, 31_500
    rec_o, dbg = oracle.call_window(P, w, p, lo, hi, debug=True)
    with gsnp.Context.from_workload(w) as ctx:
        ctx.calibrate(w)
        rec_all = ctx.call(w, 0, S)
    assert int(rec_all["depth"][30_050]) > 1024
    compare(w, rec_all[lo:hi], rec_o, dbg["L10"])
