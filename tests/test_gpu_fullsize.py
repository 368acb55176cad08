"""Exhaustive parity at BASELINE.json's full sizes, in the launch configuration bench.py times
(device-resident inputs and outputs): calibration counts and tables bit-exact over the whole input,
and EVERY record of the shard compared with the oracle's — the oracle run as P independent
single-threaded processes over windows (SURVEY.md §8(d) timing protocol; tests/_mp.py).  L10 and
post10 are compared through gsnp_debug_window on a multi-million-site window (all of C5).  The
near-tie and near-integer counts of each run are printed (run with -s) and asserted small."""
from __future__ import annotations

import json
import os

import numpy as np
import pytest

import oracle
import synth
from paper_conf_icpp_luzlwfl11_b200 import gsnp
from tests._mp import calib_parallel, call_parallel
from tests._parity import compare

pytestmark = pytest.mark.gpu

KEYS = ("pos", "len", "off", "bases", "quals", "strand", "hits")


def _report(name, d):
    print(f"\n[fullsize] {name}: {json.dumps(d)}")
    out = os.environ.get("GSNP_PARITY_REPORT")
    if out:
        with open(out, "a") as f:
            f.write(json.dumps(dict(d, name=name)) + "\n")


def _exhaustive(name, w, lo, hi, dbg_lo, dbg_hi):
    """GPU (calibrate over all of w's reads, call [lo, hi)) vs the multi-process oracle on every
    site; debug L10 / post10 on [dbg_lo, dbg_hi)."""
    import torch
    P = oracle.Params()
    C_or, cst = calib_parallel(P, w)
    p_or = oracle.p_matrix(P, C_or)
    dev = {k: torch.from_numpy(np.ascontiguousarray(w[k])).cuda() for k in KEYS}
    S = hi - lo
    with gsnp.Context.from_workload(w, stream=torch.cuda.current_stream()) as ctx:
        counts = torch.zeros(64 * 256 * 16, dtype=torch.uint64, device="cuda")
        ctx.calibrate_count(dev, counts)
        assert np.array_equal(counts.cpu().numpy().reshape(64, 256, 4, 4), C_or)
        ctx.calibrate_finalize(counts)
        t = ctx.get_tables()
        L = P.max_read_len
        assert np.array_equal(t["p"][:, :L], p_or[:, :L])
        out = torch.empty(40 * S, dtype=torch.uint8, device="cuda")
        ctx.call(dev, lo, hi, out)
        torch.cuda.synchronize()
        rec_g = out.cpu().numpy().view(gsnp.RECORD_DTYPE)
        del out
        dg = ctx.debug_window(dev, dbg_lo, dbg_hi, want=("L10", "post10", "records"))
    del dev
    assert np.array_equal(rec_g["pos"], np.arange(lo, hi, dtype=np.uint64))
    # debug-path records are the production records
    assert dg["records"].tobytes() == rec_g[dbg_lo - lo:dbg_hi - lo].tobytes()
    rec_o, L10_o, _, st = call_parallel(P, w, p_or, lo, hi, want_L10=True)
    rep = compare(w, rec_g, rec_o, L10_o, P=P)
    del rec_o, L10_o
    rw, Lw, pw, _ = call_parallel(P, w, p_or, dbg_lo, dbg_hi, want_L10=True, want_post=True)
    repw = compare(w, dg["records"], rw, Lw, pw, dg["L10"], dg["post10"], P=P)
    d = dict(sites=int(S), near_tie=rep["near_tie"],
             near_tie_uninformative=rep["near_tie_uninformative"], near_int=rep["near_int"],
             near_int_candidates=rep["near_int_candidates"],
             debug_window=[int(dbg_lo), int(dbg_hi)], debug_L10_max_rel=repw.get("L10_max_rel"),
             debug_near_tie=repw["near_tie"], oracle_procs=st["procs"],
             oracle_wall_s=round(st["wall_s"], 1), oracle_cpu_s=round(st["cpu_s"], 1),
             calib_oracle_wall_s=round(cst["wall_s"], 1))
    _report(name, d)
    # near ties / near-integer excuses stay rare (a systematic error would show up as many)
    assert rep["near_tie"] <= max(10, S // 1_000_000) and rep["near_int"] <= max(10, S // 1_000_000)
    return d


def test_c2_exhaustive():
    """C2: chr21-like 48 Mb at 20X (the bench workload): all 48 M records; L10/post10 on 4 M sites."""
    w = synth.generate("C2")
    lo, hi = w["region"]
    _exhaustive("C2", w, lo, hi, lo + 8_000_000, lo + 12_000_000)


def test_c5_exhaustive():
    """C5: 5 Mb exome-like target at 100X with 10% PCR duplicates (deep kernel, warp paths): all
    records, and L10/post10 over the whole target."""
    w = synth.generate("C5")
    lo, hi = w["region"]
    _exhaustive("C5", w, lo, hi, lo, hi)


def _region(name, k, of):
    base = synth.CONFIGS[name]
    n = base.n_sites
    return synth.generate(base.scaled(region_lo=k * n // of, region_hi=(k + 1) * n // of))


def test_c3_shard_exhaustive():
    """C3: chr1-like 249 Mb at 30X, rank 3 of 8 (31 Mb shard with read halos on both sides)."""
    w = _region("C3", 3, 8)
    lo, hi = w["region"]
    _exhaustive("C3/8 rank3", w, lo, hi, lo, lo + 4_000_000)


def test_c4_shard_exhaustive():
    """C4: whole-genome 3.1 Gb at 12.5X, a 48 Mb piece from the middle (rank 21 of 64)."""
    w = _region("C4", 21, 64)
    lo, hi = w["region"]
    _exhaustive("C4/64 rank21", w, lo, hi, hi - 4_000_000, hi)
