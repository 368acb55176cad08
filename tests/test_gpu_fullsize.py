"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (device-
resident inputs and outputs): calibration counts and tables bit-exact over the whole input;
records on sampled sites, each recomputed by the oracle from the reads covering it."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import synth
from paper_conf_icpp_luzlwfl11_b200 import gsnp
from tests._parity import compare

pytestmark = pytest.mark.gpu


def _run_full(name, n_sample, seed=0, **over):
    import torch
    w = synth.generate(name, **over)
    S = len(w["ref"])
    w0 = int(w["origin"])
    P = oracle.Params()
    C_or = oracle.calib_counts(P, w)
    p_or = oracle.p_matrix(P, C_or)
    dev = {k: torch.from_numpy(np.ascontiguousarray(w[k])).cuda()
           for k in ("pos", "len", "off", "bases", "quals", "strand", "hits")}
    with gsnp.Context.from_workload(w, stream=torch.cuda.current_stream()) as ctx:
        counts = torch.zeros(64 * 256 * 16, dtype=torch.uint64, device="cuda")
        ctx.calibrate_count(dev, counts)
        assert np.array_equal(counts.cpu().numpy().reshape(64, 256, 4, 4), C_or)
        ctx.calibrate_finalize(counts)
        t = ctx.get_tables()
        assert np.array_equal(t["p"][:, :P.max_read_len], p_or[:, :P.max_read_len])
        out = torch.empty(40 * S, dtype=torch.uint8, device="cuda")
        ctx.call(dev, w0, w0 + S, out)
        torch.cuda.synchronize()
        rec_g = out.cpu().numpy().view(gsnp.RECORD_DTYPE)
    assert np.array_equal(rec_g["pos"], np.arange(w0, w0 + S, dtype=np.uint64))
    rng = np.random.default_rng(seed)
    covered = np.nonzero(rec_g["depth"] > 0)[0]
    pick = np.unique(np.concatenate([rng.choice(S, n_sample // 2, replace=False),
                                     rng.choice(covered, n_sample // 2, replace=False)]))
    # deepest and het-called sites too
    het = np.nonzero(np.isin(rec_g["genotype"], [1, 2, 3, 5, 6, 8]))[0]
    pick = np.unique(np.concatenate([pick, het[:200], np.argsort(rec_g["depth"])[-50:]]))
    recs, L10s = [], []
    for i in pick:
        s = w0 + int(i)
        ra, rb = synth.read_range(w, s, s + 1)
        sub = synth.slice_reads(w, ra, rb)
        r, d = oracle.call_window(P, sub, p_or, s, s + 1, debug=True)
        recs.append(r)
        L10s.append(d["L10"])
    rec_o = np.concatenate(recs)
    rep = compare(w, rec_g[pick], rec_o, np.concatenate(L10s))
    return rep, len(pick)


def test_c2_fullsize_sampled():
    """C2: chr21-like 48 Mb at 20X (the bench workload)."""
    rep, n = _run_full("C2", 3000)
    assert n >= 3000


def test_c5_fullsize_sampled():
    """C5: 5 Mb exome-like target at 100X with 10% PCR duplicates (warp paths)."""
    rep, n = _run_full("C5", 2000, seed=1)
    assert n >= 2000


def _run_region(name, n_sample, seed, **cfg):
    """One rank's shard of a multi-GPU config: region generation with the read
    halo, called over the shard's own sites [lo, hi) with every read that can touch them."""
    import torch
    base = synth.CONFIGS[name].scaled(**cfg)
    w = synth.generate(base)
    lo, hi = w["region"]
    P = oracle.Params()
    C_or = oracle.calib_counts(P, w)
    p_or = oracle.p_matrix(P, C_or)
    dev = {k: torch.from_numpy(np.ascontiguousarray(w[k])).cuda()
           for k in ("pos", "len", "off", "bases", "quals", "strand", "hits")}
    with gsnp.Context.from_workload(w, stream=torch.cuda.current_stream()) as ctx:
        counts = torch.zeros(64 * 256 * 16, dtype=torch.uint64, device="cuda")
        ctx.calibrate_count(dev, counts)
        assert np.array_equal(counts.cpu().numpy().reshape(64, 256, 4, 4), C_or)
        ctx.calibrate_finalize(counts)
        out = torch.empty(40 * (hi - lo), dtype=torch.uint8, device="cuda")
        ctx.call(dev, lo, hi, out)
        torch.cuda.synchronize()
        rec_g = out.cpu().numpy().view(gsnp.RECORD_DTYPE)
    assert np.array_equal(rec_g["pos"], np.arange(lo, hi, dtype=np.uint64))
    rng = np.random.default_rng(seed)
    S = hi - lo
    covered = np.nonzero(rec_g["depth"] > 0)[0]
    pick = np.unique(np.concatenate([rng.choice(S, n_sample // 2, replace=False),
                                     rng.choice(covered, n_sample // 2, replace=False),
                                     np.arange(0, 150), np.arange(S - 150, S)]))   # shard edges
    het = np.nonzero(np.isin(rec_g["genotype"], [1, 2, 3, 5, 6, 8]))[0]
    pick = np.unique(np.concatenate([pick, het[:200], np.argsort(rec_g["depth"])[-50:]]))
    recs, L10s = [], []
    for i in pick:
        s = lo + int(i)
        ra, rb = synth.read_range(w, s, s + 1)
        sub = synth.slice_reads(w, ra, rb)
        r, d = oracle.call_window(P, sub, p_or, s, s + 1, debug=True)
        recs.append(r)
        L10s.append(d["L10"])
    compare(w, rec_g[pick], np.concatenate(recs), np.concatenate(L10s))
    return len(pick)


def test_c3_shard_sampled():
    """C3: chr1-like 249 Mb at 30X, rank 3 of 8 (31 Mb shard with halos on both sides)."""
    n = synth.CONFIGS["C3"].n_sites
    assert _run_region("C3", 2000, 3, region_lo=3 * n // 8, region_hi=4 * n // 8) >= 2000


def test_c4_shard_sampled():
    """C4: whole-genome 3.1 Gb at 12.5X, a 48 Mb piece from the middle (rank 21 of 64)."""
    n = synth.CONFIGS["C4"].n_sites
    assert _run_region("C4", 2000, 4, region_lo=21 * n // 64, region_hi=22 * n // 64) >= 2000
