"""GPU parity for the prior variants (reading R18): monoploid and
ti/tv 2:1 novel priors, and known-SNP rows from allele frequencies — CUDA path vs the oracle."""
from __future__ import annotations

import numpy as np
import pytest

import oracle
import synth
from paper_conf_icpp_luzlwfl11_b200 import gsnp
from tests._parity import compare

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("mono,titv", [(True, False), (False, True), (True, True)])
def test_prior_variants_parity(mono, titv):
    w = synth.generate("C1", n_sites=8_000, depth=12.0, seed=41)
    P = oracle.Params(monoploid=mono, titv=titv)
    C = oracle.calib_counts(P, w)
    p = oracle.p_matrix(P, C)
    rec_o, dbg = oracle.call_window(P, w, p, 0, 8_000, debug=True)
    flags = gsnp.GSNP_RANK_SUM | (gsnp.GSNP_MONOPLOID if mono else 0) | (gsnp.GSNP_TITV if titv else 0)
    with gsnp.Context.from_workload(w, flags=flags) as ctx:
        ctx.calibrate(w)
        rec_g = ctx.call(w, 0, 8_000)
        dg = ctx.debug_window(w, 0, 8_000)
        rec_d = ctx.call_dense(w, 0, 8_000, chunk_sites=2048)
    assert rec_g.tobytes() == dg["records"].tobytes() == rec_d.tobytes()
    # L10 is prior-free: bit-exact; then the north_star rules of tests/_parity.compare with the
    # variant's prior rows (posteriors within 1e-9 relative; genotype and quality exact unless a
    # near tie or 10Δ + 10 log10(rank_p) within 1e-6 of an integer, each such site justified)
    assert np.array_equal(dg["L10"], dbg["L10"])
    rep = compare(w, rec_g, rec_o, dbg["L10"], dbg["post10"], dg["L10"], dg["post10"], P=P)
    assert rep["near_tie"] + rep["near_int"] <= 2
    if mono:
        assert not np.isin(rec_g["genotype"], [1, 2, 3, 5, 6, 8]).any()


def test_priors_from_freq_library_equals_oracle_and_calls():
    rng = np.random.default_rng(7)
    f = rng.dirichlet(np.ones(4) * 0.3, 500)
    f[::7, 1] = 0.0
    assert np.array_equal(gsnp.gsnp_priors_from_freq(f, 5e-7), oracle.priors_from_freq(f, 5e-7))
    with pytest.raises(gsnp.GsnpError):
        gsnp.gsnp_priors_from_freq([[0.0, 0, 0, 0]])
    # known-SNP rows from frequencies drive the call like any caller-supplied prior10
    w = synth.generate("C1", n_sites=6_000, depth=10.0, seed=43)
    kp = np.asarray(w["known_pos"], np.uint64)
    freq = rng.dirichlet(np.ones(4), len(kp))
    w = dict(w, known_prior10=gsnp.gsnp_priors_from_freq(freq))
    P = oracle.Params()
    p = oracle.p_matrix(P, oracle.calib_counts(P, w))
    rec_o, dbg = oracle.call_window(P, w, p, 0, 6_000, debug=True)
    with gsnp.Context.from_workload(w) as ctx:
        ctx.calibrate(w)
        rec_g = ctx.call(w, 0, 6_000)
    compare(w, rec_g, rec_o, dbg["L10"])


@pytest.mark.parametrize("depth", [6.0, 12.0])
def test_rank_exact_parity(depth):
    """R20: exact small-sample rank-sum table in every call path vs the
    oracle's subset-count definition; het-rich input so the exact branch decides many sites."""
    w = synth.generate("C1", n_sites=8_000, depth=depth, seed=47, het_rate=0.05)
    P = oracle.Params(rank_exact=True)
    p = oracle.p_matrix(P, oracle.calib_counts(P, w))
    rec_o, dbg = oracle.call_window(P, w, p, 0, 8_000, debug=True)
    rec_n = oracle.call_window(oracle.Params(), w, p, 0, 8_000)
    assert (rec_o["rank_p"] != rec_n["rank_p"]).sum() >= 20       # the exact branch is exercised
    with gsnp.Context.from_workload(w, flags=gsnp.GSNP_RANK_SUM | gsnp.GSNP_RANK_EXACT) as ctx:
        ctx.calibrate(w)
        rec_g = ctx.call(w, 0, 8_000)
        dg = ctx.debug_window(w, 0, 8_000)
        rec_d = ctx.call_dense(w, 0, 8_000, chunk_sites=2048)
    assert rec_g.tobytes() == dg["records"].tobytes() == rec_d.tobytes()
    compare(w, rec_g, rec_o, dbg["L10"])


def test_rank_exact_needs_rank_sum():
    """R20 refines R8's p-value only: GSNP_RANK_EXACT without GSNP_RANK_SUM applies no test."""
    w = synth.generate("C1", n_sites=4_000, depth=6.0, seed=48, het_rate=0.05)
    P = oracle.Params(rank_sum=False, rank_exact=True)
    p = oracle.p_matrix(P, oracle.calib_counts(P, w))
    rec_o, dbg = oracle.call_window(P, w, p, 0, 4_000, debug=True)
    with gsnp.Context.from_workload(w, flags=gsnp.GSNP_RANK_EXACT) as ctx:
        ctx.calibrate(w)
        rec_g = ctx.call(w, 0, 4_000)
    assert np.all(rec_g["rank_p"] == 1.0)
    compare(w, rec_g, rec_o, dbg["L10"])
