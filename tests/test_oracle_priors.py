"""Pins for the prior variants of reading R18 (P:L216 names only
"prior probability for known SNPs"): monoploid, transition:transversion 2:1, and known-SNP rows
from allele frequencies (Hardy-Weinberg).  Each is tied to a hand-written prior vector, a closed
form, or an algebraic identity — not to the oracle's own code."""
from __future__ import annotations

import math

import numpy as np
import pytest

import oracle
from tests._util import workload, rel_err
from tests.test_oracle_pins import _closed_form_workload

GT = oracle.GENOTYPES


def _depth0_post(P, ref_code):
    """Posterior at an uncovered site = the normalised prior (L10 = 0)."""
    ref = "ACTG"[ref_code] * 50
    w = workload(ref, [])
    p = oracle.p_matrix(P, np.zeros((64, 256, 4, 4), np.uint64))
    rec, dbg = oracle.call_window(P, w, p, 10, 11, debug=True)
    return rec[0], dbg["post10"][0]


def test_titv_prior_hand_values():
    """ref A: the transition allele is G (A<->G), transversions C and T.  Hand-written priors:
    A/G het 1e-3*2, A/C and A/T 1e-3/2, GG 5e-4*2, CC and TT 5e-4/2, alt hets 5e-7*w*w."""
    P = oracle.Params(titv=True)
    want = {"AA": 1.0, "AC": 5e-4, "AT": 5e-4, "AG": 2e-3, "CC": 2.5e-4, "CT": 5e-7 * 0.25,
            "CG": 5e-7 * 1.0, "TT": 2.5e-4, "TG": 5e-7 * 1.0, "GG": 1e-3}
    prior = np.array([want[g] for g in GT])
    rec, post = _depth0_post(P, 0)
    assert np.all(rel_err(post, prior / prior.sum()) < 1e-12)
    assert GT[rec["genotype"]] == "AA"


@pytest.mark.parametrize("ref_code", [0, 1, 2, 3])
def test_titv_keeps_mean_het_prior_and_ratio(ref_code):
    """Weights average 1 over the three alternative alleles (the total novel het and hom-alt
    mass is unchanged) and the transition allele carries 2/3 of it (ratio 2:1)."""
    _, p0 = _depth0_post(oracle.Params(), ref_code)
    _, p1 = _depth0_post(oracle.Params(titv=True), ref_code)
    r = ref_code
    het = [i for i, (a, b) in enumerate(zip(oracle.GA1, oracle.GA2)) if (a == r) != (b == r)]
    hom = [i for i, (a, b) in enumerate(zip(oracle.GA1, oracle.GA2)) if a == b != r]
    ref_i = [i for i, (a, b) in enumerate(zip(oracle.GA1, oracle.GA2)) if a == b == r][0]
    # compare relative to the ref-hom entry (the normalisation differs only via alt-alt hets)
    for idx in (het, hom):
        m0 = sum(p0[i] / p0[ref_i] for i in idx)
        m1 = sum(p1[i] / p1[ref_i] for i in idx)
        assert abs(m1 - m0) <= 1e-12 * m0
        ti = [i for i in idx if (oracle.GA1[i] ^ r) == 3 or (oracle.GA2[i] ^ r) == 3][0]
        assert abs((p1[ti] / p1[ref_i]) / m1 - 2.0 / 3.0) < 1e-12


def test_monoploid_prior_and_closed_form_call():
    """Monoploid: het priors are 0; at a depth-0 site the posterior is (1, a, a, a)/(1+3a) on the
    homozygotes.  The closed-form site of test_closed_form_uniform_quality (8 A + 2 G at q30,
    diploid call AG) becomes AA; Δ = L(AA) - L(GG) - log10(5e-4) and the hom cap
    q_sum(A) - q_sum(G) = 240 - 60 -> quality min(int(10Δ), 180) clamped to 99."""
    P = oracle.Params(monoploid=True)
    rec, post = _depth0_post(P, 2)
    a = 5e-4
    want = np.array([a if g in ("AA", "CC", "GG") else 1.0 if g == "TT" else 0.0 for g in GT])
    assert np.all(np.abs(post - want / want.sum()) < 1e-15)
    assert GT[rec["genotype"]] == "TT"
    P1 = oracle.Params(global_dep=1.0, pcr_dep=1.0, monoploid=True)
    w = _closed_form_workload()
    p = oracle.p_matrix(P1, np.zeros((64, 256, 4, 4), np.uint64))
    rec, dbg = oracle.call_window(P1, w, p, 150, 151, debug=True)
    e = 1e-3
    LAA = 8 * math.log10(1 - e) + 2 * math.log10(e / 3)
    LGG = 8 * math.log10(e / 3) + 2 * math.log10(1 - e)
    delta = LAA - (LGG + math.log10(5e-4))
    assert GT[rec["genotype"][0]] == "AA"
    assert rec["quality"][0] == max(0, min(99, min(int(10 * delta), 240 - 60)))
    het = [i for i, (x, y) in enumerate(zip(oracle.GA1, oracle.GA2)) if x != y]
    assert np.all(dbg["post10"][0][het] == 0.0)
    assert abs(dbg["post10"][0].sum() - 1) < 1e-12


def test_monoploid_zeroes_known_rows_too():
    ref = "A" * 300
    reads = [dict(pos=100, strand=0, hits=1, bases="A" * 50 + "C" + "A" * 49, quals=30)
             for _ in range(3)] + \
            [dict(pos=100, strand=1, hits=1, bases="A" * 100, quals=30) for _ in range(3)]
    w = workload(ref, reads, known=[(150, [0.5] + [0.05] * 9)])
    for mono in (False, True):
        P = oracle.Params(monoploid=mono)
        p = oracle.p_matrix(P, np.zeros((64, 256, 4, 4), np.uint64))
        rec, dbg = oracle.call_window(P, w, p, 150, 151, debug=True)
        g = GT[rec["genotype"][0]]
        assert (g[0] == g[1]) if mono else g == "AC"


def test_priors_from_freq_hardy_weinberg():
    """Rows sum to (Σf)^2 = 1 when no entry is floored; hand values for f = (.6, .1, 0, .3)."""
    rng = np.random.default_rng(4)
    f = rng.random((50, 4)) + 0.05
    pr = oracle.priors_from_freq(f, 1e-12)
    assert np.all(np.abs(pr.sum(1) - 1) < 1e-12)
    pr = oracle.priors_from_freq([[6, 1, 0, 3]], 1e-6)[0]      # unnormalised input
    want = {"AA": .36, "AC": .12, "AT": 1e-6, "AG": .36, "CC": .01, "CT": 1e-6, "CG": .06,
            "TT": 1e-6, "TG": 1e-6, "GG": .09}
    assert np.all(rel_err(pr, [want[g] for g in GT]) < 1e-12)
    with pytest.raises(ValueError):
        oracle.priors_from_freq([[0, 0, 0, 0]])
    with pytest.raises(ValueError):
        oracle.priors_from_freq([[1, -1, 0, 0]])
