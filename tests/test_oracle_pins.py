"""Pins for the CPU oracle (-m "not gpu").  Each test ties the oracle to something other than
itself: a value printed in PAPER.md, a closed form, a library routine (scipy, Python's exact
rationals), a brute-force recount, or a second algorithm the paper gives (Alg. 1 vs Alg. 4)."""
from __future__ import annotations

import math
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
import synth
from tests._util import workload, site_columns, rel_err

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _gold_rows(name):
    rows = []
    with open(os.path.join(GOLD, name)) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                rows.append(line.split())
    return rows


# ---------------------------------------------------------------- C2: keys (Fig. 3)
def test_fig3_keys_and_canonical_order():
    rows = _gold_rows("fig3_base_word.txt")
    obs = [r for r in rows if r[0] != "order"]
    order = [int(x) for x in [r for r in rows if r[0] == "order"][0][1:]]
    keys = []
    for b, s, c, st, kp, ki in obs:
        b, s, c, st = int(b), int(s), int(c), int(st)
        assert oracle.key_paper(b, s, c, st) == int(kp)
        assert oracle.key(b, s, c, st) == int(ki)
        keys.append(oracle.key(b, s, c, st))
    assert list(np.argsort(keys, kind="stable")) == order


def test_key_sort_matches_alg1_loop_nest():
    """Ascending key order == Alg. 1 l.2-6 nest: base 0..3, score high..low, coord, strand."""
    rng = np.random.default_rng(7)
    t = [(int(rng.integers(4)), int(rng.integers(64)), int(rng.integers(256)), int(rng.integers(2)))
         for _ in range(500)]
    by_key = sorted(t, key=lambda x: oracle.key(*x))
    by_nest = sorted(t, key=lambda x: (x[0], -x[1], x[2], x[3]))
    assert by_key == by_nest


# ---------------------------------------------------------------- C3: adjust
def test_adjust_identity_when_coefficients_are_one():
    P = oracle.Params(global_dep=1.0, pcr_dep=1.0)
    for q in range(64):
        for pcr in (1, 2, 5):
            for g in (0, 3, 40):
                assert oracle.adjust(P, q, pcr, g) == max(1, q)


def test_adjust_matches_multiplicative_closed_form_off_ties():
    """q_adj = round(q * pcr_dep^(pcr-1) * global_dep^g), floor 1.  The log/pow evaluation may
    differ from the product form only where the product sits on an exact .5 boundary (25 cells
    at the default coefficients), e.g. q=11, pcr=2: 5.5 -> 5."""
    P = oracle.Params()
    diff = []
    for q in range(64):
        for pcr in range(1, 9):
            for g in range(64):
                x = Fraction(q) * Fraction(1, 2) ** (pcr - 1) * Fraction(9, 10) ** g
                want = max(1, math.floor(x + Fraction(1, 2)))
                got = oracle.adjust(P, q, pcr, g)
                if got != want:
                    diff.append((q, pcr, g))
                    assert x.denominator != 1 and (x - Fraction(1, 2)).denominator == 1 or \
                        (x + Fraction(1, 2)) == math.floor(x + Fraction(1, 2)), (q, pcr, g, x)
                    assert got == want - 1
    assert len(diff) == 25
    assert (11, 2, 0) in diff and oracle.adjust(P, 11, 2, 0) == 5


def test_adjust_saturation_and_monotone():
    P = oracle.Params()
    for q in range(64):
        for g in range(36, 80):
            assert oracle.adjust(P, q, 1, g) == 1
        for pcr in range(7, 20):
            assert oracle.adjust(P, q, pcr, 0) == 1
        for pcr in range(1, 8):
            row = [oracle.adjust(P, q, pcr, g) for g in range(64)]
            assert all(a >= b for a, b in zip(row, row[1:]))
    assert oracle.adjust(P, 63, 1, 35) == 2


# ---------------------------------------------------------------- C4/C5: likelihood
def _random_p(rng):
    """A random valid p matrix: for each (q, coord, allele) a probability vector over base."""
    p = rng.dirichlet(np.ones(4) * 0.7, size=(64, 256, 4))
    p = np.maximum(p, 1e-12)
    return p / p.sum(-1, keepdims=True)


def _random_site(rng, n, L=100, q_max=40):
    b = rng.choice(4, n, p=[0.7, 0.1, 0.1, 0.1])
    q = rng.integers(0, q_max + 1, n)
    c = rng.integers(0, min(L, 12), n)       # few coords -> repeated (strand, coord) slots
    s = rng.integers(0, 2, n)
    dup = rng.random(n) < 0.2                # exact duplicate tuples
    for i in np.nonzero(dup)[0]:
        if i:
            b[i], q[i], c[i], s[i] = b[i - 1], q[i - 1], c[i - 1], s[i - 1]
    return b, q, c, s


@pytest.mark.parametrize("seed", range(12))
def test_dense_alg1_equals_sparse_alg4(seed):
    """the sparse representation + sort reproduces Alg. 1 exactly."""
    rng = np.random.default_rng(seed)
    P = oracle.Params()
    p = _random_p(rng)
    n = int(rng.integers(0, 80))
    b, q, c, s = _random_site(rng, n)
    Ls, keys = oracle.sparse_likelihood(P, p, b, q, c, s)
    Ld = oracle.dense_likelihood(P, p, b, q, c, s)
    assert np.array_equal(Ls, Ld)             # same terms in the same order: bit-identical
    want = sorted(oracle.key(int(x), int(y), int(z), int(w)) for x, y, z, w in zip(b, q, c, s))
    assert list(keys) == want


@pytest.mark.parametrize("seed", range(8))
def test_log_sum_equals_log_of_exact_product(seed):
    """L[n] = log10 prod_k (0.5 p[q,c,a1,b] + 0.5 p[q,c,a2,b]) — exact rational product."""
    rng = np.random.default_rng(100 + seed)
    P = oracle.Params(global_dep=1.0, pcr_dep=1.0)   # adjust = identity (q >= 1)
    p = _random_p(rng)
    n = int(rng.integers(1, 12))
    b, q, c, s = _random_site(rng, n)
    q = np.maximum(q, 1)
    L10, _ = oracle.sparse_likelihood(P, p, b, q, c, s)
    for g in range(10):
        a1, a2 = oracle.GA1[g], oracle.GA2[g]
        prod = Fraction(1)
        for k in range(n):
            prod *= Fraction(0.5) * Fraction(p[q[k], c[k], a1, b[k]]) + \
                Fraction(0.5) * Fraction(p[q[k], c[k], a2, b[k]])
        exact = math.log10(prod.numerator) - math.log10(prod.denominator)
        assert abs(L10[g] - exact) <= 1e-12 * max(1.0, abs(exact))


def _closed_form_workload():
    ref = "A" * 300
    reads = []
    for i in range(10):                       # cycles 0..9 at site 150 (strand 0)
        bases = ["A"] * 100
        bases[i] = "G" if i >= 8 else "A"
        reads.append(dict(pos=150 - i, strand=0, hits=1, bases="".join(bases), quals=30))
    return workload(ref, reads)


def test_closed_form_uniform_quality():
    rows = _gold_rows("closed_form_uniform_q30.txt")
    gold = {r[0]: float(r[1]) for r in rows if r[0] != "call"}
    call = [r for r in rows if r[0] == "call"][0]
    e = 1e-3
    formula = {"AA": 8 * math.log10(1 - e) + 2 * math.log10(e / 3),
               "AG": 10 * math.log10(0.5 * (1 - e) + 0.5 * e / 3),
               "GG": 8 * math.log10(e / 3) + 2 * math.log10(1 - e),
               "CC": 10 * math.log10(e / 3)}
    for k in gold:
        assert abs(formula[k] - gold[k]) < 1e-11
    P = oracle.Params(global_dep=1.0, pcr_dep=1.0)
    w = _closed_form_workload()
    C = oracle.calib_counts(P, dict(w, pos=w["pos"][:0], len=w["len"][:0], off=w["off"][:1],
                                    strand=w["strand"][:0], hits=w["hits"][:0]))
    assert C.sum() == 0
    p = oracle.p_matrix(P, C)
    rec, dbg = oracle.call_window(P, w, p, 150, 151, debug=True)
    L10 = dbg["L10"][0]
    for k, v in formula.items():
        assert abs(L10[oracle.GENOTYPES.index(k)] - v) <= 1e-12 * abs(v)
    assert oracle.GENOTYPES[rec["genotype"][0]] == call[1]
    assert rec["quality"][0] == int(call[2])
    assert rec["rank_p"][0] == 1.0
    assert rec["base1"][0] == 0 and rec["base2"][0] == 3


# ---------------------------------------------------------------- C7: posterior
def test_posterior_sums_to_one_and_depth0_is_prior():
    w = synth.generate("C1")
    P = oracle.Params()
    p = oracle.p_matrix(P, oracle.calib_counts(P, w))
    rec, dbg = oracle.call_window(P, w, p, 0, 10_000, debug=True)
    s = dbg["post10"].sum(1)
    assert np.all(np.abs(s - 1) < 1e-12)
    d0 = np.nonzero(rec["depth"] == 0)[0]
    assert len(d0) > 0
    for i in d0[:50]:
        r = int(w["ref"][i])
        if r == 4:
            assert rec["genotype"][i] == 255
            continue
        assert rec["genotype"][i] == oracle.GENOTYPES.index("AACCTTGG"[2 * r:2 * r + 2])
        assert rec["quality"][i] == 0
        prior = np.array([1.0 if (a == r and b == r) else 1e-3 if (a == r or b == r) else
                          5e-4 if a == b else 5e-7 for a, b in zip(oracle.GA1, oracle.GA2)])
        assert np.all(rel_err(dbg["post10"][i], prior / prior.sum()) < 1e-12)


# ---------------------------------------------------------------- C8: rank-sum
def test_rank_sum_matches_scipy_asymptotic():
    from scipy.stats import mannwhitneyu
    rng = np.random.default_rng(3)
    for _ in range(40):
        n1, n2 = int(rng.integers(1, 40)), int(rng.integers(1, 40))
        X = rng.integers(2, 41, n1)
        Y = rng.integers(2, 41, n2)
        if len(set(X) | set(Y)) == 1:
            continue
        want = mannwhitneyu(X, Y, alternative="two-sided", use_continuity=False,
                            method="asymptotic").pvalue
        assert abs(oracle.rank_sum(X, Y) - want) <= 1e-12 * max(want, 1e-300) + 1e-15


def test_rank_sum_special_cases():
    assert oracle.rank_sum([30, 31, 32], [30, 31, 32]) == 1.0          # W == mu
    assert oracle.rank_sum([30] * 5, [30] * 4) == 1.0                   # all tied: var = 0
    assert oracle.rank_sum([], [30]) == 0.0 and oracle.rank_sum([30], []) == 0.0
    # disjoint ranges: textbook normal approximation, no ties within either side
    X, Y = list(range(10, 20)), list(range(30, 40))
    n1 = n2 = 10
    W = sum(range(1, 11))
    z = (W - n1 * (n1 + n2 + 1) / 2) / math.sqrt(n1 * n2 * (n1 + n2 + 1) / 12)
    assert abs(oracle.rank_sum(X, Y) - math.erfc(abs(z) / math.sqrt(2))) < 1e-15


# R20: exact small-sample rank-sum
def test_rank_sum_exact_matches_scipy_exact():
    from scipy.stats import mannwhitneyu
    rng = np.random.default_rng(5)
    for _ in range(60):
        n1, n2 = int(rng.integers(1, 33)), int(rng.integers(1, 33))
        v = rng.permutation(np.arange(2, 2 + n1 + n2 + int(rng.integers(0, 20))))  # no ties
        X, Y = v[:n1], v[n1:n1 + n2]
        want = mannwhitneyu(X, Y, alternative="two-sided", method="exact").pvalue
        assert abs(oracle.rank_sum_exact(X, Y) - want) <= 1e-12 * want + 1e-300


def test_rank_sum_exact_closed_forms_and_fallbacks():
    # n1 = 1: U is uniform on 0..n2, so P(U <= u) = (u+1)/(n2+1)
    for n2 in (1, 5, 32):
        for rank in range(1, n2 + 2):                       # rank of the single X among N
            Y = [q for q in range(10, 10 + n2 + 1) if q != 9 + rank]
            u = rank - 1
            want = min(1.0, 2 * min(u + 1, n2 + 1 - u) / (n2 + 1))
            assert abs(oracle.rank_sum_exact([9 + rank], Y) - want) < 1e-15
    # complete separation of n1 = n2 = 10: one of C(20,10) rank sets at each extreme
    assert abs(oracle.rank_sum_exact(range(10, 20), range(30, 40)) - 2 / math.comb(20, 10)) < 1e-20
    # brute force over all n1-subsets for small N
    import itertools
    X, Y = [3, 17, 8, 25], [11, 2, 30, 14, 6]
    ranks = {q: r + 1 for r, q in enumerate(sorted(X + Y))}
    W = sum(ranks[q] for q in X)
    sums = [sum(c) for c in itertools.combinations(range(1, 10), 4)]
    le, ge = sum(s <= W for s in sums), sum(s >= W for s in sums)
    assert abs(oracle.rank_sum_exact(X, Y) - min(1, 2 * min(le, ge) / len(sums))) < 1e-15
    # ties or a group above 32 -> the normal approximation of R8; empty group -> 0
    assert oracle.rank_sum_exact([30, 31, 32], [30, 33]) == oracle.rank_sum([30, 31, 32], [30, 33])
    big = list(range(2, 35))
    assert oracle.rank_sum_exact(big, [40]) == oracle.rank_sum(big, [40])
    assert oracle.rank_sum_exact([], [30]) == 0.0


# ---------------------------------------------------------------- C0 / C1: counting
def test_site_counters_match_bruteforce_recount():
    w = synth.generate("C1")
    P = oracle.Params()
    p = oracle.p_matrix(P, oracle.calib_counts(P, w))
    rec, dbg = oracle.call_window(P, w, p, 0, 10_000, debug=True)
    bf = site_columns(w, 0, 10_000)
    c = dbg["counters"]
    assert np.array_equal(c[:, 0], bf["depth"])
    assert np.array_equal(c[:, 1], bf["dep_uni"])
    assert np.array_equal(c[:, 2], bf["repeat"])
    assert np.array_equal(c[:, 3:7], bf["count_all"])
    assert np.array_equal(c[:, 7:11], bf["count_uni"])
    assert np.array_equal(c[:, 11:15], bf["q_sum"])
    assert np.array_equal(np.diff(dbg["off"].astype(np.int64)), bf["dep_uni"])
    assert np.array_equal(rec["depth"], bf["depth"])
    assert dbg["off"][-1] == bf["dep_uni"].sum()


def test_calibration_counts_bruteforce_and_estimator_invariants():
    w = synth.generate("C1")
    P = oracle.Params()
    C = oracle.calib_counts(P, w)
    # brute force (numpy): unique reads, non-N base, non-N ref, not a known SNP
    ln = w["len"].astype(np.int64)
    rid = np.repeat(np.arange(len(ln)), ln)
    i = np.arange(len(rid)) - np.repeat(w["off"][:-1].astype(np.int64), ln)
    site = w["pos"].astype(np.int64)[rid] + i
    st = w["strand"][rid].astype(np.int64)
    cyc = np.where(st == 1, ln[rid] - 1 - i, i)
    t = w["ref"][site].astype(np.int64)
    o = w["bases"].astype(np.int64)
    q = w["quals"].astype(np.int64)
    m = (w["hits"][rid] == 1) & (o < 4) & (t < 4) & ~np.isin(site, w["known_pos"].astype(np.int64))
    bf = np.zeros(64 * 256 * 16, np.int64)
    np.add.at(bf, q[m] << 12 | cyc[m] << 4 | t[m] << 2 | o[m], 1)
    assert np.array_equal(C.reshape(-1).astype(np.int64), bf)
    p = oracle.p_matrix(P, C)
    L = P.max_read_len
    assert np.all(p[:, :L] > 0) and np.all(p[:, :L] <= 1)


def test_estimator_rules_on_constructed_counts():
    """Reading R1, rule by rule, on a hand-made count matrix."""
    P = oracle.Params()
    tau = P.calib_min_count
    rng = np.random.default_rng(2)
    C = np.zeros((64, 256, 4, 4), np.uint64)
    C[30, :100] = rng.integers(tau + 1, 1000, (100, 4, 4))          # q30: rule 1 everywhere
    C[20, :100, :, :] = 0
    C[20, :100, 0, 0] = 50                                          # q20: diagonal-only for t=A
    C[20, 7, 0, 1] = 3                                              #   a few mismatches (pool=3)
    C[25, 0, 1, 1] = 5                                              # q25: tiny -> rule 3
    C[25, 0, 1, 2] = 1
    p = oracle.p_matrix(P, C)
    # rule 1: rows sum to 1, p = n / N_ct
    assert np.all(np.abs(p[30, :100].sum(-1) - 1) < 1e-12)
    assert p[30, 3, 2, 1] == C[30, 3, 2, 1] / C[30, 3, 2].sum()
    # rule 1 on the q20 diagonal; rule 2 (pooled over cycles) for A->A where n <= tau? n=50 > tau
    assert p[20, 7, 0, 0] == 50 / 53
    # q20 A->C: n = 3 <= tau at cycle 7 and pooled 3 <= tau -> rule 3: mm/(3 tot)
    tot = 50 * 100 + 3
    assert p[20, 7, 0, 1] == 3 / (3 * tot)
    assert p[20, 5, 2, 2] == (tot - 3) / tot                        # no T data at all: rule 3
    # q25: tot = 6, mm = 1 -> rule 3
    assert p[25, 0, 1, 2] == 1 / (3 * 6) and p[25, 0, 1, 1] == 5 / 6
    # q10: no data -> rule 4 theoretical value
    e = 10 ** -1.0
    assert p[10, 0, 0, 0] == 1 - e and p[10, 0, 0, 1] == e / 3
    assert p[0, 0, 0, 0] == 0.25 and p[0, 0, 0, 3] == 0.25           # e capped at 0.75
    assert np.all(p[:, :100] > 0) and np.all(p[:, :100] <= 1)


def test_calibration_error_free_reads_are_diagonal():
    rng = np.random.default_rng(5)
    ref = rng.integers(0, 4, 400).astype(np.uint8)
    reads = [dict(pos=int(s), strand=int(rng.integers(2)), hits=1,
                  bases=list(ref[s:s + 100]), quals=int(rng.integers(2, 41)))
             for s in sorted(rng.integers(0, 300, 60))]
    w = workload(ref, reads)
    P = oracle.Params()
    C = oracle.calib_counts(P, w)
    off = C.copy()
    for t in range(4):
        off[:, :, t, t] = 0
    assert off.sum() == 0 and C.sum() == 6000


def test_calibration_recovers_error_rate():
    """Off-diagonal pooled probability ~ e/3 at the generated error rate 10^(-q/10)."""
    w = synth.generate("C1", n_sites=200_000, depth=20.0, seed=11, het_rate=0.0, hom_rate=0.0)
    P = oracle.Params()
    C = oracle.calib_counts(P, w).astype(np.float64)
    for q in (30, 35, 40):
        tot = C[q].sum()
        mm = tot - sum(C[q, :, t, t].sum() for t in range(4))
        e = 10 ** (-q / 10)
        sd = math.sqrt(tot * e) / tot
        assert abs(mm / tot - e) < 5 * sd + 1e-6, (q, mm / tot, e)


# ---------------------------------------------------------------- C9: consensus quality
def test_quality_cases_hand_computed():
    P = oracle.Params()
    p = oracle.p_matrix(P, np.zeros((64, 256, 4, 4), np.uint64))   # theoretical p (rule 4)
    ref = "A" * 300
    # (a) deep hom-ref: raw quality > 99 -> clamp 99
    reads = [dict(pos=100 + i, strand=0, bases="A" * 100, quals=40) for i in range(30)]
    # (b) one low-quality C read at site 250 (ref A): called AA, base1 = C != A -> quality 0
    reads += [dict(pos=200, strand=1, bases="A" * 50 + "C" + "A" * 49, quals=[2] * 100)]
    w = workload(ref, reads)
    rec = oracle.call_window(P, w, p, 0, 300)
    assert rec["genotype"][129] == 0 and rec["quality"][129] == 99
    r = rec[250]
    assert r["base1"] == 1 and r["base2"] == 0 and r["genotype"] == 0 and r["quality"] == 0
    # (c) het site, hand-computed with adjust = identity (coefficients 1, reading R3):
    #     3 A + 3 G at q35, distinct cycles; ref A -> AG; rank-sum all tied -> rank_p = 1;
    #     raw quality (int)(10 (lp1 - lp2)), het cap = min(q_sum[A], q_sum[G]) = 105
    P1 = oracle.Params(global_dep=1.0, pcr_dep=1.0)
    reads = [dict(pos=10 + k, strand=0, bases="A" * 100 if k < 3 else
                  "A" * (40 - k) + "G" + "A" * (59 + k), quals=35) for k in range(6)]
    w = workload(ref, reads)
    rec = oracle.call_window(P1, w, p, 50, 51)
    lp = {}
    for g, name in enumerate(oracle.GENOTYPES):
        a1, a2 = oracle.GA1[g], oracle.GA2[g]
        prior = 1.0 if name == "AA" else 1e-3 if "A" in name else 5e-4 if name[0] == name[1] \
            else 5e-7
        lp[name] = 3 * math.log10(0.5 * p[35, 0, a1, 0] + 0.5 * p[35, 0, a2, 0]) + \
            3 * math.log10(0.5 * p[35, 0, a1, 3] + 0.5 * p[35, 0, a2, 3]) + math.log10(prior)
    top = sorted(lp, key=lambda n: -lp[n])
    assert top[0] == "AG" and oracle.GENOTYPES[rec["genotype"][0]] == "AG"
    want = min(int(10 * (lp["AG"] - lp[top[1]])), 105)
    assert rec["quality"][0] == max(0, min(99, want))
    assert rec["rank_p"][0] == 1.0
    assert (rec["cnt_uni1"][0], rec["cnt_uni2"][0], rec["avgq1"][0]) == (3, 3, 35)
    # (d) known-SNP prior forces a het call whose second allele is unseen -> quality 0
    kp = [0.0] * 10
    kp[oracle.GENOTYPES.index("AA")] = 1e-6
    kp[oracle.GENOTYPES.index("AG")] = 1.0
    kp = [x if x else 1e-9 for x in kp]
    w = workload(ref, [dict(pos=20, strand=0, bases="A" * 100, quals=10)], known=[(50, kp)])
    rec = oracle.call_window(P1, w, p, 50, 51)
    assert oracle.GENOTYPES[rec["genotype"][0]] == "AG" and rec["known"][0] == 1
    assert rec["quality"][0] == 0 and rec["rank_p"][0] == 0.0


# ---------------------------------------------------------------- hand-computed pins (round 2)
def _theory_p(q, a, o):
    """Rule 4 of the estimator (R1) — what calibrating on no reads yields: e = min(.75, 10^-q/10)."""
    e = min(0.75, 10 ** (-q / 10))
    return 1 - e if a == o else e / 3


def _hand_L10(obs):
    """Alg. 2 per observation, summed in the given order: obs = [(q_adj, base)]."""
    out = []
    for n in range(10):
        a1, a2 = oracle.GA1[n], oracle.GA2[n]
        s = 0.0
        for qa, b in obs:
            s += math.log10(0.5 * _theory_p(qa, a1, b) + 0.5 * _theory_p(qa, a2, b))
        out.append(s)
    return np.array(out)


def _site_reads(site, specs, L=100):
    """Reads of length L covering `site`: specs = [(pos, strand, base_at_site, q_at_site)]; every
    other base matches the all-A reference."""
    reads = []
    for pos, st, b, q in specs:
        bases = ["A"] * L
        bases[site - pos] = b
        quals = [30] * L
        quals[site - pos] = q
        reads.append(dict(pos=pos, strand=st, bases="".join(bases), quals=quals))
    return reads


def test_dependency_counters_hand_computed_default_coefficients():
    """pcr and g of Alg. 4 l.8-12 under reading R3 at the default 0.5 / 0.9, written
    out by hand.  Site 50, reference A.  Six A keys at q30 on '+': reads at 43, 42, 41 give cycles
    7, 8, 9 (distinct (strand, coord) slots) and three reads at 40 share cycle 10 (PCR duplicates).
    Canonical order is cycle 7, 8, 9, 10, 10, 10, so (pcr, g) = (1,0) (1,1) (1,2) (1,3) (2,3) (3,3)
    and q_adj = round(30 * .5^(pcr-1) * .9^g) = 30, 27, 24 (24.3), 22 (21.87), 11 (10.935),
    5 (5.4675).  Two G keys at q20 on '-' (reads at 45 and 46: cycles 99-5 = 94 and 95) restart the
    counters for the new base (l.8-11): g = 0, 1 -> 20, 18."""
    site = 50
    specs = [(40, 0, "A", 30)] * 3 + [(41, 0, "A", 30), (42, 0, "A", 30), (43, 0, "A", 30),
                                      (45, 1, "G", 20), (46, 1, "G", 20)]
    w = workload("A" * 200, _site_reads(site, specs))
    P = oracle.Params()
    p = oracle.p_matrix(P, np.zeros((64, 256, 4, 4), np.uint64))
    rec, dbg = oracle.call_window(P, w, p, site, site + 1, debug=True)
    q_adj_A = [30, 27, 24, 22, 11, 5]
    q_adj_G = [20, 18]
    want = _hand_L10([(q, 0) for q in q_adj_A] + [(q, 3) for q in q_adj_G])
    assert np.all(np.abs(dbg["L10"][0] - want) <= 1e-12 * np.abs(want))
    # the pin separates the plausible misreadings: g counted before the increment, g not reset per
    # base, pcr ignored, and adjust without the 0.5 rounding
    wrong = {
        "g_before_increment": [30, 30, 27, 24, 11, 5],
        "no_pcr": [30, 27, 24, 22, 22, 22],
        "truncate": [30, 27, 24, 21, 10, 5],
    }
    for name, seq in wrong.items():
        alt = _hand_L10([(q, 0) for q in seq] + [(q, 3) for q in q_adj_G])
        assert np.max(np.abs(alt - dbg["L10"][0]) / np.abs(want)) > 1e-6, name
    alt = _hand_L10([(q, 0) for q in q_adj_A] + [(q, 3) for q in (16, 15)])   # g carried over
    assert np.max(np.abs(alt - dbg["L10"][0]) / np.abs(want)) > 1e-6
    # the same counters drive the dense Alg. 1 walk (C5)
    L_dense = oracle.dense_likelihood(P, p, [0] * 6 + [3] * 2, [30] * 6 + [20] * 2,
                                      [10, 10, 10, 9, 8, 7, 94, 95], [0] * 6 + [1] * 2)
    assert np.all(np.abs(L_dense - want) <= 1e-12 * np.abs(want))


def _hand_quality(obs_raw, ref, rank_sum_p=1.0):
    """Raw consensus quality (C9 step 2) with identity adjust: int(10 (lp1 - lp2) + 10 log10 p)."""
    L = _hand_L10(obs_raw)
    pri = []
    for n in range(10):
        a1, a2 = oracle.GA1[n], oracle.GA2[n]
        v = 1.0 if (a1 == ref and a2 == ref) else 1e-3 if (a1 == ref or a2 == ref) else \
            5e-4 if a1 == a2 else 5e-7
        pri.append(math.log10(v))
    lp = L + np.array(pri)
    o = np.argsort(-lp, kind="stable")
    return int(o[0]), int(10 * (lp[o[0]] - lp[o[1]]) + 10 * math.log10(rank_sum_p))


def test_quality_caps_bind_below_99():
    """C9 steps 3-4 where the caps decide the quality (the earlier cases never bind below 99).
    Identity adjust (coefficients 1, R3) and theoretical p, so each raw quality is a hand sum.
    Hom: 3 A at q12 + 1 C at q2 on distinct cycles, ref A -> AA, raw 37 > cap
    q_sum[A] - q_sum[C] = 36 - 2 = 34.  Het (rank-sum off): 8 A at q8 + 3 G at q40, ref A -> AG,
    raw 68 > cap min(q_sum[A], q_sum[G]) = min(64, 120) = 64."""
    site = 50
    P1 = oracle.Params(global_dep=1.0, pcr_dep=1.0)
    p = oracle.p_matrix(P1, np.zeros((64, 256, 4, 4), np.uint64))
    specs = [(40 + k, 0, "A", 12) for k in range(3)] + [(44, 0, "C", 2)]
    w = workload("A" * 200, _site_reads(site, specs))
    t1, raw = _hand_quality([(12, 0)] * 3 + [(2, 1)], 0)
    assert (t1, raw) == (0, 37)
    r = oracle.call_window(P1, w, p, site, site + 1)[0]
    assert (r["genotype"], r["base1"], r["base2"]) == (0, 0, 1)
    assert r["quality"] == 34
    P2 = oracle.Params(global_dep=1.0, pcr_dep=1.0, rank_sum=False)
    specs = [(30 + k, 0, "A", 8) for k in range(8)] + [(40 + k, 0, "G", 40) for k in range(3)]
    w = workload("A" * 200, _site_reads(site, specs))
    t1, raw = _hand_quality([(8, 0)] * 8 + [(40, 3)] * 3, 0)
    assert (oracle.GENOTYPES[t1], raw) == ("AG", 68)
    r = oracle.call_window(P2, w, p, site, site + 1)[0]
    assert oracle.GENOTYPES[r["genotype"]] == "AG" and r["rank_p"] == 1.0
    assert r["quality"] == 64
    # with the rank-sum on, the same site pays 10 log10(p) of the disjoint quality groups
    # (N = 11, W = 36, mu = 48, sigma^2 = 2 (12 - 528/110) = 14.4, z = -12/3.795): raw
    # int(68.x - 28.05) = 40 < cap
    r = oracle.call_window(P1, w, p, site, site + 1)[0]
    pz = math.erfc(12 / math.sqrt(14.4) / math.sqrt(2))
    assert abs(r["rank_p"] - pz) <= 1e-6 * pz
    assert r["quality"] == _hand_quality([(8, 0)] * 8 + [(40, 3)] * 3, 0, pz)[1] == 40
