"""Parity rules (BASELINE.json north_star) for comparing the CUDA path with the oracle.

- bit-exact: key multisets, sorted keys, calibration counts, per-site counters, depths, genotypes
  and every integer record field;
- L10 and post10 within 1e-9 relative (posteriors below 1e-300 compared absolutely);
- a site whose top two lp differ by < 1e-9 relative is a *near tie*: listed, not a mismatch;
- quality must match unless 10*(lp1-lp2) + 10*log10(rank_p) is within 1e-6 of an integer
  (listed as a near-integer site).
"""
from __future__ import annotations

import math

import numpy as np

GA1 = (0, 0, 0, 0, 1, 1, 1, 2, 2, 3)
GA2 = (0, 1, 2, 3, 1, 2, 3, 2, 3, 3)
INT_FIELDS = ("pos", "ref", "base1", "base2", "avgq1", "avgq2", "known", "cnt_uni1", "cnt_all1",
              "cnt_uni2", "cnt_all2", "depth")
REL = 1e-9
FLOAT_ULP2 = 2.0 ** -22          # two float32 ulps, relative


def _novel_prior(ref, het=1e-3, hom=5e-4):
    if ref == 4:
        return np.zeros(10)
    out = []
    for a, b in zip(GA1, GA2):
        v = 1.0 if (a == ref and b == ref) else het if (a == ref or b == ref) else \
            hom if a == b else het * hom
        out.append(math.log10(v))
    return np.array(out)


def prior_rows(w, sites, P=None):
    """log10 prior row of every site (R6; R18 variants from P: monoploid / ti/tv), vectorised:
    the novel row of the site's reference code, or the known-SNP row."""
    het = P.het_novel if P is not None else 1e-3
    hom = P.althom_novel if P is not None else 5e-4
    mono = bool(P is not None and P.monoploid)
    titv = bool(P is not None and P.titv)
    tab = np.zeros((5, 10))
    for r in range(4):
        for n, (a, b) in enumerate(zip(GA1, GA2)):
            wt = (lambda x: (2.0 if (r ^ x) == 3 else 0.5) if titv else 1.0)
            v = 1.0 if (a == r and b == r) else het * wt(b) if a == r else het * wt(a) if b == r \
                else hom * wt(a) if a == b else het * hom * wt(a) * wt(b)
            tab[r, n] = math.log10(v)
    het_mask = np.array([a != b for a, b in zip(GA1, GA2)])
    sites = np.asarray(sites, np.int64)
    origin = int(w["origin"])
    out = tab[np.asarray(w["ref"])[sites - origin].astype(np.int64)]
    kp = np.asarray(w["known_pos"], np.int64)
    if len(kp):
        kpr = np.log10(np.asarray(w["known_prior10"], np.float64).reshape(-1, 10))
        j = np.searchsorted(kp, sites)
        jc = np.minimum(j, len(kp) - 1)
        hit = (j < len(kp)) & (kp[jc] == sites)
        out[hit] = kpr[jc[hit]]
    if mono:
        out[:, het_mask] = -np.inf
    return out


def lp_rows(w, sites, L10, P=None):
    return np.asarray(L10, np.float64) + prior_rows(w, sites, P)


def rel_ok(a, b, rel=REL, abs_floor=0.0):
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    den = np.maximum(np.abs(a), np.abs(b))
    d = np.abs(a - b)
    return (d <= rel * den) | (d <= abs_floor)


def compare(w, rec_g, rec_o, L10_o, post_o=None, L10_g=None, post_g=None, sites=None, P=None):
    """Compare records (and optionally debug L10/post10).  Returns a report dict; raises
    AssertionError on any mismatch that is not an allowed near tie / near integer.  P: the oracle
    Params the records were called with (prior variants R18), default Params()."""
    n = len(rec_o)
    assert len(rec_g) == n
    sites = rec_o["pos"] if sites is None else sites
    lp = lp_rows(w, sites, L10_o, P)
    srt = np.sort(lp, 1)
    top1, top2 = srt[:, -1], srt[:, -2]
    with np.errstate(invalid="ignore"):
        near_tie = np.abs(top1 - top2) <= REL * np.maximum(np.abs(top1), np.abs(top2))
    # sites without a unique key have L = 0: their ties come from equal priors (e.g. reference N)
    # and carry no evidence — reported apart from the informative near ties
    informative = np.asarray(rec_o["cnt_uni1"]) > 0
    rep = dict(sites=n, near_tie=int((near_tie & informative).sum()),
               near_tie_uninformative=int((near_tie & ~informative).sum()), near_int=0)
    # integer fields (bit exact)
    for f in INT_FIELDS:
        bad = rec_g[f] != rec_o[f]
        assert not bad.any(), (f, np.nonzero(bad)[0][:10], rec_g[f][bad][:5], rec_o[f][bad][:5])
    gbad = (rec_g["genotype"] != rec_o["genotype"]) & ~near_tie
    assert not gbad.any(), ("genotype", np.nonzero(gbad)[0][:10])
    # quality: exact unless near an integer boundary (or a near tie)
    qbad = (rec_g["quality"] != rec_o["quality"]) & ~near_tie
    for i in np.nonzero(qbad)[0]:
        t = np.argsort(-lp[i], kind="stable")
        rp = float(rec_o["rank_p"][i])
        x = 10 * (lp[i][t[0]] - lp[i][t[1]]) + (10 * math.log10(rp) if rp > 0 else 0)
        assert abs(x - round(x)) < 1e-6, ("quality", i, rec_g["quality"][i], rec_o["quality"][i], x)
        rep["near_int"] += 1
    # the near-integer sites the rule could excuse, mismatching or not (reported)
    with np.errstate(invalid="ignore"):
        dl = 10 * (top1 - top2)
    rep["near_int_candidates"] = int(np.count_nonzero((np.abs(dl - np.round(dl)) < 1e-6) & informative))
    # floats
    ok = rel_ok(rec_g["copy_num"], rec_o["copy_num"], 0)
    assert ok.all(), ("copy_num", np.nonzero(~ok)[0][:10])
    # rank_p and post1 are doubles rounded to float32 on both sides: libm erfc / exp10 may differ
    # in the last double bits, which can move the float by at most one ulp (2^-23 relative); two
    # ulps are allowed
    ok = rel_ok(rec_g["rank_p"], rec_o["rank_p"], FLOAT_ULP2, 1e-30) | near_tie
    assert ok.all(), ("rank_p", np.nonzero(~ok)[0][:10])
    ok = rel_ok(rec_g["post1"], rec_o["post1"], FLOAT_ULP2, 1e-30) | near_tie
    assert ok.all(), ("post1", np.nonzero(~ok)[0][:10])
    if L10_g is not None:
        ok = rel_ok(L10_g, L10_o)
        assert ok.all(), ("L10", np.argwhere(~ok)[:10])
        rep["L10_max_rel"] = float(np.max(np.abs(L10_g - L10_o) /
                                          np.maximum(np.abs(L10_o), 1e-300)))
    if post_g is not None and post_o is not None:
        ok = rel_ok(post_g, post_o, REL, 1e-300) | near_tie[:, None]
        assert ok.all(), ("post10", np.argwhere(~ok)[:10])
    return rep
