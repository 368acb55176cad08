"""Small hand-built workloads and field comparison helpers for the tests (no method arithmetic)."""
from __future__ import annotations

import numpy as np

BASE = {"A": 0, "C": 1, "T": 2, "G": 3, "N": 4}


def workload(ref, reads, known=(), origin=0, read_len=100):
    """ref: str or u8 array; reads: list of dicts {pos, strand, hits, bases (str/list), quals}.
    known: list of (pos, prior10)."""
    if isinstance(ref, str):
        ref = np.array([BASE[c] for c in ref], np.uint8)
    reads = sorted(reads, key=lambda r: r["pos"])
    n = len(reads)
    pos = np.array([r["pos"] for r in reads], np.uint64)
    bl = []
    ql = []
    for r in reads:
        b = r["bases"]
        b = [BASE[c] for c in b] if isinstance(b, str) else list(b)
        q = r["quals"]
        q = [q] * len(b) if np.isscalar(q) else list(q)
        assert len(q) == len(b)
        bl.append(np.array(b, np.uint8))
        ql.append(np.array(q, np.uint8))
    ln = np.array([len(b) for b in bl], np.uint16)
    off = np.zeros(n + 1, np.uint64)
    off[1:] = np.cumsum(ln.astype(np.uint64))
    kp = np.array([k[0] for k in known], np.uint64)
    kpr = np.array([k[1] for k in known], np.float64).reshape(-1, 10)
    return dict(ref=ref, origin=origin, pos=pos, len=ln, off=off,
                bases=np.concatenate(bl) if bl else np.zeros(0, np.uint8),
                quals=np.concatenate(ql) if ql else np.zeros(0, np.uint8),
                strand=np.array([r.get("strand", 0) for r in reads], np.uint8),
                hits=np.array([r.get("hits", 1) for r in reads], np.uint16),
                known_pos=kp, known_prior10=kpr, read_len=read_len)


def site_columns(w, lo, hi):
    """Brute-force per-site recount (numpy, vectorised; independent of the oracle's loops).
    Returns dict of arrays over sites [lo, hi): depth, dep_uni, repeat, count_all[4],
    count_uni[4], q_sum[4]."""
    S = hi - lo
    ln = w["len"].astype(np.int64)
    rid = np.repeat(np.arange(len(ln)), ln)
    i = np.arange(len(rid)) - np.repeat(w["off"][:-1].astype(np.int64), ln)
    site = w["pos"].astype(np.int64)[rid] + i
    b = w["bases"].astype(np.int64)
    q = w["quals"].astype(np.int64)
    h = w["hits"].astype(np.int64)[rid]
    m = (site >= lo) & (site < hi) & (b < 4)
    s = site[m] - lo
    out = dict(depth=np.bincount(s, minlength=S), repeat=np.bincount(s, h[m], minlength=S))
    u = m & (h == 1)
    su = site[u] - lo
    out["dep_uni"] = np.bincount(su, minlength=S)
    out["count_all"] = np.stack([np.bincount(s[b[m] == k], minlength=S) for k in range(4)], 1)
    out["count_uni"] = np.stack([np.bincount(su[b[u] == k], minlength=S) for k in range(4)], 1)
    out["q_sum"] = np.stack([np.bincount(su[b[u] == k], q[u][b[u] == k], minlength=S)
                             for k in range(4)], 1)
    return out


def rel_err(a, b):
    a = np.asarray(a, np.float64)
    b = np.asarray(b, np.float64)
    den = np.maximum(np.abs(a), np.abs(b))
    with np.errstate(invalid="ignore", divide="ignore"):
        r = np.where(den > 0, np.abs(a - b) / den, 0.0)
    return r
