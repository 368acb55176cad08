"""Seeded synthetic record tables for the compression tests (input generator only: no method
arithmetic).  Shapes follow the call output: long runs of equal quality columns, N gaps, sparse
SNP-related exceptions, a dense-ish second allele; plus adversarial variants."""
from __future__ import annotations

import numpy as np

from oracle import RECORD_DTYPE

HOM = np.array([0, 4, 7, 9, 255], np.uint8)


def records(n: int, seed: int = 0, kind: str = "call", pos0: int = 1000) -> np.ndarray:
    rng = np.random.default_rng(seed)
    r = np.zeros(n, RECORD_DTYPE)
    r["pos"] = np.arange(n, dtype=np.uint64) + np.uint64(pos0)
    ref = rng.integers(0, 4, n).astype(np.uint8)
    if kind in ("call", "runs"):
        # N gaps
        for _ in range(max(1, n // 5000)):
            a = int(rng.integers(0, max(n, 1)))
            ref[a:a + int(rng.integers(1, 3000))] = 4
    else:
        ref[rng.random(n) < 0.2] = 4
    r["ref"] = ref
    depth = np.repeat(rng.poisson(20, n // 3 + 1), 3)[:n].astype(np.uint32)
    depth[ref == 4] = 0
    r["depth"] = depth
    r["genotype"] = HOM[ref]
    snp = rng.random(n) < 0.002
    r["genotype"][snp] = rng.integers(0, 10, snp.sum())
    r["known"][rng.random(n) < 0.001] = 1
    r["base1"] = np.where(depth > 0, ref, 4)
    r["base1"][ref == 4] = np.where(rng.random((ref == 4).sum()) < 0.1, 2, 4)
    sec = (rng.random(n) < 0.3) & (depth > 0)
    r["base2"] = np.where(sec, (ref + 1) % 4, 4)
    r["avgq2"] = np.where(sec, rng.integers(2, 40, n), 0)
    r["cnt_uni2"] = np.where(sec, rng.integers(0, 3, n), 0)
    r["cnt_all2"] = np.where(sec, r["cnt_uni2"] + rng.integers(0, 2, n), 0)
    r["cnt_all2"][sec & (r["cnt_all2"] == 0)] = 1
    q = np.repeat(np.minimum(99, rng.integers(20, 120, n // 11 + 1)), 11)[:n]
    r["quality"] = np.where(depth > 0, q, 0)
    r["avgq1"] = np.where(depth > 0, np.repeat(rng.integers(25, 38, n // 4 + 1), 4)[:n], 0)
    r["cnt_uni1"] = np.minimum(depth, 65535)
    r["cnt_all1"] = np.minimum(depth + (rng.random(n) < 0.05), 65535)
    r["rank_p"] = np.float32(1.0)
    het = rng.random(n) < 0.001
    r["rank_p"][het] = rng.random(het.sum()).astype(np.float32)
    r["post1"] = np.where(rng.random(n) < 0.03, rng.random(n), 1.0).astype(np.float32)
    r["copy_num"] = np.where(depth > 0, 1.0, 0.0).astype(np.float32)
    r["copy_num"][rng.random(n) < 0.01] = np.float32(1.25)
    if kind == "random":
        # every column high-entropy: exercises RAW dictionaries and 1-site runs
        for f in ("quality", "avgq1", "avgq2", "known", "genotype"):
            r[f] = rng.integers(0, 256, n)
        for f in ("cnt_uni1", "cnt_all1", "cnt_uni2", "cnt_all2"):
            r[f] = rng.integers(0, 65536, n)
        r["depth"] = rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32)
        for f in ("base1", "base2"):
            r[f] = rng.integers(0, 5, n)
        for f in ("rank_p", "copy_num", "post1"):
            r[f] = rng.integers(0, 2**32, n, dtype=np.uint64).astype(np.uint32).view(np.float32)
    if kind == "const":
        for f in RECORD_DTYPE.names:
            if f != "pos":
                r[f] = r[f][0] if n else 0
    return r
