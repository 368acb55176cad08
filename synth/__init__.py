"""Seeded synthetic workloads (shared input module; holds none of the method's arithmetic).

Python wrapper around ``synth.c``.  Both the CUDA path (bench.py, GPU tests) and the CPU oracle
(tests, cpu_baseline) consume the dictionaries returned by :func:`generate`.  The named configs
follow BASELINE.json ``configs`` / SURVEY.md §8(d); the recipe is written out in DESIGN.md.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field, asdict

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "synth.c")
_LIB = os.path.join(_HERE, "libsynth.so")


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-ffp-contract=off", "-pthread",
                               "-o", _LIB, _SRC, "-lm"])
    return _LIB


class _Cfg(ctypes.Structure):
    _fields_ = [("seed", ctypes.c_uint64), ("n_sites", ctypes.c_uint64),
                ("origin", ctypes.c_uint64), ("depth", ctypes.c_double),
                ("read_len", ctypes.c_uint32), ("q_hi", ctypes.c_uint32),
                ("n_frac", ctypes.c_double), ("n_lead_frac", ctypes.c_double),
                ("n_blocks", ctypes.c_uint32), ("het_rate", ctypes.c_double),
                ("hom_rate", ctypes.c_double), ("multi_hit_rate", ctypes.c_double),
                ("dup_rate", ctypes.c_double), ("base_n_rate", ctypes.c_double),
                ("known_frac", ctypes.c_double), ("n_threads", ctypes.c_uint32),
                ("_pad", ctypes.c_uint32), ("region_lo", ctypes.c_uint64),
                ("region_hi", ctypes.c_uint64)]


@dataclass
class SynthConfig:
    name: str = "custom"
    seed: int = 1
    n_sites: int = 10_000
    origin: int = 0
    depth: float = 10.0
    read_len: int = 100
    q_hi: int = 40
    n_frac: float = 0.0
    n_lead_frac: float = 0.0
    n_blocks: int = 0
    het_rate: float = 1e-3
    hom_rate: float = 5e-4
    multi_hit_rate: float = 0.05
    dup_rate: float = 0.02
    base_n_rate: float = 1e-3
    known_frac: float = 0.5
    n_threads: int = field(default_factory=lambda: min(32, os.cpu_count() or 1))
    region_lo: int = 0           # generate only genome sites [region_lo, region_hi) plus the
    region_hi: int = 0           # reads covering them and the reference under those (0,0 = all)

    def scaled(self, **kw) -> "SynthConfig":
        d = asdict(self)
        d.update(kw)
        return SynthConfig(**d)


# BASELINE.json configs (C3/C4 are multi-GPU shards of the same recipe).
CONFIGS = {
    # C1: 10 kb window, 10X, ~20 planted SNPs (2e-3: 2/3 het, 1/3 hom)
    "C1": SynthConfig(name="C1", seed=1, n_sites=10_000, depth=10.0,
                      het_rate=4e-3 / 3, hom_rate=2e-3 / 3),
    # C2: chr21-like 48 Mb, 20X, ~14% N including a leading block
    "C2": SynthConfig(name="C2", seed=2, n_sites=48_000_000, depth=20.0,
                      n_frac=0.14, n_lead_frac=0.10, n_blocks=8),
    # C3: chr1-like 249 Mb, 30X, ~8% N
    "C3": SynthConfig(name="C3", seed=3, n_sites=249_000_000, depth=30.0,
                      n_frac=0.08, n_lead_frac=0.04, n_blocks=16),
    # C4: whole genome 3.1 Gb, 12.5X, ~5% N (generated per shard)
    "C4": SynthConfig(name="C4", seed=4, n_sites=3_100_000_000, depth=12.5,
                      n_frac=0.05, n_lead_frac=0.01, n_blocks=48),
    # C5: exome-like 5 Mb target at 100X with 10% PCR duplicates
    "C5": SynthConfig(name="C5", seed=5, n_sites=5_000_000, depth=100.0, dup_rate=0.10),
}


def _lib():
    lib = ctypes.CDLL(build())
    P = ctypes.c_void_p
    lib.syn_window.restype = None
    lib.syn_window.argtypes = [ctypes.POINTER(_Cfg), P]
    lib.syn_plan.restype = ctypes.c_uint64
    lib.syn_plan.argtypes = [ctypes.POINTER(_Cfg), P, P, P, P]
    lib.syn_fill.restype = ctypes.c_uint64
    lib.syn_fill.argtypes = [ctypes.POINTER(_Cfg), P, P, P, P] + [P] * 7
    lib.syn_soap_text.restype = ctypes.c_uint64
    lib.syn_soap_text.argtypes = [ctypes.c_uint64] + [P] * 7 + [ctypes.c_char_p, ctypes.c_uint32,
                                                               ctypes.c_uint64, P]
    lib.syn_n_intervals.restype = ctypes.c_uint64
    lib.syn_n_intervals.argtypes = [ctypes.POINTER(_Cfg), P]
    lib.syn_known.restype = ctypes.c_uint64
    lib.syn_known.argtypes = [ctypes.POINTER(_Cfg), P, P, P, P, P]
    return lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _cfg(cfg: SynthConfig) -> _Cfg:
    return _Cfg(cfg.seed, cfg.n_sites, cfg.origin, cfg.depth, cfg.read_len, cfg.q_hi, cfg.n_frac,
                cfg.n_lead_frac, cfg.n_blocks, cfg.het_rate, cfg.hom_rate, cfg.multi_hit_rate,
                cfg.dup_rate, cfg.base_n_rate, cfg.known_frac, cfg.n_threads, 0, cfg.region_lo,
                cfg.region_hi)


def n_intervals(cfg: SynthConfig | str) -> np.ndarray:
    """The genome's N blocks as an (k, 2) array of [begin, end) genome indices (no generation)."""
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    lib = _lib()
    c = _cfg(cfg)
    k = lib.syn_n_intervals(ctypes.byref(c), None)
    out = np.zeros(2 * max(k, 1), np.uint64)
    lib.syn_n_intervals(ctypes.byref(c), _p(out))
    return out[:2 * k].reshape(-1, 2).astype(np.int64)


def sample_read_starts(cfg: SynthConfig | str, n: int = 1_000_000, seed: int = 0) -> np.ndarray:
    """n read starts drawn uniformly over the genome's non-N sites (sorted): a thin sample with the
    placement density of the generated reads, for planning shards (shard.plan_by_bases)."""
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    iv = n_intervals(cfg)
    cuts = [0]
    for a, b in iv:
        cuts += [int(a), int(b)]
    cuts.append(cfg.n_sites)
    seg = np.array(cuts, np.int64).reshape(-1, 2)          # non-N segments [a, b)
    seg = seg[seg[:, 1] > seg[:, 0]]
    w = (seg[:, 1] - seg[:, 0]).astype(np.float64)
    rng = np.random.default_rng(seed)
    k = rng.choice(len(seg), n, p=w / w.sum())
    pos = seg[k, 0] + (rng.random(n) * (seg[k, 1] - seg[k, 0])).astype(np.int64)
    return np.sort(pos).astype(np.uint64) + np.uint64(cfg.origin)


def generate(cfg: SynthConfig | str, **overrides) -> dict:
    """Generate one workload (or one region of it).  Returns a dict of numpy arrays:

    ref (u8, 0=A 1=C 2=T 3=G 4=N) over the generated window, origin (global coordinate of
    ref[0]), region (global [lo, hi) the reads cover completely), snp/alt (planted truth),
    known_pos (u64[k]), known_prior10 (f64[k,10]),
    pos (u64[n]), len (u16[n]), off (u64[n+1]), bases (u8), quals (u8), strand (u8), hits (u16).
    """
    if isinstance(cfg, str):
        cfg = CONFIGS[cfg]
    if overrides:
        cfg = cfg.scaled(**overrides)
    c = _Cfg(cfg.seed, cfg.n_sites, cfg.origin, cfg.depth, cfg.read_len, cfg.q_hi, cfg.n_frac,
             cfg.n_lead_frac, cfg.n_blocks, cfg.het_rate, cfg.hom_rate, cfg.multi_hit_rate,
             cfg.dup_rate, cfg.base_n_rate, cfg.known_frac, cfg.n_threads, 0, cfg.region_lo,
             cfg.region_hi)
    lib = _lib()
    win = np.zeros(2, np.uint64)
    lib.syn_window(ctypes.byref(c), _p(win))
    g0, g1 = int(win[0]), int(win[1])
    n = g1 - g0
    ref = np.empty(n, np.uint8)
    snp = np.empty(n, np.uint8)
    alt = np.empty(n, np.uint8)
    elig = np.empty(n, np.uint8)
    nr = lib.syn_plan(ctypes.byref(c), _p(ref), _p(snp), _p(alt), _p(elig))
    if nr == (1 << 64) - 1:
        raise ValueError("bad synth config")
    L = cfg.read_len
    pos = np.empty(nr, np.uint64)
    ln = np.empty(nr, np.uint16)
    off = np.empty(nr + 1, np.uint64)
    bases = np.empty(nr * L, np.uint8)
    quals = np.empty(nr * L, np.uint8)
    strand = np.empty(nr, np.uint8)
    hits = np.empty(nr, np.uint16)
    lib.syn_fill(ctypes.byref(c), _p(ref), _p(snp), _p(alt), _p(elig), _p(pos), _p(ln),
                 _p(off), _p(bases), _p(quals), _p(strand), _p(hits))
    nk = lib.syn_known(ctypes.byref(c), _p(ref), _p(snp), _p(alt), None, None)
    kpos = np.empty(nk, np.uint64)
    kpr = np.empty((nk, 10), np.float64)
    lib.syn_known(ctypes.byref(c), _p(ref), _p(snp), _p(alt), _p(kpos), _p(kpr))
    del elig
    lo = cfg.region_lo if cfg.region_hi > cfg.region_lo else 0
    hi = min(cfg.region_hi, cfg.n_sites) if cfg.region_hi > cfg.region_lo else cfg.n_sites
    return dict(config=cfg, ref=ref, origin=cfg.origin + g0, snp=snp, alt=alt, known_pos=kpos,
                known_prior10=kpr, pos=pos, len=ln, off=off, bases=bases, quals=quals,
                strand=strand, hits=hits, read_len=L,
                region=(cfg.origin + lo, cfg.origin + hi))


def read_range(w: dict, lo: int, hi: int, max_read_len: int | None = None):
    """Index range [ra, rb) of reads that can touch sites [lo, hi): pos in [lo-L+1, hi)."""
    L = max_read_len or w["read_len"]
    ra = int(np.searchsorted(w["pos"], np.uint64(max(lo - L + 1, 0)), "left"))
    rb = int(np.searchsorted(w["pos"], np.uint64(hi), "left"))
    return ra, rb


def slice_reads(w: dict, ra: int, rb: int) -> dict:
    """A standalone read set holding reads [ra, rb) (offsets rebased to 0)."""
    o0, o1 = int(w["off"][ra]), int(w["off"][rb])
    out = dict(w)
    out.update(pos=w["pos"][ra:rb], len=w["len"][ra:rb], strand=w["strand"][ra:rb],
               hits=w["hits"][ra:rb], off=(w["off"][ra:rb + 1] - np.uint64(o0)),
               bases=w["bases"][o0:o1], quals=w["quals"][o0:o1])
    return out


def soap_text(w: dict, chr_name: str = "chr1", q_offset: int = 33, loc_base: int | None = None,
              ra: int = 0, rb: int | None = None) -> bytes:
    """Reads [ra, rb) of a workload as SOAP alignment text (reading R19): one tab-separated line
    per read — id, seq, qual, n_hits, a/b, len, strand, chr, 1-based location, n_mismatch.
    location = pos - loc_base + 1 (loc_base defaults to the workload's origin)."""
    lib = _lib()
    rb = len(w["pos"]) if rb is None else rb
    lb = int(w["origin"]) if loc_base is None else loc_base
    arr = dict(pos=np.ascontiguousarray(w["pos"][ra:rb], np.uint64),
               len=np.ascontiguousarray(w["len"][ra:rb], np.uint16),
               off=np.ascontiguousarray(w["off"][ra:rb + 1], np.uint64),
               strand=np.ascontiguousarray(w["strand"][ra:rb], np.uint8),
               hits=np.ascontiguousarray(w["hits"][ra:rb], np.uint16))
    bases = np.ascontiguousarray(w["bases"], np.uint8)
    quals = np.ascontiguousarray(w["quals"], np.uint8)
    a = [rb - ra, _p(arr["pos"]), _p(arr["len"]), _p(arr["off"]), _p(bases), _p(quals),
         _p(arr["strand"]), _p(arr["hits"]), chr_name.encode(), q_offset, lb]
    n = lib.syn_soap_text(*a, None)
    out = np.empty(n, np.uint8)
    lib.syn_soap_text(*a, _p(out))
    return out.tobytes()
