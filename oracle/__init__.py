"""CPU ORACLE for the GSNP hot path — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline`` leg and
``--impl reference``) may import this package.  The product path (``libgsnp`` and
``paper_conf_icpp_luzlwfl11_b200``) never imports, links or executes it, and this package never
imports the product.  The arithmetic lives in ``oracle.c`` (plain single-threaded C, fp64,
glibc libm, ``-O2 -ffp-contract=off``); this file is argument marshalling.

Every function cites the PAPER.md passage it follows (see oracle.c).  Pins live in
``tests/test_oracle_pins.py``.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_SRC_C = os.path.join(_HERE, "compress.c")          # output compression (§V-B, reading R17)
_LIB = os.path.join(_HERE, "liboracle.so")

GA1 = (0, 0, 0, 0, 1, 1, 1, 2, 2, 3)
GA2 = (0, 1, 2, 3, 1, 2, 3, 2, 3, 3)
GENOTYPES = ("AA", "AC", "AT", "AG", "CC", "CT", "CG", "TT", "TG", "GG")


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or any(os.path.getmtime(_LIB) < os.path.getmtime(s)
                                                  for s in (_SRC, _SRC_C)):
        subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-ffp-contract=off",
                               "-o", _LIB, _SRC, _SRC_C, "-lm"])
    return _LIB


class _Params(ctypes.Structure):
    _fields_ = [("max_read_len", ctypes.c_uint32), ("q_max", ctypes.c_uint32),
                ("het_novel", ctypes.c_double), ("althom_novel", ctypes.c_double),
                ("global_dep", ctypes.c_double), ("pcr_dep", ctypes.c_double),
                ("calib_min_count", ctypes.c_uint32), ("rank_sum", ctypes.c_uint32),
                ("prior_mode", ctypes.c_uint32)]


class _Reads(ctypes.Structure):
    _fields_ = [("n_reads", ctypes.c_uint64)] + [(k, ctypes.c_void_p) for k in
                                                 ("pos", "len", "off", "bases", "quals",
                                                  "strand", "hits")]


RECORD_DTYPE = np.dtype([("pos", "<u8"), ("ref", "u1"), ("genotype", "u1"), ("quality", "u1"),
                         ("base1", "u1"), ("base2", "u1"), ("avgq1", "u1"), ("avgq2", "u1"),
                         ("known", "u1"), ("cnt_uni1", "<u2"), ("cnt_all1", "<u2"),
                         ("cnt_uni2", "<u2"), ("cnt_all2", "<u2"), ("depth", "<u4"),
                         ("rank_p", "<f4"), ("copy_num", "<f4"), ("post1", "<f4")])
assert RECORD_DTYPE.itemsize == 40

COUNTER_FIELDS = ("depth", "dep_uni", "repeat", "all_A", "all_C", "all_T", "all_G",
                  "uni_A", "uni_C", "uni_T", "uni_G", "qs_A", "qs_C", "qs_T", "qs_G")


@dataclass
class Params:
    max_read_len: int = 100
    q_max: int = 40
    het_novel: float = 1e-3
    althom_novel: float = 5e-4
    global_dep: float = 0.9
    pcr_dep: float = 0.5
    calib_min_count: int = 10
    rank_sum: bool = True
    monoploid: bool = False      # R18: heterozygous genotypes get prior 0
    titv: bool = False           # R18: novel transition:transversion 2:1
    rank_exact: bool = False     # R20: exact small-sample rank-sum when nothing ties

    def c(self) -> _Params:
        return _Params(self.max_read_len, self.q_max, self.het_novel, self.althom_novel,
                       self.global_dep, self.pcr_dep, self.calib_min_count,
                       int(self.rank_sum) * (2 if self.rank_exact else 1),
                       int(self.monoploid) | 2 * int(self.titv))


_lib_cache = None


def lib():
    global _lib_cache
    if _lib_cache is None:
        L = ctypes.CDLL(build())
        P = ctypes.c_void_p
        PP = ctypes.POINTER(_Params)
        L.or_key.restype = ctypes.c_uint32
        L.or_key.argtypes = [ctypes.c_int] * 4
        L.or_key_paper.restype = ctypes.c_uint32
        L.or_key_paper.argtypes = [ctypes.c_int] * 4
        L.or_adjust.restype = ctypes.c_int
        L.or_adjust.argtypes = [PP, ctypes.c_int, ctypes.c_int, ctypes.c_int]
        L.or_calib_counts.restype = ctypes.c_int
        L.or_calib_counts.argtypes = [PP, P, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64, P,
                                      ctypes.POINTER(_Reads), P]
        L.or_p_matrix.restype = ctypes.c_int
        L.or_p_matrix.argtypes = [PP, P, P]
        L.or_sparse_likelihood.argtypes = [PP, P, ctypes.c_uint64, P, P, P, P, P, P]
        L.or_dense_likelihood.argtypes = [PP, P, ctypes.c_uint64, P, P, P, P, P]
        L.or_rank_sum.restype = ctypes.c_double
        L.or_rank_sum.argtypes = [ctypes.c_uint64, P, ctypes.c_uint64, P]
        L.or_rank_sum_exact.restype = ctypes.c_double
        L.or_rank_sum_exact.argtypes = [ctypes.c_uint64, P, ctypes.c_uint64, P]
        L.or_call_window.restype = ctypes.c_int
        L.or_call_window.argtypes = [PP, P, ctypes.c_uint64, ctypes.c_uint64, ctypes.c_uint64, P, P,
                                     P, ctypes.POINTER(_Reads), ctypes.c_uint64, ctypes.c_uint64,
                                     P, P, P, P, P, P]
        L.or_priors_from_freq.restype = ctypes.c_int
        L.or_priors_from_freq.argtypes = [P, ctypes.c_uint64, ctypes.c_double, P]
        L.oc_compress.restype = ctypes.c_uint64
        L.oc_compress.argtypes = [P, ctypes.c_uint64, ctypes.c_uint32, P, ctypes.c_uint64]
        L.oc_decompress.restype = ctypes.c_int64
        L.oc_decompress.argtypes = [P, ctypes.c_uint64, P, ctypes.c_uint64]
        L.or_sizeof_record.restype = ctypes.c_int
        assert L.or_sizeof_record() == RECORD_DTYPE.itemsize
        _lib_cache = L
    return _lib_cache


def _p(a):
    return None if a is None else np.ascontiguousarray(a).ctypes.data_as(ctypes.c_void_p)


def _reads(w: dict):
    arrs = dict(pos=np.ascontiguousarray(w["pos"], np.uint64),
                len=np.ascontiguousarray(w["len"], np.uint16),
                off=np.ascontiguousarray(w["off"], np.uint64),
                bases=np.ascontiguousarray(w["bases"], np.uint8),
                quals=np.ascontiguousarray(w["quals"], np.uint8),
                strand=np.ascontiguousarray(w["strand"], np.uint8),
                hits=np.ascontiguousarray(w["hits"], np.uint16))
    r = _Reads(len(arrs["pos"]), *[arrs[k].ctypes.data_as(ctypes.c_void_p) for k in
                                   ("pos", "len", "off", "bases", "quals", "strand", "hits")])
    return r, arrs  # keep arrays alive


def key(base, q, coord, strand) -> int:
    return lib().or_key(base, q, coord, strand)


def key_paper(base, score, coord, strand) -> int:
    return lib().or_key_paper(base, score, coord, strand)


def adjust(P: Params, q: int, pcr: int, g: int) -> int:
    c = P.c()
    return lib().or_adjust(ctypes.byref(c), q, pcr, g)


def calib_counts(P: Params, w: dict) -> np.ndarray:
    """C1 counts, uint64[64][256][4][4] (index q<<12|cyc<<4|t<<2|o)."""
    c = P.c()
    r, keep = _reads(w)
    C = np.zeros(64 * 256 * 16, np.uint64)
    ref = np.ascontiguousarray(w["ref"], np.uint8)
    kp = np.ascontiguousarray(w["known_pos"], np.uint64)
    rc = lib().or_calib_counts(ctypes.byref(c), _p(ref), len(ref), int(w["origin"]), len(kp),
                               _p(kp), ctypes.byref(r), _p(C))
    if rc != 0:
        raise ValueError(f"or_calib_counts: {rc}")
    return C.reshape(64, 256, 4, 4)


def p_matrix(P: Params, C: np.ndarray) -> np.ndarray:
    c = P.c()
    Cc = np.ascontiguousarray(C, np.uint64).reshape(-1)
    p = np.zeros(64 * 256 * 16, np.float64)
    lib().or_p_matrix(ctypes.byref(c), _p(Cc), _p(p))
    return p.reshape(64, 256, 4, 4)


def _tuples(b, q, coord, strand):
    return [np.ascontiguousarray(x, np.uint8) for x in (b, q, coord, strand)]


def sparse_likelihood(P: Params, p: np.ndarray, b, q, coord, strand):
    """Alg. 4 over a list of aligned bases -> (L10[10], sorted keys)."""
    c = P.c()
    t = _tuples(b, q, coord, strand)
    n = len(t[0])
    L10 = np.zeros(10)
    ks = np.zeros(max(n, 1), np.uint32)
    pp = np.ascontiguousarray(p, np.float64)
    lib().or_sparse_likelihood(ctypes.byref(c), _p(pp), n, *[_p(x) for x in t], _p(L10), _p(ks))
    return L10, ks[:n]


def dense_likelihood(P: Params, p: np.ndarray, b, q, coord, strand):
    """Alg. 1 over a dense base_occ materialisation -> L10[10]."""
    c = P.c()
    t = _tuples(b, q, coord, strand)
    L10 = np.zeros(10)
    pp = np.ascontiguousarray(p, np.float64)
    lib().or_dense_likelihood(ctypes.byref(c), _p(pp), len(t[0]), *[_p(x) for x in t], _p(L10))
    return L10


def rank_sum(X, Y) -> float:
    X = np.ascontiguousarray(X, np.uint8)
    Y = np.ascontiguousarray(Y, np.uint8)
    return lib().or_rank_sum(len(X), _p(X), len(Y), _p(Y))


def rank_sum_exact(X, Y) -> float:
    """R20: exact two-sided p when len(X), len(Y) <= 32 and nothing ties, else rank_sum."""
    X = np.ascontiguousarray(X, np.uint8)
    Y = np.ascontiguousarray(Y, np.uint8)
    return lib().or_rank_sum_exact(len(X), _p(X), len(Y), _p(Y))


def call_window(P: Params, w: dict, p: np.ndarray, w0: int, w1: int, debug: bool = False,
                want=("off", "keys", "counters", "L10", "post10"), out=None):
    """C0-C9 over sites [w0, w1).  Returns records (RECORD_DTYPE) and, with debug=True, a dict
    with off (u32[S+1]), keys (sorted, CSR), counters (u32[S,15]), L10, post10 (f64[S,10]) —
    only the parts named in `want`.  `out` may supply the destination arrays (dict with "rec" and
    any of the debug names), e.g. views of shared memory."""
    c = P.c()
    r, keep = _reads(w)
    S = w1 - w0
    out = out or {}
    rec = out["rec"] if "rec" in out else np.zeros(S, RECORD_DTYPE)
    ref = np.ascontiguousarray(w["ref"], np.uint8)
    kp = np.ascontiguousarray(w["known_pos"], np.uint64)
    kpr = np.ascontiguousarray(w["known_prior10"], np.float64)
    pp = np.ascontiguousarray(p, np.float64)
    dbg = None
    if debug:
        nb = int(w["off"][-1]) if len(w["off"]) else 0
        make = dict(off=lambda: np.zeros(S + 1, np.uint32), keys=lambda: np.zeros(max(nb, 1), np.uint32),
                    counters=lambda: np.zeros((S, 15), np.uint32), L10=lambda: np.zeros((S, 10)),
                    post10=lambda: np.zeros((S, 10)))
        dbg = {k: (out[k] if k in out else make[k]()) for k in want}
        if "keys" in dbg and "off" not in dbg:
            dbg["off"] = make["off"]()
    g = (lambda k: _p(dbg[k]) if dbg and k in dbg else None)
    rc = lib().or_call_window(ctypes.byref(c), _p(ref), len(ref), int(w["origin"]), len(kp),
                              _p(kp), _p(kpr), _p(pp), ctypes.byref(r), w0, w1, _p(rec),
                              g("off"), g("keys"), g("counters"), g("L10"), g("post10"))
    if rc != 0:
        raise ValueError(f"or_call_window: {rc}")
    if dbg:
        if "keys" in dbg:
            dbg["keys"] = dbg["keys"][: dbg["off"][-1]]
        return rec, dbg
    return rec


def priors_from_freq(freq, floor_prior: float = 5e-7) -> np.ndarray:
    """R18: Hardy-Weinberg known-SNP prior rows (n x 10) from allele frequencies (n x 4)."""
    f = np.ascontiguousarray(freq, np.float64).reshape(-1, 4)
    out = np.zeros((len(f), 10), np.float64)
    if lib().or_priors_from_freq(_p(f), len(f), float(floor_prior), _p(out)) != 0:
        raise ValueError("allele frequencies must be >= 0 with a positive row sum")
    return out


def compress(rec: np.ndarray, block_sites: int) -> np.ndarray:
    """RLE-DICT column compression of records (§V-B, format R17 in compress.c).
    Returns the stream as uint32 words."""
    rec = np.ascontiguousarray(rec, RECORD_DTYPE)
    need = lib().oc_compress(_p(rec), len(rec), block_sites, None, 0)
    out = np.zeros(max(int(need), 1), np.uint32)
    got = lib().oc_compress(_p(rec), len(rec), block_sites, _p(out), len(out))
    assert got == need
    return out[:need]


def decompress(words: np.ndarray, n_max: int) -> np.ndarray:
    """Inverse of compress(); raises ValueError on a malformed stream."""
    words = np.ascontiguousarray(words, np.uint32)
    rec = np.zeros(max(n_max, 1), RECORD_DTYPE)
    n = lib().oc_decompress(_p(words), len(words), _p(rec), n_max)
    if n < 0:
        raise ValueError("malformed compressed stream")
    return rec[:n]
