"""Thin ctypes binding of libgsnp (include/gsnp.h).  Argument marshalling only: every step of the
hot path runs in the library's CUDA kernels.  Arrays may be numpy (host) or torch tensors
(host or CUDA; CUDA tensors are used in place).  There is no fallback: if ``libgsnp.so`` is
missing the import fails (run ``__graft_entry__.build()``).
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("GSNP_LIB") or os.path.join(_HERE, "libgsnp.so")   # GSNP_LIB: A/B builds

GSNP_ABI_VERSION = 1
GSNP_RANK_SUM = 0x1
GSNP_TIMING = 0x2
GSNP_MONOPLOID = 0x4
GSNP_TITV = 0x8
GSNP_RANK_EXACT = 0x10      # R20 exact small-sample rank-sum (include/gsnp.h)
STAGES = ("validate", "calib_count", "tile_ranges", "call_tile", "finalize", "big_sites",
          "compress", "warp_sites", "dense_count", "dense_lik", "dense_recycle", "parse", "unpack")
STATUS = {0: "GSNP_OK", -1: "GSNP_E_INVAL", -2: "GSNP_E_RANGE", -3: "GSNP_E_UNSORTED",
          -4: "GSNP_E_STATE", -5: "GSNP_E_NOMEM", -6: "GSNP_E_CUDA", -7: "GSNP_E_CAPACITY"}

# exported symbols declared in include/gsnp.h
SYMBOLS = ("gsnp_params_default", "gsnp_create", "gsnp_calibrate", "gsnp_calibrate_count",
           "gsnp_calibrate_finalize", "gsnp_call", "gsnp_debug_window", "gsnp_get_tables",
           "gsnp_compress", "gsnp_call_compressed", "gsnp_call_dense", "gsnp_priors_from_freq", "gsnp_parse_soap",
           "gsnp_pack_reads", "gsnp_packed_sizes", "gsnp_unpack_reads", "gsnp_call_async",
           "gsnp_wait",
           "gsnp_launch_count", "gsnp_stage_times", "gsnp_strerror", "gsnp_last_error",
           "gsnp_destroy")


class GsnpError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class gsnp_params(ctypes.Structure):
    _fields_ = [("abi_version", ctypes.c_uint32), ("max_read_len", ctypes.c_uint32),
                ("q_max", ctypes.c_uint32), ("calib_min_count", ctypes.c_uint32),
                ("het_novel", ctypes.c_double), ("althom_novel", ctypes.c_double),
                ("global_dep", ctypes.c_double), ("pcr_dep", ctypes.c_double),
                ("flags", ctypes.c_uint32), ("device", ctypes.c_int32),
                ("stream", ctypes.c_void_p)]


class gsnp_reference(ctypes.Structure):
    _fields_ = [("code", ctypes.c_void_p), ("n_sites", ctypes.c_uint64),
                ("origin", ctypes.c_uint64)]


class gsnp_priors(ctypes.Structure):
    _fields_ = [("n", ctypes.c_uint64), ("pos", ctypes.c_void_p), ("prior10", ctypes.c_void_p)]


class gsnp_reads(ctypes.Structure):
    _fields_ = [("n_reads", ctypes.c_uint64), ("pos", ctypes.c_void_p), ("len", ctypes.c_void_p),
                ("off", ctypes.c_void_p), ("bases", ctypes.c_void_p), ("quals", ctypes.c_void_p),
                ("strand", ctypes.c_void_p), ("hits", ctypes.c_void_p),
                ("on_device", ctypes.c_int32)]


RECORD_DTYPE = np.dtype([("pos", "<u8"), ("ref", "u1"), ("genotype", "u1"), ("quality", "u1"),
                         ("base1", "u1"), ("base2", "u1"), ("avgq1", "u1"), ("avgq2", "u1"),
                         ("known", "u1"), ("cnt_uni1", "<u2"), ("cnt_all1", "<u2"),
                         ("cnt_uni2", "<u2"), ("cnt_all2", "<u2"), ("depth", "<u4"),
                         ("rank_p", "<f4"), ("copy_num", "<f4"), ("post1", "<f4")])
assert RECORD_DTYPE.itemsize == 40

_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: build it with __graft_entry__.build()")
        L = ctypes.CDLL(LIB_PATH)
        P = ctypes.c_void_p
        S = ctypes.c_int32
        u64 = ctypes.c_uint64
        L.gsnp_params_default.restype = S
        L.gsnp_params_default.argtypes = [ctypes.POINTER(gsnp_params)]
        L.gsnp_create.restype = S
        L.gsnp_create.argtypes = [ctypes.POINTER(gsnp_reference), ctypes.POINTER(gsnp_priors),
                                  ctypes.POINTER(gsnp_params), ctypes.POINTER(P)]
        L.gsnp_calibrate.restype = S
        L.gsnp_calibrate.argtypes = [P, ctypes.POINTER(gsnp_reads)]
        L.gsnp_calibrate_count.restype = S
        L.gsnp_calibrate_count.argtypes = [P, ctypes.POINTER(gsnp_reads), P]
        L.gsnp_calibrate_finalize.restype = S
        L.gsnp_calibrate_finalize.argtypes = [P, P]
        L.gsnp_call.restype = S
        L.gsnp_call.argtypes = [P, ctypes.POINTER(gsnp_reads), u64, u64, P, u64,
                                ctypes.POINTER(u64)]
        L.gsnp_debug_window.restype = S
        L.gsnp_debug_window.argtypes = [P, ctypes.POINTER(gsnp_reads), u64, u64] + [P] * 7
        L.gsnp_get_tables.restype = S
        L.gsnp_get_tables.argtypes = [P, P, P, P, P, P]
        L.gsnp_compress.restype = S
        L.gsnp_compress.argtypes = [P, P, u64, ctypes.c_uint32, P, u64, ctypes.POINTER(u64)]
        L.gsnp_call_compressed.restype = S
        L.gsnp_call_compressed.argtypes = [P, ctypes.POINTER(gsnp_reads), u64, u64,
                                           ctypes.c_uint32, P, u64, ctypes.POINTER(u64)]
        L.gsnp_call_dense.restype = S
        L.gsnp_call_dense.argtypes = [P, ctypes.POINTER(gsnp_reads), u64, u64, ctypes.c_uint32,
                                      P, u64, ctypes.POINTER(u64)]
        L.gsnp_priors_from_freq.restype = S
        L.gsnp_priors_from_freq.argtypes = [P, u64, ctypes.c_double, P]
        L.gsnp_parse_soap.restype = S
        L.gsnp_parse_soap.argtypes = [P, P, u64, ctypes.c_char_p, ctypes.c_uint32, u64] + [P] * 7 + \
            [u64, u64, ctypes.POINTER(u64), ctypes.POINTER(u64)]
        L.gsnp_pack_reads.restype = S
        L.gsnp_pack_reads.argtypes = [ctypes.POINTER(gsnp_reads), ctypes.POINTER(gsnp_reference),
                                      ctypes.c_uint32, P, u64, ctypes.POINTER(u64)]
        L.gsnp_packed_sizes.restype = S
        L.gsnp_packed_sizes.argtypes = [P, u64, ctypes.POINTER(u64), ctypes.POINTER(u64)]
        L.gsnp_unpack_reads.restype = S
        L.gsnp_unpack_reads.argtypes = [P, P, u64] + [P] * 7
        L.gsnp_call_async.restype = S
        L.gsnp_call_async.argtypes = [P, ctypes.POINTER(gsnp_reads), u64, u64, P, u64]
        L.gsnp_wait.restype = S
        L.gsnp_wait.argtypes = [P]
        L.gsnp_launch_count.restype = u64
        L.gsnp_launch_count.argtypes = [P]
        L.gsnp_stage_times.restype = S
        L.gsnp_stage_times.argtypes = [P, P, P, ctypes.c_int, ctypes.c_int]
        L.gsnp_strerror.restype = ctypes.c_char_p
        L.gsnp_strerror.argtypes = [S]
        L.gsnp_last_error.restype = ctypes.c_char_p
        L.gsnp_last_error.argtypes = [P]
        L.gsnp_destroy.restype = None
        L.gsnp_destroy.argtypes = [P]
        _lib = L
    return _lib


def _ptr(a):
    """Data pointer of a numpy array or torch tensor (host or CUDA)."""
    if a is None:
        return None
    if hasattr(a, "data_ptr"):
        return ctypes.c_void_p(a.data_ptr())
    return a.ctypes.data_as(ctypes.c_void_p)


def _on_device(a) -> bool:
    return bool(getattr(a, "is_cuda", False))


def _contig(a, dtype):
    if hasattr(a, "data_ptr"):
        import torch
        tmap = {np.uint8: torch.uint8, np.uint16: torch.uint16, np.uint64: torch.uint64,
                np.float64: torch.float64}
        t = a.contiguous()
        assert t.dtype == tmap[dtype], f"expected {tmap[dtype]}, got {t.dtype}"
        return t
    return np.ascontiguousarray(a, dtype)


def make_reads(w: dict):
    """gsnp_reads from a dict with pos/len/off/bases/quals/strand/hits (numpy or torch)."""
    arrs = dict(pos=_contig(w["pos"], np.uint64), len=_contig(w["len"], np.uint16),
                off=_contig(w["off"], np.uint64), bases=_contig(w["bases"], np.uint8),
                quals=_contig(w["quals"], np.uint8), strand=_contig(w["strand"], np.uint8),
                hits=_contig(w["hits"], np.uint16))
    dev = _on_device(arrs["pos"])
    n = int(arrs["pos"].shape[0])
    r = gsnp_reads(n, *[_ptr(arrs[k]) for k in ("pos", "len", "off", "bases", "quals",
                                                "strand", "hits")], int(dev))
    r._keep = arrs
    return r


def params_default(**kw) -> gsnp_params:
    p = gsnp_params()
    _check(lib().gsnp_params_default(ctypes.byref(p)), None)
    for k, v in kw.items():
        if k == "stream" and v is not None and not isinstance(v, int):
            v = int(getattr(v, "cuda_stream", v))
        setattr(p, k, v)
    return p


def _check(st: int, ctx):
    if st != 0:
        msg = lib().gsnp_last_error(ctx).decode() if ctx else lib().gsnp_strerror(st).decode()
        raise GsnpError(st, msg)


class Context:
    """RAII wrapper over gsnp_ctx*.  Methods mirror the ABI calls."""

    def __init__(self, ref, origin: int = 0, known_pos=None, known_prior10=None, **params):
        self.params = params_default(**params)
        ref = np.ascontiguousarray(ref, np.uint8)
        self._ref = ref
        r = gsnp_reference(_ptr(ref), len(ref), int(origin))
        kp = np.ascontiguousarray(known_pos if known_pos is not None else [], np.uint64)
        kpr = np.ascontiguousarray(known_prior10 if known_prior10 is not None else
                                   np.zeros((0, 10)), np.float64)
        pri = gsnp_priors(len(kp), _ptr(kp), _ptr(kpr))
        h = ctypes.c_void_p()
        st = lib().gsnp_create(ctypes.byref(r), ctypes.byref(pri), ctypes.byref(self.params),
                               ctypes.byref(h))
        if st != 0:
            raise GsnpError(st, lib().gsnp_strerror(st).decode())
        self.h = h
        self.origin = int(origin)
        self.n_sites = len(ref)

    @classmethod
    def from_workload(cls, w: dict, **params):
        return cls(w["ref"], w["origin"], w["known_pos"], w["known_prior10"], **params)

    def close(self):
        if getattr(self, "h", None):
            try:
                lib().gsnp_destroy(self.h)
            except TypeError:            # interpreter shutdown: module globals already cleared
                pass
            self.h = None

    __del__ = close

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def calibrate(self, reads: dict):
        r = make_reads(reads)
        _check(lib().gsnp_calibrate(self.h, ctypes.byref(r)), self.h)

    def calibrate_count(self, reads: dict, counts=None):
        """Returns (or fills) this shard's counts, uint64[64*256*16] (numpy or CUDA tensor)."""
        if counts is None:
            counts = np.zeros(64 * 256 * 16, np.uint64)
        r = make_reads(reads)
        _check(lib().gsnp_calibrate_count(self.h, ctypes.byref(r), _ptr(counts)), self.h)
        return counts

    def calibrate_finalize(self, counts):
        _check(lib().gsnp_calibrate_finalize(self.h, _ptr(counts)), self.h)

    def call(self, reads: dict, w0: int, w1: int, out=None):
        """Records for sites [w0, w1).  out: None (numpy result), a numpy RECORD_DTYPE array,
        or a CUDA uint8 tensor of >= 40*(w1-w0) bytes (device output)."""
        S = w1 - w0
        if out is None:
            out = np.zeros(S, RECORD_DTYPE)
        cap = (out.numel() // 40) if hasattr(out, "numel") else len(out)
        r = make_reads(reads)
        n = ctypes.c_uint64(0)
        _check(lib().gsnp_call(self.h, ctypes.byref(r), w0, w1, _ptr(out), cap, ctypes.byref(n)),
               self.h)
        return out

    def call_reads(self, r: gsnp_reads, w0: int, w1: int, out):
        """Low-overhead variant with prebuilt gsnp_reads (bench loop)."""
        cap = (out.numel() // 40) if hasattr(out, "numel") else len(out)
        n = ctypes.c_uint64(0)
        _check(lib().gsnp_call(self.h, ctypes.byref(r), w0, w1, _ptr(out), cap, ctypes.byref(n)),
               self.h)
        return out

    def call_dense(self, reads, w0: int, w1: int, out=None, chunk_sites: int = 16384):
        """The dense ablation (gsnp_call_dense): same records as call(),
        through per-site dense base_occ arrays, chunk_sites sites at a time."""
        S = w1 - w0
        if out is None:
            out = np.zeros(S, RECORD_DTYPE)
        cap = (out.numel() // 40) if hasattr(out, "numel") else len(out)
        r = reads if isinstance(reads, gsnp_reads) else make_reads(reads)
        n = ctypes.c_uint64(0)
        _check(lib().gsnp_call_dense(self.h, ctypes.byref(r), w0, w1, chunk_sites, _ptr(out), cap,
                                     ctypes.byref(n)), self.h)
        return out

    def parse_soap(self, text, chr_name=None, q_offset: int = 33, loc_base: int = 0,
                   device: bool = True, out: dict | None = None):
        """SOAP alignment text -> reads dict (gsnp_parse_soap).  text: bytes /
        numpy uint8 (host) or a CUDA uint8 tensor.  Returns CUDA tensors (device=True) or numpy
        arrays, trimmed to the parsed sizes; out: preallocated arrays to fill instead (sizes are
        then the caller's, e.g. from a previous parse)."""
        if isinstance(text, (bytes, bytearray)):
            text = np.frombuffer(bytes(text), np.uint8)
        nb = int(text.numel() if hasattr(text, "numel") else len(text))
        chr_b = chr_name.encode() if chr_name else None
        nr, nbs = ctypes.c_uint64(0), ctypes.c_uint64(0)
        if out is None:
            st = lib().gsnp_parse_soap(self.h, _ptr(text), nb, chr_b, q_offset, loc_base,
                                       *([None] * 7), 0, 0, ctypes.byref(nr), ctypes.byref(nbs))
            if st not in (0, -7):
                _check(st, self.h)
            R, B = int(nr.value), int(nbs.value)
            spec = dict(pos=(R, "uint64"), len=(R, "uint16"), off=(R + 1, "uint64"),
                        bases=(B, "uint8"), quals=(B, "uint8"), strand=(R, "uint8"),
                        hits=(R, "uint16"))
            if device:
                import torch
                out = {k: torch.empty(max(n, 1), dtype=getattr(torch, d), device="cuda")
                       for k, (n, d) in spec.items()}
            else:
                out = {k: np.zeros(max(n, 1), d) for k, (n, d) in spec.items()}
        cap_r = int(out["pos"].numel() if hasattr(out["pos"], "numel") else len(out["pos"]))
        cap_b = int(out["bases"].numel() if hasattr(out["bases"], "numel") else len(out["bases"]))
        _check(lib().gsnp_parse_soap(self.h, _ptr(text), nb, chr_b, q_offset, loc_base,
                                     *[_ptr(out[k]) for k in ("pos", "len", "off", "bases", "quals",
                                                              "strand", "hits")],
                                     cap_r, cap_b, ctypes.byref(nr), ctypes.byref(nbs)), self.h)
        R, B = int(nr.value), int(nbs.value)
        return {k: v[:(R + 1 if k == "off" else B if k in ("bases", "quals") else R)]
                for k, v in out.items()}

    def compress(self, rec, block_sites: int = 65536, out=None):
        """§V-B compression of records (numpy RECORD_DTYPE array, or a CUDA uint8 tensor of
        40*n bytes).  out: None (numpy uint32 result, sized by a query call) or a uint32 buffer
        (numpy or CUDA tensor); returns (out, n_words)."""
        n = (rec.numel() // 40) if hasattr(rec, "numel") else len(rec)
        nw = ctypes.c_uint64(0)
        if out is None:
            st = lib().gsnp_compress(self.h, _ptr(rec), n, block_sites, None, 0, ctypes.byref(nw))
            if st not in (0, -7):
                _check(st, self.h)
            out = np.zeros(int(nw.value), np.uint32)
        cap = out.numel() if hasattr(out, "numel") else len(out)
        _check(lib().gsnp_compress(self.h, _ptr(rec), n, block_sites, _ptr(out), cap,
                                   ctypes.byref(nw)), self.h)
        return out[:int(nw.value)], int(nw.value)

    def call_compressed(self, reads, w0: int, w1: int, out, block_sites: int = 65536):
        """gsnp_call + gsnp_compress with the records kept on the device; out: uint32 buffer
        (numpy or CUDA tensor).  Returns the number of words written."""
        r = reads if isinstance(reads, gsnp_reads) else make_reads(reads)
        cap = out.numel() if hasattr(out, "numel") else len(out)
        nw = ctypes.c_uint64(0)
        _check(lib().gsnp_call_compressed(self.h, ctypes.byref(r), w0, w1, block_sites, _ptr(out),
                                          cap, ctypes.byref(nw)), self.h)
        return int(nw.value)

    def debug_window(self, reads: dict, w0: int, w1: int,
                     want=("off", "keys_built", "keys_sorted", "counters", "L10", "post10",
                           "records")):
        """gsnp_debug_window into host arrays; only the parts named in `want` are returned."""
        S = w1 - w0
        nb = int(reads["off"][-1]) - int(reads["off"][0]) if len(reads["off"]) else 0
        make = dict(off=lambda: np.zeros(S + 1, np.uint32),
                    keys_built=lambda: np.zeros(max(nb, 1), np.uint32),
                    keys_sorted=lambda: np.zeros(max(nb, 1), np.uint32),
                    counters=lambda: np.zeros((S, 15), np.uint32), L10=lambda: np.zeros((S, 10)),
                    post10=lambda: np.zeros((S, 10)), records=lambda: np.zeros(S, RECORD_DTYPE))
        out = {k: make[k]() for k in want}
        if ("keys_built" in out or "keys_sorted" in out) and "off" not in out:
            out["off"] = make["off"]()
        r = make_reads(reads)
        g = (lambda k: _ptr(out[k]) if k in out else None)
        _check(lib().gsnp_debug_window(self.h, ctypes.byref(r), w0, w1, g("off"), g("keys_built"),
                                       g("keys_sorted"), g("counters"), g("L10"), g("post10"),
                                       g("records")), self.h)
        if "off" in out:
            K = int(out["off"][-1])
            for k in ("keys_built", "keys_sorted"):
                if k in out:
                    out[k] = out[k][:K]
        return out

    def call_async(self, r: gsnp_reads, w0: int, w1: int, out):
        """gsnp_call_async: device reads (a gsnp_reads from make_reads) and a device uint8 tensor
        of >= 40*(w1-w0) bytes; no host round trip (errors surface at wait())."""
        _check(lib().gsnp_call_async(self.h, ctypes.byref(r), w0, w1, _ptr(out),
                                     _nbytes(out) // 40), self.h)

    def wait(self):
        _check(lib().gsnp_wait(self.h), self.h)

    def unpack_reads(self, packed, out=None):
        """gsnp_unpack_reads: a packed stream (numpy / pinned or CUDA tensor) -> device read
        arrays (dict of CUDA tensors; allocated when out is None)."""
        import torch
        n_reads, n_bases = packed_sizes(packed)
        if out is None:
            dev = "cuda"
            out = dict(pos=torch.empty(n_reads, dtype=torch.uint64, device=dev),
                       len=torch.empty(n_reads, dtype=torch.uint16, device=dev),
                       off=torch.empty(n_reads + 1, dtype=torch.uint64, device=dev),
                       bases=torch.empty(max(n_bases, 1), dtype=torch.uint8, device=dev),
                       quals=torch.empty(max(n_bases, 1), dtype=torch.uint8, device=dev),
                       strand=torch.empty(n_reads, dtype=torch.uint8, device=dev),
                       hits=torch.empty(n_reads, dtype=torch.uint16, device=dev))
        nb = _nbytes(packed)
        _check(lib().gsnp_unpack_reads(self.h, _ptr(packed), nb, *[_ptr(out[k]) for k in
                                       ("pos", "len", "off", "bases", "quals", "strand", "hits")]),
               self.h)
        return out

    def get_tables(self, calibrated: bool = True):
        dims = np.zeros(3, np.uint32)
        _check(lib().gsnp_get_tables(self.h, None, None, None, None, _ptr(dims)), self.h)
        L, P, G = (int(x) for x in dims)
        adj = np.zeros(64 * P * G, np.uint8)
        out = dict(L=L, adjP=P, adjG=G)
        if calibrated:
            counts = np.zeros(64 * 256 * 16, np.uint64)
            p = np.zeros(64 * 256 * 16)
            T = np.zeros(64 * L * 40)
            _check(lib().gsnp_get_tables(self.h, _ptr(counts), _ptr(p), _ptr(T), _ptr(adj), None),
                   self.h)
            out.update(counts=counts.reshape(64, 256, 4, 4), p=p.reshape(64, 256, 4, 4),
                       T=T.reshape(64, L, 4, 10))
        else:
            _check(lib().gsnp_get_tables(self.h, None, None, None, _ptr(adj), None), self.h)
        out["adj"] = adj.reshape(64, P, G)
        return out

    def launch_count(self) -> int:
        return int(lib().gsnp_launch_count(self.h))

    def stage_times(self, reset: bool = False) -> dict:
        """{stage: (ms, launches)} accumulated with GSNP_TIMING (CUDA events in the library)."""
        ms = np.zeros(len(STAGES))
        n = np.zeros(len(STAGES), np.uint64)
        _check(lib().gsnp_stage_times(self.h, _ptr(ms), _ptr(n), len(STAGES), int(reset)), self.h)
        return {k: (float(ms[i]), int(n[i])) for i, k in enumerate(STAGES)}


# ABI-named free functions (thin aliases)
def _nbytes(a) -> int:
    if hasattr(a, "element_size"):
        return a.numel() * a.element_size()
    return np.asarray(a).nbytes


def pack_reads(reads: dict, block_reads: int = 1024, ref=None, origin: int = 0) -> np.ndarray:
    """gsnp_pack_reads: host read arrays -> the packed stream R21 (numpy uint8); with ref (the
    reference codes the reads are aligned to, origin = coordinate of ref[0]) version 2."""
    r = make_reads(reads)
    rr = None
    if ref is not None:
        refa = np.ascontiguousarray(ref, np.uint8)
        rr = gsnp_reference(_ptr(refa), len(refa), int(origin))
        rr._keep = refa
    n = ctypes.c_uint64(0)
    rp = ctypes.byref(rr) if rr is not None else None
    st = lib().gsnp_pack_reads(ctypes.byref(r), rp, block_reads, None, 0, ctypes.byref(n))
    if st not in (0, -7):
        _check(st, None)
    out = np.zeros(max(int(n.value), 1), np.uint8)
    _check(lib().gsnp_pack_reads(ctypes.byref(r), rp, block_reads, _ptr(out), out.nbytes,
                                 ctypes.byref(n)), None)
    return out[:int(n.value)]


def packed_sizes(packed) -> tuple:
    """(n_reads, n_bases) of a packed stream (its header is read from host memory)."""
    hdr = packed[:128]
    if hasattr(hdr, "cpu"):
        hdr = hdr.cpu().numpy()
    hdr = np.ascontiguousarray(hdr, np.uint8)
    a, b = ctypes.c_uint64(0), ctypes.c_uint64(0)
    _check(lib().gsnp_packed_sizes(_ptr(hdr), _nbytes(packed), ctypes.byref(a), ctypes.byref(b)), None)
    return int(a.value), int(b.value)


def gsnp_create(ref, origin=0, known_pos=None, known_prior10=None, **params) -> Context:
    return Context(ref, origin, known_pos, known_prior10, **params)


def gsnp_calibrate(ctx: Context, reads):
    return ctx.calibrate(reads)


def gsnp_calibrate_count(ctx: Context, reads, counts=None):
    return ctx.calibrate_count(reads, counts)


def gsnp_calibrate_finalize(ctx: Context, counts):
    return ctx.calibrate_finalize(counts)


def gsnp_call(ctx: Context, reads, w0, w1, out=None):
    return ctx.call(reads, w0, w1, out)


def gsnp_compress(ctx: Context, rec, block_sites=65536, out=None):
    return ctx.compress(rec, block_sites, out)


def gsnp_call_compressed(ctx: Context, reads, w0, w1, out, block_sites=65536):
    return ctx.call_compressed(reads, w0, w1, out, block_sites)


def gsnp_call_dense(ctx: Context, reads, w0, w1, out=None, chunk_sites=16384):
    return ctx.call_dense(reads, w0, w1, out, chunk_sites)


def gsnp_priors_from_freq(freq, floor_prior: float = 5e-7) -> np.ndarray:
    """Known-SNP prior rows (n x 10) from allele frequencies (n x 4, A C T G), reading R18."""
    f = np.ascontiguousarray(freq, np.float64).reshape(-1, 4)
    out = np.zeros((len(f), 10), np.float64)
    _check(lib().gsnp_priors_from_freq(_ptr(f), len(f), float(floor_prior), _ptr(out)), None)
    return out


def gsnp_parse_soap(ctx: Context, text, chr_name=None, q_offset=33, loc_base=0, device=True):
    return ctx.parse_soap(text, chr_name, q_offset, loc_base, device)


def gsnp_debug_window(ctx: Context, reads, w0, w1):
    return ctx.debug_window(reads, w0, w1)


def gsnp_get_tables(ctx: Context):
    return ctx.get_tables()


def gsnp_destroy(ctx: Context):
    ctx.close()
