"""Multi-process runs of the CPU oracle (test infrastructure): P independent single-threaded oracle
processes, each over a contiguous range of windows, as SURVEY.md §8(d)'s timing protocol
describes for the large configs — used for exhaustive full-size parity and by bench.py's
cpu_baseline / --impl reference legs.  Workers are forked after the workload is built (the read
arrays are shared copy-on-write) and write their records / likelihoods into shared memory."""
from __future__ import annotations

import mmap
import multiprocessing as mp
import os
import time

import numpy as np

import oracle
import synth

_W = None           # the workload, visible to forked workers
_JOB = None


def _shared(shape, dtype):
    dtype = np.dtype(dtype)
    n = int(np.prod(shape)) * dtype.itemsize
    buf = mmap.mmap(-1, max(n, 1), flags=mmap.MAP_SHARED | mmap.MAP_ANONYMOUS)
    return np.frombuffer(buf, dtype=dtype, count=int(np.prod(shape))).reshape(shape)


def _work_call(task):
    a, b = task
    P, p, w0, rec, L10, post, L = _JOB
    t0 = time.process_time()
    ra, rb = synth.read_range(_W, a, b, L)
    sub = synth.slice_reads(_W, ra, rb)
    want = tuple(k for k, v in (("L10", L10), ("post10", post)) if v is not None)
    out = {"rec": rec[a - w0:b - w0]}
    if L10 is not None:
        out["L10"] = L10[a - w0:b - w0]
    if post is not None:
        out["post10"] = post[a - w0:b - w0]
    oracle.call_window(P, sub, p, a, b, debug=bool(want), want=want, out=out)
    return time.process_time() - t0


def _work_calib(task):
    ra, rb = task
    P = _JOB
    t0 = time.process_time()
    C = oracle.calib_counts(P, synth.slice_reads(_W, ra, rb))
    return C, time.process_time() - t0


def nproc() -> int:
    return max(1, len(os.sched_getaffinity(0)) if hasattr(os, "sched_getaffinity") else os.cpu_count())


def call_parallel(P, w, p, w0: int, w1: int, want_L10=False, want_post=False, procs=None,
                  chunk=None):
    """Oracle records (and optionally L10 / post10) for sites [w0, w1) from `procs` single-threaded
    processes.  Returns (rec, L10, post10, stats) with stats = {procs, wall_s, cpu_s}."""
    global _W, _JOB
    procs = procs or nproc()
    S = w1 - w0
    rec = _shared((S,), oracle.RECORD_DTYPE)
    L10 = _shared((S, 10), np.float64) if want_L10 else None
    post = _shared((S, 10), np.float64) if want_post else None
    chunk = chunk or max(50_000, -(-S // (procs * 8)))
    tasks = [(a, min(w1, a + chunk)) for a in range(w0, w1, chunk)]
    _W, _JOB = w, (P, p, w0, rec, L10, post, P.max_read_len)
    t0 = time.perf_counter()
    if procs == 1:
        cpu = sum(_work_call(t) for t in tasks)
    else:
        with mp.get_context("fork").Pool(procs) as pool:
            cpu = sum(pool.map(_work_call, tasks, chunksize=1))
    wall = time.perf_counter() - t0
    _W, _JOB = None, None
    return rec, L10, post, {"procs": procs, "wall_s": wall, "cpu_s": cpu, "sites": S}


def calib_parallel(P, w, procs=None):
    """Oracle calibration counts over all reads of w, summed over `procs` processes (integer
    sums: identical to one pass).  Returns (C, stats)."""
    global _W, _JOB
    procs = procs or nproc()
    n = len(w["pos"])
    k = max(1, min(procs * 4, n // 1000 + 1))
    cuts = [n * i // k for i in range(k + 1)]
    tasks = [(cuts[i], cuts[i + 1]) for i in range(k) if cuts[i + 1] > cuts[i]]
    _W, _JOB = w, P
    t0 = time.perf_counter()
    if procs == 1 or len(tasks) <= 1:
        res = [_work_calib(t) for t in tasks]
    else:
        with mp.get_context("fork").Pool(procs) as pool:
            res = pool.map(_work_calib, tasks, chunksize=1)
    wall = time.perf_counter() - t0
    _W, _JOB = None, None
    C = np.zeros((64, 256, 4, 4), np.uint64)
    for c, _ in res:
        C += c
    return C, {"procs": procs, "wall_s": wall, "cpu_s": sum(t for _, t in res)}
