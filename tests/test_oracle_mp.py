"""The multi-process oracle runner (tests/_mp.py) reproduces the single-process oracle exactly."""
from __future__ import annotations

import numpy as np

import oracle
import synth
from tests._mp import calib_parallel, call_parallel


def test_parallel_oracle_equals_single_process():
    w = synth.generate("C1", n_sites=30_000, depth=15.0, seed=5)
    P = oracle.Params()
    C1 = oracle.calib_counts(P, w)
    C4, _ = calib_parallel(P, w, procs=4)
    assert np.array_equal(C1, C4)
    p = oracle.p_matrix(P, C1)
    rec, dbg = oracle.call_window(P, w, p, 0, 30_000, debug=True)
    rec4, L4, post4, st = call_parallel(P, w, p, 0, 30_000, want_L10=True, want_post=True,
                                        procs=4, chunk=3_001)
    assert rec4.tobytes() == rec.tobytes()
    assert np.array_equal(L4, dbg["L10"]) and np.array_equal(post4, dbg["post10"])
    assert st["procs"] == 4 and st["cpu_s"] > 0
