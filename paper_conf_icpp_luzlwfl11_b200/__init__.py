"""paper_conf_icpp_luzlwfl11_b200 — B200-native (sm_100a) GSNP hot path.

GSNP (Lu et al., ICPP 2011): SOAPsnp-model per-site genotype likelihood and consensus calling.
The compute path lives in ``libgsnp.so`` (CUDA kernels + C ABI, include/gsnp.h); this package is
its ctypes binding and build helper.  See DESIGN.md.
"""
from .gsnp import (Context, GsnpError, RECORD_DTYPE, SYMBOLS, gsnp_calibrate,  # noqa: F401
                   gsnp_calibrate_count, gsnp_calibrate_finalize, gsnp_call, gsnp_create,
                   gsnp_debug_window, gsnp_destroy, gsnp_get_tables, lib, make_reads,
                   params_default)
