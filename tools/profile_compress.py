"""Run the §V-B compressor on a C2-sized record table for ncu / timing:
python tools/profile_compress.py [n_records] [block_sites] [reps]"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_icpp_luzlwfl11_b200 import gsnp  # noqa: E402
from tests._records import records  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 48_000_000
B = int(sys.argv[2]) if len(sys.argv) > 2 else 65536
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
r = records(n, seed=11)
ctx = gsnp.Context(np.zeros(16, np.uint8), flags=gsnp.GSNP_TIMING)
rd = torch.from_numpy(r.view(np.uint8)).cuda()
nw = gsnp.ctypes.c_uint64(0)
gsnp.lib().gsnp_compress(ctx.h, gsnp._ptr(rd), n, B, None, 0, gsnp.ctypes.byref(nw))
out = torch.empty(int(nw.value), dtype=torch.int32, device="cuda")
ctx.compress(rd, B, out)
ctx.stage_times(reset=True)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(reps):
    ctx.compress(rd, B, out)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / reps
print({"n": n, "B": B, "words": int(nw.value), "ratio": 40 * n / (4 * int(nw.value)), "ms": ms,
       "kernel_ms": ctx.stage_times()["compress"][0] / reps})
