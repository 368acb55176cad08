"""Run the hot path once on a (scaled) config for ncu: python tools/profile_call.py C2 4800000"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_icpp_luzlwfl11_b200 import gsnp  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C2"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 4_800_000
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
w = synth.generate(synth.CONFIGS[name].scaled(n_sites=n))
dev = {k: torch.from_numpy(np.ascontiguousarray(w[k])).cuda()
       for k in ("pos", "len", "off", "bases", "quals", "strand", "hits")}
ctx = gsnp.Context.from_workload(w, flags=gsnp.GSNP_RANK_SUM | gsnp.GSNP_TIMING)
counts = torch.zeros(64 * 256 * 16, dtype=torch.uint64, device="cuda")
ctx.calibrate_count(dev, counts)
ctx.calibrate_finalize(counts)
out = torch.empty(40 * n, dtype=torch.uint8, device="cuda")
rd = gsnp.make_reads(dev)
for _ in range(reps):
    ctx.call_reads(rd, 0, n, out)
torch.cuda.synchronize()
print(ctx.stage_times())
