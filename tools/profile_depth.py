"""Like profile_call.py at a chosen depth: python tools/profile_depth.py CONFIG DEPTH NSITES [REPS]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_icpp_luzlwfl11_b200 import gsnp  # noqa: E402

name, depth, n = sys.argv[1], float(sys.argv[2]), int(sys.argv[3])
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 3
w = synth.generate(synth.CONFIGS[name].scaled(n_sites=n, depth=depth))
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
d = ctx.stage_times()
print({k: round(v[0] / reps, 3) for k, v in d.items() if k in ("call_tile", "warp_sites")},
      "sum", round((d["call_tile"][0] + d["warp_sites"][0]) / reps, 3))
