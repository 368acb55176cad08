"""Dense ablation (gsnp_call_dense) vs sparse on a C2 sub-window, for ncu / timing:
python tools/profile_dense.py [n_sites]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_icpp_luzlwfl11_b200 import gsnp  # noqa: E402

n = int(sys.argv[1]) if len(sys.argv) > 1 else 2_000_000
w = synth.generate(synth.CONFIGS["C2"].scaled(n_sites=n, n_lead_frac=0.0))
dev = {k: torch.from_numpy(np.ascontiguousarray(w[k])).cuda()
       for k in ("pos", "len", "off", "bases", "quals", "strand", "hits")}
ctx = gsnp.Context.from_workload(w, flags=gsnp.GSNP_RANK_SUM | gsnp.GSNP_TIMING)
ctx.calibrate(dev)
out = torch.empty(40 * n, dtype=torch.uint8, device="cuda")
ctx.call_dense(dev, 0, n, out, chunk_sites=16384)
torch.cuda.synchronize()
print({k: v for k, v in ctx.stage_times().items() if v[1]})
