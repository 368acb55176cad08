"""SOAP-text parse of a (scaled) config for ncu / timing: python tools/profile_parse.py C2 [n_sites]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_icpp_luzlwfl11_b200 import gsnp  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C2"
n = int(sys.argv[2]) if len(sys.argv) > 2 else synth.CONFIGS[name].n_sites
w = synth.generate(synth.CONFIGS[name].scaled(n_sites=n))
text = torch.frombuffer(bytearray(synth.soap_text(w, "chr1", 33)), dtype=torch.uint8).cuda()
ctx = gsnp.Context.from_workload(w, flags=gsnp.GSNP_RANK_SUM | gsnp.GSNP_TIMING)
out = ctx.parse_soap(text, "chr1", 33, int(w["origin"]))
for _ in range(3):
    ctx.parse_soap(text, "chr1", 33, int(w["origin"]), out=out)
torch.cuda.synchronize()
st = ctx.stage_times()["parse"]
print({"text_bytes": int(text.numel()), "parse_kernel_ms_per_call": st[0] / 4, "launch_groups": st[1]})
