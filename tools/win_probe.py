"""Windowed-calling probe: python tools/win_probe.py CFG WIN [timing]  — ms per pass over the shard."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_icpp_luzlwfl11_b200 import gsnp  # noqa: E402

cfg, WIN = sys.argv[1], int(sys.argv[2])
timing = len(sys.argv) > 3
w = synth.generate(cfg)
lo, hi = w["region"]
dev = {k: torch.from_numpy(np.ascontiguousarray(w[k])).cuda()
       for k in ("pos", "len", "off", "bases", "quals", "strand", "hits")}
flags = gsnp.GSNP_RANK_SUM | (gsnp.GSNP_TIMING if timing else 0)
ctx = gsnp.Context.from_workload(w, stream=torch.cuda.current_stream(), flags=flags)
ctx.calibrate(dev)
out = torch.empty(40 * (hi - lo), dtype=torch.uint8, device="cuda")
wins = [(a, min(hi, a + WIN)) for a in range(lo, hi, WIN)]
rds = []
for a, b in wins:
    ra, rb = synth.read_range(w, a, b)
    rds.append(gsnp.make_reads(dict(dev, pos=dev["pos"][ra:rb], len=dev["len"][ra:rb],
                                    off=dev["off"][ra:rb + 1], strand=dev["strand"][ra:rb],
                                    hits=dev["hits"][ra:rb])))
import time
for rep in range(3):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    e0.record()
    for (a, b), r in zip(wins, rds):
        ctx.call_async(r, a, b, out[40 * (a - lo):40 * (b - lo)])
    t1 = time.perf_counter()
    e1.record()
    ctx.wait()
    print(f"{cfg} win={WIN} windows={len(wins)} gpu_ms={e0.elapsed_time(e1):.2f} host_enqueue_ms={1e3 * (t1 - t0):.2f}")
