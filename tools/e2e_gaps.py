"""Where the e2e calls phase loses time: per API call, host wall time and device span
(events on the library stream).  python tools/e2e_gaps.py [K]"""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_icpp_luzlwfl11_b200 import gsnp  # noqa: E402

K = int(sys.argv[1]) if len(sys.argv) > 1 else 2
w = synth.generate("C2")
S = len(w["ref"])
dev = {k: torch.from_numpy(np.ascontiguousarray(w[k])).cuda()
       for k in ("pos", "len", "off", "bases", "quals", "strand", "hits")}
stream = torch.cuda.current_stream()
ctx = gsnp.Context.from_workload(w, stream=stream, flags=gsnp.GSNP_RANK_SUM | gsnp.GSNP_TIMING)
ctx.calibrate(dev)
rd = gsnp.make_reads(dev)
zcap = 11 * (S // K + 1) + 4096
z = torch.empty(K * zcap, dtype=torch.int32, device="cuda")
cut = [S * i // K for i in range(K + 1)]
for rep in range(3):
    torch.cuda.synchronize()
    ctx.stage_times(reset=True)
    evs, host = [], []
    for j in range(K):
        e0 = torch.cuda.Event(enable_timing=True); e0.record(stream)
        t0 = time.perf_counter()
        nw = ctx.call_compressed(rd, cut[j], cut[j + 1], z[j * zcap:(j + 1) * zcap])
        host.append((time.perf_counter() - t0) * 1e3)
        e1 = torch.cuda.Event(enable_timing=True); e1.record(stream)
        evs.append((e0, e1))
    torch.cuda.synchronize()
    spans = [a.elapsed_time(b) for a, b in evs]
    gaps = [evs[i][1].elapsed_time(evs[i + 1][0]) for i in range(K - 1)]
    st = {k: round(v[0], 3) for k, v in ctx.stage_times(reset=True).items() if v[1]}
    print(f"rep {rep}: host ms {[round(h, 3) for h in host]} device spans {[round(s, 3) for s in spans]} "
          f"gaps {[round(g, 3) for g in gaps]} stages {st}")
