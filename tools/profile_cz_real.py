"""§V-B compression of real records (a whole C2 call) for ncu / timing:
python tools/profile_cz_real.py [config] [n_sites] [block_sites] [reps] [chunks]"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_icpp_luzlwfl11_b200 import gsnp  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C2"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 48_000_000
B = int(sys.argv[3]) if len(sys.argv) > 3 else 32768
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 3
chunks = int(sys.argv[5]) if len(sys.argv) > 5 else 1
w = synth.generate(synth.CONFIGS[name].scaled(n_sites=n))
dev = {k: torch.from_numpy(np.ascontiguousarray(w[k])).cuda()
       for k in ("pos", "len", "off", "bases", "quals", "strand", "hits")}
ctx = gsnp.Context.from_workload(w, flags=gsnp.GSNP_RANK_SUM | gsnp.GSNP_TIMING)
counts = torch.zeros(64 * 256 * 16, dtype=torch.uint64, device="cuda")
ctx.calibrate_count(dev, counts)
ctx.calibrate_finalize(counts)
rec = torch.empty(40 * n, dtype=torch.uint8, device="cuda")
rd = gsnp.make_reads(dev)
ctx.call_reads(rd, 0, n, rec)
nw = gsnp.ctypes.c_uint64(0)
gsnp.lib().gsnp_compress(ctx.h, gsnp._ptr(rec), n, B, None, 0, gsnp.ctypes.byref(nw))
out = torch.empty(int(nw.value) + 1024, dtype=torch.int32, device="cuda")
ref, _ = ctx.compress(rec, B, out)
ref = ref.cpu().clone()
torch.cuda.synchronize()
ctx.stage_times(reset=True)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
step = (n + chunks - 1) // chunks
e0.record()
for _ in range(reps):
    for c in range(chunks):
        a, b = c * step, min(n, (c + 1) * step)
        ctx.compress(rec[40 * a:40 * b], B, out)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / reps
print({"n": n, "B": B, "chunks": chunks, "words": int(nw.value), "ratio": 40 * n / (4 * int(nw.value)),
       "ms": round(ms, 3), "kernel_ms": round(ctx.stage_times()["compress"][0] / reps, 3),
       "crc": int(np.bitwise_xor.reduce(ref.numpy().view(np.uint32)))})
