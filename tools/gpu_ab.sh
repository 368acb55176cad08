#!/bin/bash
# A/B: tools/gpu_ab.sh "C2 48000000" lib1.so ...
mkdir -p gpurun_out
CFGN=$1; shift
python - "$CFGN" "$@" <<'PY' 2>&1 | tee gpurun_out/ab.txt
import os, subprocess, sys, re
cfg, n = sys.argv[1].split()
libs = ["default"] + sys.argv[2:]
for rep in range(2):
    for L in libs:
        env = dict(os.environ)
        if L != "default":
            env["GSNP_LIB"] = os.path.abspath(L)
        out = subprocess.run([sys.executable, "tools/profile_call.py", cfg, n, "3"], env=env,
                             capture_output=True, text=True).stdout.strip().splitlines()
        d = eval(out[-1]) if out else {}
        ct = d.get("call_tile", (0, 1)); ws = d.get("warp_sites", (0, 1)); cc = d.get("calib_count", (0, 1))
        print(f"{cfg} {L:22s} call (3 variants) {3*ct[0]/max(ct[1],1):8.3f} ms  warp_sites {ws[0]/max(ws[1],1):8.3f} ms  calib {cc[0]/max(cc[1],1):7.3f} ms", flush=True)
PY
