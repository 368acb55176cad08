#!/bin/bash
# ncu --set full + per-source-line summary of the C2 hot kernels: tools/gpu_lines.sh TAG
TAG=${1:-x}
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_call_tile|k_calib_count" -c 2 \
    -o gpurun_out/full_${TAG} python tools/profile_call.py C2 48000000 1 > gpurun_out/full_${TAG}.log 2>&1
echo "ncu rc=$?"
python tools/ncu_lines.py gpurun_out/full_${TAG}.ncu-rep 60 > gpurun_out/lines_${TAG}.txt 2>&1
ls -la gpurun_out/
