#!/bin/bash
# usage: tools/gpu_ncu1.sh TAG REGEX CONFIG NSITES  — one ncu --set full capture of a kernel
TAG=$1; RX=$2; CFG=${3:-C2}; NS=${4:-4800000}
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"$RX" -c 1 \
    -o gpurun_out/full_${TAG} python tools/profile_call.py $CFG $NS 1 > gpurun_out/full_${TAG}.log 2>&1
echo "ncu rc=$?"; tail -3 gpurun_out/full_${TAG}.log
