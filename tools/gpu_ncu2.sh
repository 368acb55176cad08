#!/bin/bash
# usage: tools/gpu_ncu2.sh TAG REGEX SKIP CONFIG NSITES — ncu --set full of the (SKIP+1)-th matching launch
TAG=$1; RX=$2; SKIP=$3; CFG=${4:-C2}; NS=${5:-4800000}
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"$RX" --launch-skip $SKIP -c 1 \
    -o gpurun_out/full_${TAG} python tools/profile_call.py $CFG $NS 1 > gpurun_out/full_${TAG}.log 2>&1
echo "ncu rc=$?"; tail -3 gpurun_out/full_${TAG}.log
