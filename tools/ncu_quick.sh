#!/bin/bash
# ncu --set full of one kernel (regex $1) on a C2 call: tools/ncu_quick.sh REGEX TAG [NSITES]
mkdir -p gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"$1" -c 1 \
    -o gpurun_out/full_$2 python tools/profile_call.py C2 ${3:-48000000} 1 > gpurun_out/full_$2.log 2>&1
echo "ncu rc=$?"
