#!/bin/bash
# Round-2 profiles: launch list of the bench command + ncu --set full captures (C2 shallow call,
# calibration; C5 deep call).  Summaries are written by tools/ncu_summary.py into profiles/.
TAG=${1:-r2}
mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_${TAG}.csv python bench.py --steps 2 --warmup 1 --no-cpu \
    > gpurun_out/launches_${TAG}.log 2>&1
echo "launches rc=$?"
# first gsnp_call of profile_call: k_call_tile launches 32-slot, 64-slot, 128-slot in that order
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_call_tile|k_calib_count" -c 2 \
    -o gpurun_out/full_${TAG} python tools/profile_call.py C2 48000000 1 > gpurun_out/full_${TAG}.log 2>&1
echo "full rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_call_tile" --launch-skip 2 -c 1 \
    -o gpurun_out/full_${TAG}_c5 python tools/profile_call.py C5 5000000 1 > gpurun_out/full_${TAG}_c5.log 2>&1
echo "c5 rc=$?"
