#!/bin/bash
# Full measurement pass on the GPU box: tests, bench, ncu launch list, ncu full capture.
# usage: tools/gpu_measure.sh TAG
TAG=${1:-r1}
mkdir -p gpurun_out
bash tools/gpu_check.sh
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err
tail -1 gpurun_out/bench_${TAG}.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_${TAG}.csv python bench.py --steps 2 --warmup 1 --no-cpu \
    > gpurun_out/launches_${TAG}.log 2>&1
echo "launches rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_call_tile|k_calib_count" -c 2 \
    -o gpurun_out/full_${TAG} python tools/profile_call.py C2 48000000 2 > gpurun_out/full_${TAG}.log 2>&1
echo "full rc=$?"
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_parse_meta|k_parse_emit|k_nl_tiles" -c 4 \
    -o gpurun_out/parse_${TAG} python tools/profile_parse.py C2 > gpurun_out/parse_${TAG}.log 2>&1
echo "parse rc=$?"
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_dense" -c 2 \
    -o gpurun_out/dense_${TAG} python tools/profile_dense.py 200000 > gpurun_out/dense_${TAG}.log 2>&1
echo "dense rc=$?"
