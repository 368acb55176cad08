#!/bin/bash
# Full round check: all GPU tests + smoke + the default bench line (+ C5 line).
TAG=${1:-r2}
mkdir -p gpurun_out
bash tools/gpu_tests.sh
timeout 1200 python bench.py --steps 20 --warmup 3 > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err
python tools/bsum.py gpurun_out/bench_${TAG}.json; tail -2 gpurun_out/bench_${TAG}.err
timeout 900 python bench.py --config C5 --steps 20 --warmup 3 --no-dense --no-parse > gpurun_out/bench_${TAG}_c5.json 2> gpurun_out/bench_${TAG}_c5.err
python tools/bsum.py gpurun_out/bench_${TAG}_c5.json; tail -2 gpurun_out/bench_${TAG}_c5.err
