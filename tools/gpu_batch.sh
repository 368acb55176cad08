#!/bin/bash
# One GPU call: new-feature tests, the full gpu suite, A/B of knob builds, bench.
# usage: tools/gpu_batch.sh TAG [ab-libs...]
TAG=${1:-x}; shift
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_dense.py tests/test_gpu_priors.py tests/test_gpu_parse.py -x -q \
    > gpurun_out/new_${TAG}.log 2>&1; echo "new rc=$?" >> gpurun_out/new_${TAG}.log; tail -15 gpurun_out/new_${TAG}.log
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_${TAG}.log 2>&1; echo "all rc=$?" >> gpurun_out/pytest_${TAG}.log; tail -3 gpurun_out/pytest_${TAG}.log
if [ $# -gt 0 ]; then timeout 900 bash tools/ab.sh C2 48000000 "$@" > gpurun_out/ab_${TAG}.txt 2>&1; cat gpurun_out/ab_${TAG}.txt; fi
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err
tail -1 gpurun_out/bench_${TAG}.json; tail -3 gpurun_out/bench_${TAG}.err
