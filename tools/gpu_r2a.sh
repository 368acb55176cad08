#!/bin/bash
mkdir -p gpurun_out
./tools/l2_gather_peak > gpurun_out/l2q.json 2> gpurun_out/l2q.err; cat gpurun_out/l2q.json gpurun_out/l2q.err
timeout 900 python -m pytest tests/test_gpu_edges.py tests/test_gpu_parity.py -x -q > gpurun_out/pytest_edges.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_edges.log
tail -15 gpurun_out/pytest_edges.log
