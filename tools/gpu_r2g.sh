#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_windows.py tests/test_gpu_parity.py -x -q > gpurun_out/pytest_g.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_g.log
tail -15 gpurun_out/pytest_g.log
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu --no-dense --no-parse > gpurun_out/bench_g_C2.json 2> gpurun_out/bench_g_C2.err
python tools/bsum.py gpurun_out/bench_g_C2.json; tail -3 gpurun_out/bench_g_C2.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_g_C2.json').read().strip().splitlines()[-1]); print(d['windowed'])"
