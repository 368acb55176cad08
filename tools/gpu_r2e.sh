#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_pack.py -x -q > gpurun_out/pytest_e.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_e.log
tail -15 gpurun_out/pytest_e.log
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu --no-dense --no-parse > gpurun_out/bench_e_C2.json 2> gpurun_out/bench_e_C2.err
python tools/bsum.py gpurun_out/bench_e_C2.json; tail -3 gpurun_out/bench_e_C2.err
python -c "
import json; d=json.loads(open('gpurun_out/bench_e_C2.json').read().strip().splitlines()[-1]); e=d['e2e']
print({k: e[k] for k in ('value','ms_per_step','h2d_bytes_per_step','d2h_bytes_per_step','check')}); print(e['breakdown_ms']); print('raw', e['raw_input']['value'], e['raw_input']['ms_per_step'])"
