#!/bin/bash
# Box facts + a quick state check (tests, smoke, bench without the CPU legs).
mkdir -p gpurun_out
{ nproc; lscpu | head -20; free -g; nvidia-smi; } > gpurun_out/box.txt 2>&1
bash tools/gpu_check.sh
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu --no-dense --no-parse > gpurun_out/bench_probe.json 2> gpurun_out/bench_probe.err
tail -c 600 gpurun_out/bench_probe.json
