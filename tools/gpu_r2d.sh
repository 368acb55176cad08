#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cluster.py tests/test_gpu_edges.py tests/test_gpu_priors.py -x -q > gpurun_out/pytest_d.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_d.log
tail -4 gpurun_out/pytest_d.log
timeout 900 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_d_C2.json 2> gpurun_out/bench_d_C2.err
python tools/bsum.py gpurun_out/bench_d_C2.json; tail -3 gpurun_out/bench_d_C2.err
timeout 900 python bench.py --config C3 --steps 5 --warmup 3 --no-cpu > gpurun_out/bench_d_C3.json 2> gpurun_out/bench_d_C3.err
python tools/bsum.py gpurun_out/bench_d_C3.json; tail -3 gpurun_out/bench_d_C3.err
GSNP_BENCH_BACKEND=gloo GSNP_BENCH_SAME_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --config C3 --steps 3 --warmup 3 --no-cpu > gpurun_out/bench_d_C3_n2.json 2> gpurun_out/bench_d_C3_n2.err
python tools/bsum.py gpurun_out/bench_d_C3_n2.json; tail -3 gpurun_out/bench_d_C3_n2.err
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/bench_d_ref.json 2> gpurun_out/bench_d_ref.err
python tools/bsum.py gpurun_out/bench_d_ref.json; tail -3 gpurun_out/bench_d_ref.err
