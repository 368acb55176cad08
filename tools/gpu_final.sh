#!/bin/bash
# Final round-2 measurements: full GPU suite + smoke, default bench (C2), C5, C3 (one GPU, strong
# mode), C3 over two ranks sharing the GPU (flow check, gloo), and the reference arm.
TAG=${1:-r2}
mkdir -p gpurun_out
bash tools/gpu_tests.sh
cp gpurun_out/parity_report.jsonl gpurun_out/parity_${TAG}.jsonl 2>/dev/null
timeout 1200 python bench.py > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err
python tools/bsum.py gpurun_out/bench_${TAG}.json; tail -2 gpurun_out/bench_${TAG}.err
timeout 900 python bench.py --config C5 --no-dense --no-parse > gpurun_out/bench_${TAG}_c5.json 2> gpurun_out/bench_${TAG}_c5.err
python tools/bsum.py gpurun_out/bench_${TAG}_c5.json; tail -2 gpurun_out/bench_${TAG}_c5.err
timeout 1500 python bench.py --config C3 --steps 5 --warmup 3 --no-cpu > gpurun_out/bench_${TAG}_c3.json 2> gpurun_out/bench_${TAG}_c3.err
python tools/bsum.py gpurun_out/bench_${TAG}_c3.json; tail -2 gpurun_out/bench_${TAG}_c3.err
GSNP_BENCH_BACKEND=gloo GSNP_BENCH_SAME_GPU=1 timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --config C3 --steps 3 --warmup 3 --no-cpu > gpurun_out/bench_${TAG}_c3_n2_samegpu.json 2> gpurun_out/bench_${TAG}_c3_n2_samegpu.err
python tools/bsum.py gpurun_out/bench_${TAG}_c3_n2_samegpu.json; tail -2 gpurun_out/bench_${TAG}_c3_n2_samegpu.err
timeout 900 python bench.py --impl reference > gpurun_out/bench_${TAG}_ref.json 2> gpurun_out/bench_${TAG}_ref.err
tail -c 400 gpurun_out/bench_${TAG}_ref.json; tail -2 gpurun_out/bench_${TAG}_ref.err
