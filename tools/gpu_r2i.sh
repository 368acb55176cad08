#!/bin/bash
mkdir -p gpurun_out
timeout 1200 compute-sanitizer --tool initcheck --error-exitcode 99 --print-limit 20 python -m pytest tests/test_gpu_edges.py tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider -k "contract or c1_window or short_reads or errors" > gpurun_out/sanitize_initcheck2.log 2>&1
echo "initcheck rc=$?"; grep -E "ERROR SUMMARY|passed|failed" gpurun_out/sanitize_initcheck2.log | tail -3
bash tools/gpu_ab.sh "C2 48000000" build/sg3.so build/sg4.so build/cl1.so build/cl8.so build/nopre.so build/pf.so build/pfnopre.so
