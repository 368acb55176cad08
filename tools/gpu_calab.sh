#!/bin/bash
# calibration A/B: parity tests that check counts, then C2 / C5 timings of the default build vs $@
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_fullsize.py -m gpu -x -q 2>&1 | tail -3
bash tools/gpu_ab.sh "C2 48000000" "$@"
