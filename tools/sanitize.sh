#!/bin/bash
# compute-sanitizer (memcheck / racecheck / synccheck / initcheck) over the small GPU parity
# cases: every k_call_tile path (thread 16/32, thread-deep, warp, warp-deep, CTA), calibration,
# tile ranges, validation and the compressor.  SURVEY.md §4 tier 5.  Runs on the GPU box.
mkdir -p gpurun_out
SEL=${SEL:-'c1_window or depth_classes or deep_pile or edge_cases or empty_reads or variable_length or compress_matches or adversarial or call_compressed'}
for tool in ${TOOLS:-memcheck racecheck synccheck initcheck}; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 50 \
      python -m pytest tests/test_gpu_parity.py tests/test_gpu_compress.py ${EXTRA} -m gpu -x -q -p no:cacheprovider -k "$SEL" \
      > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?" | tee -a gpurun_out/sanitize_summary.txt
  grep -E "ERROR SUMMARY|passed|failed" gpurun_out/sanitize_$tool.log | tail -3 | tee -a gpurun_out/sanitize_summary.txt
done
