#!/bin/bash
# compute-sanitizer over the small GPU cases (round 2 selection: parity paths, edges incl. contract
# violations and short reads, packed-read decode, async windows, compression).
mkdir -p gpurun_out
rm -f gpurun_out/sanitize_summary.txt
SEL='c1_window or listed_sites or depth_classes or deep_pile or edge_cases or empty_reads or variable_length or short_reads or one_bp or contract or pile_inside or oracle_stream or bad_stream or async_errors or compress_matches or call_compressed'
for tool in memcheck synccheck initcheck racecheck; do
  FILES="tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_pack.py tests/test_gpu_windows.py tests/test_gpu_compress.py"
  K="$SEL"
  if [ $tool = racecheck ]; then K='c1_window or deep_pile or short_reads or oracle_stream or listed_sites'; fi
  timeout 2400 compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 50 \
      python -m pytest $FILES -m gpu -x -q -p no:cacheprovider -k "$K" \
      > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?" | tee -a gpurun_out/sanitize_summary.txt
  grep -E "ERROR SUMMARY|RACECHECK SUMMARY|passed|failed" gpurun_out/sanitize_$tool.log | tail -3 | tee -a gpurun_out/sanitize_summary.txt
done
