#!/bin/bash
# Full GPU test suite (+ smoke), parity report of the exhaustive full-size tests.
mkdir -p gpurun_out
rm -f gpurun_out/parity_report.jsonl
export GSNP_PARITY_REPORT=gpurun_out/parity_report.jsonl
timeout 1800 python -m pytest tests -m gpu -x -q -s -p no:cacheprovider > gpurun_out/pytest_all.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_all.log
grep -E "passed|failed|error|\[fullsize\]" gpurun_out/pytest_all.log | tail -12
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
tail -2 gpurun_out/smoke.log
