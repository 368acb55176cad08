#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py -x -q > gpurun_out/pytest_f.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_f.log
tail -3 gpurun_out/pytest_f.log
for cfg in "C3 31000000" "C2 48000000" "C5 5000000"; do
  for envs in "GSNP_MID_AT=1000" "GSNP_MID_AT=24" "GSNP_MID_AT=24 GSNP_MID_ADJ_SMEM=1" "GSNP_MID_AT=20" ; do
    echo "$cfg $envs: $(env $envs python tools/profile_call.py $cfg 3 2>/dev/null | tail -1 | python -c "
import sys; d=eval(sys.stdin.read()); f=lambda k: round(d[k][0]/max(d[k][1],1),3)
print('call_tile(sum of 3 variants)', round(d['call_tile'][0]/3,3), 'warp', f('warp_sites'), 'big', f('big_sites'))")"
  done
done
