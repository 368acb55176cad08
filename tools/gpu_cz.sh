#!/bin/bash
# compression timing + launch list on real C2 records: tools/gpu_cz.sh TAG [B]
TAG=${1:-cz}; B=${2:-32768}
mkdir -p gpurun_out
python tools/profile_cz_real.py C2 48000000 $B 3 1 | tee gpurun_out/cz_${TAG}.txt
python tools/profile_cz_real.py C2 48000000 $B 3 4 | tee -a gpurun_out/cz_${TAG}.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_cz" --csv \
  --log-file gpurun_out/cz_${TAG}_launches.csv python tools/profile_cz_real.py C2 48000000 $B 1 1 > /dev/null 2>&1
python tools/launches.py gpurun_out/cz_${TAG}_launches.csv
