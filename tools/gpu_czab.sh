#!/bin/bash
# compression A/B on real C2 records: tools/gpu_czab.sh lib1.so ... (default first)
for L in "" "$@"; do
  echo "lib=${L:-default}: $(GSNP_LIB=${L:+$PWD/$L} python tools/profile_cz_real.py C2 48000000 32768 3 1)"
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_cz" --csv --log-file gpurun_out/cz_ab_launches.csv python tools/profile_cz_real.py C2 48000000 32768 1 1 > /dev/null 2>&1
python tools/launches.py gpurun_out/cz_ab_launches.csv | tail -6
