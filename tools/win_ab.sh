#!/bin/bash
# windowed-call A/B: bench.py's windowed leg (C2) for the default build and $1
for i in 1 2; do
  for L in default "$1"; do
    if [ "$L" = default ]; then unset GSNP_LIB; else export GSNP_LIB=$PWD/$L; fi
    timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu --no-dense --no-parse 2>/dev/null | tail -1 | \
      python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$L', d['ms_per_step'], [(w['window_sites'], round(w['ms_per_step'],2), round(w['vs_one_window'],3)) for w in d['windowed']])"
  done
done
unset GSNP_LIB
