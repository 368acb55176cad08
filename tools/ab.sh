#!/bin/bash
# A/B timing of library builds: tools/ab.sh CONFIG NSITES lib1.so lib2.so ...  (default lib first)
CFG=$1; N=$2; shift 2
echo "default: $(python tools/profile_call.py $CFG $N 3 2>/dev/null | head -1)"
for L in "$@"; do
  echo "$L: $(GSNP_LIB=$PWD/$L python tools/profile_call.py $CFG $N 3 2>/dev/null | head -1)"
done
