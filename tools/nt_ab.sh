#!/bin/bash
# C2 / C5 k_call_tile timing of the default build (and of extra builds passed as arguments)
for cfg in "C2 48000000" "C5 5000000"; do
  echo "$cfg default: $(python tools/profile_call.py $cfg 3 2>/dev/null | head -1 | sed -E 's/.*call_tile.: \(([0-9.]+), ([0-9]+)\).*warp_sites.: \(([0-9.]+), ([0-9]+)\).*/call_tile \1 warp \3/')"
  for L in "$@"; do
    echo "$cfg $L: $(GSNP_LIB=$PWD/$L python tools/profile_call.py $cfg 3 2>/dev/null | head -1 | sed -E 's/.*call_tile.: \(([0-9.]+), ([0-9]+)\).*warp_sites.: \(([0-9.]+), ([0-9]+)\).*/call_tile \1 warp \3/')"
  done
done
