# k_call_tile variant thresholds: per-call stage ms (call_tile sums its three instantiations)
for i in 1 2; do
for cfg in "C5 5000000" "C3 48000000"; do
  for env in "" "GSNP_DEEP_AT=1000" "GSNP_DEEP_AT=20"; do
    echo "$cfg [$env] $(env $env python tools/profile_call.py $cfg 3 2>/dev/null | tail -1 | python -c "
import sys; d=eval(sys.stdin.read()); print({k: round(v[0]/3, 3) for k, v in d.items() if k in ('call_tile','warp_sites','big_sites')})")"
  done
done
done
