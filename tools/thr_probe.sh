# k_call_tile variant thresholds: per-call stage ms (call_tile sums its three instantiations)
for i in 1 2; do
  for pair in "C2 48000000|" "C2 48000000|GSNP_MID_AT=10" "C3 48000000|" "C3 48000000|GSNP_MID_AT=40"; do
    cfg=${pair%%|*}; env=${pair#*|}
    echo "$cfg [$env] $(env $env python tools/profile_call.py $cfg 3 2>/dev/null | tail -1 | python -c "
import sys; d=eval(sys.stdin.read()); print({k: round(v[0]/3, 3) for k, v in d.items() if k in ('call_tile','warp_sites','big_sites')})")"
  done
done
