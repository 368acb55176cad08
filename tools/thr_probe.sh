# 32-slot (+ k_list_sites) vs 64-slot kernel by depth: per-call ms of call + warp stages
for d in 26 30 34 38 42 48; do
  for env in "GSNP_MID_AT=200" "GSNP_MID_AT=1"; do
    echo "C3 depth $d [$env] $(env $env python tools/profile_depth.py C3 $d 24000000 2 2>/dev/null | tail -1)"
  done
done
