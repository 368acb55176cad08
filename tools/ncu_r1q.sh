mkdir -p gpurun_out
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches_r1q.csv python bench.py --steps 2 --warmup 1 --no-cpu \
    > gpurun_out/launches_r1q.log 2>&1
echo "launches rc=$?"
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_call_tile|k_calib_count" -c 2 \
    -o gpurun_out/full_r1q python tools/profile_call.py C2 48000000 2 > gpurun_out/full_r1q.log 2>&1
echo "full rc=$?"
