#!/bin/bash
for envs in "GSNP_E2E_CZ_B=65536" "GSNP_E2E_CZ_B=32768" "GSNP_E2E_CZ_B=16384" "GSNP_E2E_CZ_B=32768 GSNP_E2E_CHUNKS=2" "GSNP_E2E_CZ_B=32768 GSNP_E2E_CHUNKS=4"; do
  env $envs timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu --no-dense --no-parse > gpurun_out/bench_czb.json 2>/dev/null
  echo "$envs: $(python -c "
import json; d=json.loads(open('gpurun_out/bench_czb.json').read().strip().splitlines()[-1]); e=d['e2e']
print(round(e['ms_per_step'],2), 'ms', round(e['value']/1e9,3), 'G', e['d2h_bytes_per_step'], e['breakdown_ms']['call_spans'], e['breakdown_ms']['device_stage_ms'].get('compress'))")"
done
