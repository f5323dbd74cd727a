#!/bin/bash
O=gpurun_out/s2m
mkdir -p $O
for rnd in 1 2 3; do
  for ts in 0 1; do
    timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 20 --two-step $ts > $O/ts${ts}_$rnd.json 2>/dev/null
    python -c "
import json; d=json.load(open('$O/ts${ts}_$rnd.json')); r=d['roofline']; print('two_step=$ts', $rnd, round(d['value'],2), round(d['ms_per_step'],3), r.get('kernel'), 'frac', round(r['frac'],3), 'launch_us', round(r['avg_launch_ms']*1e3,2), 'B/launch', r.get('algorithmic_bytes_per_launch'))"
  done
done
