#!/bin/bash
# A/B of stream-through unit/copy knobs on the C2 e2e step (alternating rounds).
O=gpurun_out/s2d
mkdir -p $O
for rnd in 1 2 3; do
  for cfg in "A:" "B:TILES_ST_MINUNIT=32 TILES_ST_H2D_MERGE=1" "C:TILES_ST_MINUNIT=32 TILES_ST_H2D_MERGE=1 TILES_ST_OFFSET=1" "D:TILES_ST_H2D_MERGE=1 TILES_ST_OFFSET=1"; do
    name=${cfg%%:*}; envs=${cfg#*:}
    env $envs timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 20 > $O/ab_${name}_$rnd.json 2>/dev/null
    python -c "
import json; d=json.load(open('$O/ab_${name}_$rnd.json')); print('$name', $rnd, round(d['value'],2), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'launch_us', round(d['roofline']['avg_launch_ms']*1e3,1))"
  done
done
