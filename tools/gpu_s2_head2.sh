#!/bin/bash
O=gpurun_out/s2o
mkdir -p $O
for rnd in 1 2 3 4 5 6 7 8; do
  for h in 2 4; do
    TILES_ST_HEAD=$h timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 20 > $O/h${h}_$rnd.json 2>/dev/null
    python -c "
import json; d=json.load(open('$O/h${h}_$rnd.json')); print('head=$h', $rnd, round(d['value'],2), round(d['ms_per_step'],3))"
  done
done
