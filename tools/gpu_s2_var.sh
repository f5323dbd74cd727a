#!/bin/bash
# (experiment script: the knob it sets was measured and reverted; kept as the record of the A/B)
# A/B of tile-column sweep variants (TILES_SWEEP_VAR) on the C2 e2e step, alternating rounds.
O=gpurun_out/s2h
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || { tail -20 $O/build.txt; exit 1; }
for rnd in 1 2; do
  for v in 0 1 2 3 4 5; do
    TILES_SWEEP_VAR=$v timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 20 > $O/var${v}_$rnd.json 2>/dev/null
    python -c "
import json; d=json.load(open('$O/var${v}_$rnd.json')); print('var$v', $rnd, round(d['value'],2), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'launch_us', round(d['roofline']['avg_launch_ms']*1e3,2))"
  done
done
