#!/bin/bash
# A/B of the tile-column sweep's L2 policies (TILES_SWEEP_ST stores, TILES_SWEEP_LD staged loads)
# on the C2 e2e step (dominant-kernel roofline from comp-only interval events), alternating rounds.
O=gpurun_out/s2e
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || { tail -20 $O/build.txt; exit 1; }
for rnd in 1 2 3; do
  for cfg in "A:" "B:TILES_SWEEP_ST=1" "C:TILES_SWEEP_ST=2" "D:TILES_SWEEP_LD=1" "E:TILES_SWEEP_ST=1 TILES_SWEEP_LD=1" "F:TILES_SWEEP_ST=2 TILES_SWEEP_LD=1"; do
    name=${cfg%%:*}; envs=${cfg#*:}
    env $envs timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 20 > $O/ab_${name}_$rnd.json 2>/dev/null
    python -c "
import json; d=json.load(open('$O/ab_${name}_$rnd.json')); print('$name', $rnd, round(d['value'],2), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'launch_us', round(d['roofline']['avg_launch_ms']*1e3,2))"
  done
done
