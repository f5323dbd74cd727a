#!/bin/bash
# (experiment script: the knob it sets was measured and reverted; kept as the record of the A/B)
# Chained tile-column sweeps: parity (stream-through / wavefront / random shapes / full size),
# repeated to shake out races, then A/B chain on/off on the C2 e2e step.
O=gpurun_out/s2i
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || { tail -20 $O/build.txt; exit 1; }
for i in 1 2 3; do
  timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -q -x -k "stream_through or wavefront or random or fullsize or c2 or split" 2>&1 | tail -4 | tee -a $O/tests.txt
done
for rnd in 1 2 3; do
  for cfg in "A:TILES_SWEEP_CHAIN=0" "B:TILES_SWEEP_CHAIN=1"; do
    name=${cfg%%:*}; envs=${cfg#*:}
    env $envs timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 20 > $O/ab_${name}_$rnd.json 2>/dev/null
    python -c "
import json; d=json.load(open('$O/ab_${name}_$rnd.json')); r=d['roofline']; print('$name', $rnd, round(d['value'],2), round(d['ms_per_step'],3), 'frac', round(r['frac'],3), 'launch_us', round(r['avg_launch_ms']*1e3,2), 'pipe', round(r.get('frac_in_pipeline') or 0,3))"
  done
done
