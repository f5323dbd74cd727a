#!/bin/bash
# GPU error-contract tests, then A/B of the sweep store policy (TILES_SWEEP_ST 0 vs 2) on the
# C2 e2e step, five alternating rounds, and the Fig. 5 stream-through Ts.
O=gpurun_out/s2g
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || { tail -20 $O/build.txt; exit 1; }
timeout 600 python -m pytest tests/test_errors.py tests/test_host_regions.py -m gpu -q 2>&1 | tail -5 | tee $O/tests.txt
for rnd in 1 2 3 4 5; do
  for cfg in "A:TILES_SWEEP_ST=0" "C:TILES_SWEEP_ST=2"; do
    name=${cfg%%:*}; envs=${cfg#*:}
    env $envs timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 20 > $O/ab_${name}_$rnd.json 2>/dev/null
    python -c "
import json; d=json.load(open('$O/ab_${name}_$rnd.json')); print('$name', $rnd, round(d['value'],2), round(d['ms_per_step'],3), 'frac', round(d['roofline']['frac'],3), 'pipe', round(d['roofline'].get('frac_in_pipeline',0),3))"
  done
done
for cfg in "A:TILES_SWEEP_ST=0" "C:TILES_SWEEP_ST=2"; do
  name=${cfg%%:*}; envs=${cfg#*:}
  env $envs timeout 600 python bench.py --config fig5 --steps 5 --warmup 3 --sweep 1,10,16,32 > $O/fig5_${name}.json 2>/dev/null
  python -c "
import json; d=json.load(open('$O/fig5_${name}.json'))
print('$name', {k: round(v['tiled']['ms'],2) for k,v in d['sweep'].items()})"
done
