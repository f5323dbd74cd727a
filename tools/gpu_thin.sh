#!/bin/bash
# e2e A/B: thin head/tail units (TILES_ST_THIN=3) vs uniform units (0)
mkdir -p gpurun_out/thin
python __graft_entry__.py > /dev/null 2>&1
for v in 3 0 3 0 3 0 3 0; do
TILES_ST_THIN=$v timeout 600 python bench.py --no-cpu-baseline --no-extras --steps 30 > gpurun_out/thin/bench_t$v.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/thin/bench_t$v.json'));print('thin=$v', round(d['value'],1), 'e2e', round(d['e2e']['value'],2), round(d['e2e']['ms_per_step'],2))"
done
python tools/timeline.py c2 gpurun_out/thin/c2st > /dev/null 2>&1; echo tl rc=$?
