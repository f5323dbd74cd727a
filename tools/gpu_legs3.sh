#!/bin/bash
# refresh every bench leg with the current code (results table)
mkdir -p gpurun_out/legs
python __graft_entry__.py > /dev/null 2>&1
timeout 900 python bench.py > gpurun_out/legs/bench.json 2> gpurun_out/legs/bench.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/legs/bench.json'));print('C2', round(d['value'],1), round(d['roofline']['frac'],4), 'e2e', round(d['e2e']['value'],2), 'hidden', round(d['overlap']['hidden_frac'],3), 'e2e_roof', round(d['e2e_roofline']['frac'],3), 'sync', round(d['sync_baseline_e2e']['value'],2))"
timeout 1200 python bench.py --config c3 --steps 2 --warmup 1 > gpurun_out/legs/c3.json 2> gpurun_out/legs/c3.err; echo "c3 rc=$?"
python -c "import json;d=json.load(open('gpurun_out/legs/c3.json'));print('C3', d['value'], d['roofline'].get('frac'))"
timeout 900 python bench.py --config c4 --no-cpu-baseline > gpurun_out/legs/c4.json 2> gpurun_out/legs/c4.err; echo "c4 rc=$?"
python -c "import json;d=json.load(open('gpurun_out/legs/c4.json'));print('C4', d['value'], d['roofline'].get('frac'), d.get('e2e',{}).get('value'))"
timeout 900 python bench.py --config c5 --no-cpu-baseline > gpurun_out/legs/c5.json 2> gpurun_out/legs/c5.err; echo "c5 rc=$?"
python -c "import json;d=json.load(open('gpurun_out/legs/c5.json'));print('C5', d['value'], d['roofline'].get('frac'), d['e2e'])"
timeout 1500 python bench.py --config fig5 --sweep 1,10,16,32,48,64,100,1000 > gpurun_out/legs/fig5.json 2>/dev/null; echo "fig5 rc=$?"
python -c "import json;d=json.load(open('gpurun_out/legs/fig5.json'));print({T:(round(r['tiled']['ms'],2),round(r['sync']['ms'],2),round(r['sync_pageable']['ms'],2)) for T,r in d['sweep'].items()})"
timeout 1200 python bench.py --config fig8 > gpurun_out/legs/fig8.json 2> gpurun_out/legs/fig8.err; echo "fig8 rc=$?"; head -c 600 gpurun_out/legs/fig8.json
