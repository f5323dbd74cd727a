#!/bin/bash
# headline bench + Fig. 5 sweep + C5, for the results table
mkdir -p gpurun_out/res
timeout 900 python bench.py > gpurun_out/res/bench.json 2> gpurun_out/res/bench.err; echo "bench rc=$?"; cat gpurun_out/res/bench.json | head -c 1500; echo
timeout 1500 python bench.py --config fig5 --sweep 1,10,16,32,48,64,100,1000 > gpurun_out/res/fig5.json 2>/dev/null; echo "fig5 rc=$?"
python -c "import json;d=json.load(open('gpurun_out/res/fig5.json'));print({T:(round(r['tiled']['ms'],2),round(r['sync']['ms'],2),round(r['sync_pageable']['ms'],2)) for T,r in d['sweep'].items()})"
timeout 900 python bench.py --config c5 --no-cpu-baseline > gpurun_out/res/c5.json 2>/dev/null; echo "c5 rc=$?"; python -c "import json;d=json.load(open('gpurun_out/res/c5.json'));print(d['value'], d['e2e'])"
