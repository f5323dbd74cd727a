#!/bin/bash
mkdir -p gpurun_out/legs
python __graft_entry__.py > /dev/null 2>&1
timeout 1500 python bench.py --config fig5 --sweep 1,10,16,32,48,64,100,1000 > gpurun_out/legs/fig5.json 2>/dev/null; echo "fig5 rc=$?"
python -c "import json;d=json.load(open('gpurun_out/legs/fig5.json'));print({T:(round(r['tiled']['ms'],2),round(r['sync']['ms'],2),round(r['sync_pageable']['ms'],2)) for T,r in d['sweep'].items()})"
timeout 1500 python bench.py --config c3 --steps 2 --warmup 1 > gpurun_out/legs/c3.json 2>/dev/null; echo "c3 rc=$?"
python -c "import json;j=json.load(open('gpurun_out/legs/c3.json'));print('C3',round(j['value'],1),j['roofline']['frac'],j['overlap']['hidden_frac'])"
timeout 1500 python bench.py --config c4 --steps 3 --warmup 1 > gpurun_out/legs/c4.json 2>/dev/null; echo "c4 rc=$?"
python -c "import json;j=json.load(open('gpurun_out/legs/c4.json'));print('C4',round(j['value'],2),j['roofline']['frac'],j.get('overlap'))"
