#!/bin/bash
mkdir -p gpurun_out/tune
python __graft_entry__.py > /dev/null 2>&1
for cfg in "64 4" "64 5" "64 6" "32 6" "32 4" "64 4"; do
  set -- $cfg
  TILES_HEAT_BAND=$1 TILES_HEAT_STAGES=$2 timeout 300 python bench.py --no-cpu-baseline --no-extras --steps 20 > gpurun_out/tune/b$1_s$2.json 2>/dev/null
  python -c "import json;j=json.load(open('gpurun_out/tune/b$1_s$2.json'));print('band',$1,'stages',$2,'value',round(j['value'],1),'frac',round(j['roofline']['frac'],4))"
done
for k in 24 64 96; do
  TILES_SNAKE_KEEP=$k timeout 300 python bench.py --no-cpu-baseline --no-extras --steps 20 > gpurun_out/tune/k$k.json 2>/dev/null
  python -c "import json;j=json.load(open('gpurun_out/tune/k$k.json'));print('keep',$k,'value',round(j['value'],1),'frac',round(j['roofline']['frac'],4))"
done
