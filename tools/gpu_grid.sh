#!/bin/bash
mkdir -p gpurun_out/grid
python __graft_entry__.py > /dev/null 2>&1
for gcap in 0 128 0 128 64; do
  TILES_HEAT_GRID=$gcap timeout 300 python bench.py --no-cpu-baseline --no-extras --steps 20 > gpurun_out/grid/g$gcap.json 2>/dev/null
  python -c "import json;j=json.load(open('gpurun_out/grid/g$gcap.json'));print('grid cap',$gcap,'value',round(j['value'],1),'frac',round(j['roofline']['frac'],4))"
done
TILES_HEAT_GRID=128 STEPS=4 timeout 900 ncu --set full --clock-control none -k regex:heat7_fixed -s 8 -c 1 -o gpurun_out/grid/g128 -f python tools/prof_heat.py > /dev/null 2>&1; echo ncu rc=$?
