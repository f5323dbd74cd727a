#!/bin/bash
# C2 e2e (stream-through) vs unit size / thin end units (env knobs of runtime.cpp)
mkdir -p gpurun_out/stsweep
python __graft_entry__.py > /dev/null 2>&1
for cfg in "3 16" "0 16" "5 16" "3 32" "6 32" "3 16"; do
  set -- $cfg
  TILES_ST_THIN=$1 TILES_ST_MINUNIT=$2 timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 10 > gpurun_out/stsweep/t$1_u$2.json 2>/dev/null
  python -c "import json;j=json.load(open('gpurun_out/stsweep/t$1_u$2.json'));print('thin',$1,'minunit',$2,'e2e ms',round(j['e2e']['ms_per_step'],3),'val',round(j['value'],1))"
done
