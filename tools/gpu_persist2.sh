#!/bin/bash
# persistent kernel cost breakdown: deps off (invalid results, timing only) vs on vs separate launches
mkdir -p gpurun_out/pers2
python __graft_entry__.py > /dev/null 2>&1
for cfg in "1 2" "1 18" "0 2" "1 2" "1 18" "0 2"; do
set -- $cfg
TILES_PERSIST=$1 TILES_HEAT_CACHE=$2 timeout 600 python bench.py --no-cpu-baseline --no-extras > gpurun_out/pers2/b.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/pers2/b.json'));print('persist=$1 flags=$2', round(d['value'],1), round(d['ms_per_step'],3), round(d['roofline']['avg_launch_ms'],3))"
done
