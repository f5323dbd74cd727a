#!/bin/bash
# C5 shape (tiles 256 wide): persistent / direct A/B, resident value only
mkdir -p gpurun_out/c5ab
python __graft_entry__.py > /dev/null 2>&1
for cfg in "1 1" "0 1" "0 0" "1 1"; do
set -- $cfg
TILES_PERSIST=$1 TILES_DIRECT=$2 timeout 900 python bench.py --config c5 --no-cpu-baseline --no-extras > gpurun_out/c5ab/c5.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/c5ab/c5.json'));print('persist=$1 direct=$2', round(d['value'],1), round(d['roofline']['frac'],4), d['roofline'].get('kernel'))"
done
