#!/bin/bash
for i in 1 2; do for th in 1 0; do
TILES_ST_THIN=$th timeout 300 python bench.py --no-cpu-baseline > gpurun_out/b_th$th.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/b_th$th.json'));print('thin=$th', round(d['e2e']['value'],2), round(d['e2e']['ms_per_step'],2))"
done; done
