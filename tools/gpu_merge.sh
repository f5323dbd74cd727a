#!/bin/bash
# C2 e2e (stream-through) vs units per H2D copy; parity of the merged schedule
mkdir -p gpurun_out/merge
python __graft_entry__.py > /dev/null 2>&1
for m in 1 2 3 4 2 1; do
  TILES_ST_H2D_MERGE=$m timeout 300 python bench.py --no-cpu-baseline --steps 10 > gpurun_out/merge/m$m.json 2>/dev/null
  python -c "import json;j=json.load(open('gpurun_out/merge/m$m.json'));print('merge',$m,'e2e ms',round(j['e2e']['ms_per_step'],3),'hidden',round(j['overlap']['hidden_frac'],3),'xo',round(j['overlap']['t_xfer_only_ms'],2),'co',round(j['overlap']['t_comp_only_ms'],2),'frac',round(j['e2e_roofline']['frac'],3),'h2d',round(j['e2e_roofline']['pcie_gbs']['h2d'],1))"
done
for m in 2 4; do TILES_ST_H2D_MERGE=$m timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "stream_through or c1 or c2_full" 2>&1 | tail -1; done
TILES_ST_H2D_MERGE=2 timeout 300 python tools/timeline.py c2 gpurun_out/merge/tl_m2 > /dev/null 2>&1; tail -c 600 gpurun_out/merge/tl_m2.summary.json
