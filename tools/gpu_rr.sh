#!/bin/bash
# round-robin band order (HeatParams::rr_rounds): parity, then C5 / C2 A/B
mkdir -p gpurun_out/rr
python __graft_entry__.py > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q > gpurun_out/rr/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/rr/pytest.log
for rr in 1 0 1 0; do
  TILES_HEAT_RR=$rr timeout 600 python bench.py --config c5 --steps 6 --no-cpu-baseline > gpurun_out/rr/c5_rr$rr.json 2>/dev/null
  python -c "import json;j=json.load(open('gpurun_out/rr/c5_rr$rr.json'));print('C5 rr',$rr,'value',round(j['value'],1),'frac',round(j['roofline']['frac'],3),'e2e',round(j['e2e']['value'],1))"
done
for rr in 1 0; do
  TILES_HEAT_RR=$rr timeout 300 python bench.py --no-cpu-baseline --no-extras --steps 10 > gpurun_out/rr/c2_rr$rr.json 2>/dev/null
  python -c "import json;j=json.load(open('gpurun_out/rr/c2_rr$rr.json'));print('C2 rr',$rr,'value',round(j['value'],1),'frac',round(j['roofline']['frac'],3))"
done
