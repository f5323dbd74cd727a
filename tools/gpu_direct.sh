#!/bin/bash
# direct ghosts + stacked z-march: GPU tests, A/B bench, ncu of heat7 (cache control all/none)
mkdir -p gpurun_out/dir
python __graft_entry__.py > /dev/null 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/dir/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/dir/smoke.log
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/dir/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/dir/pytest_gpu.log
for v in 1 0 1 0; do
TILES_DIRECT=$v timeout 600 python bench.py --no-cpu-baseline --no-extras > gpurun_out/dir/bench_d$v.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/dir/bench_d$v.json'));print('direct=$v', round(d['value'],1), round(d['roofline']['frac'],4), round(d['roofline']['avg_launch_ms']*1000,1), 'e2e', round(d['e2e']['value'],1))"
done
for cc in all none; do
timeout 900 ncu --set full --clock-control none --cache-control $cc --import-source on -k regex:heat7 -s 10 -c 1 \
  -o gpurun_out/dir/heat7_direct_cc$cc -f python tools/prof_heat.py > gpurun_out/dir/ncu_$cc.log 2>&1; echo "ncu $cc rc=$?"
done
