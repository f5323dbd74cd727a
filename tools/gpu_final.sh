#!/bin/bash
# round-end refresh: smoke, all GPU tests, headline bench x2, ncu launch list + full capture
mkdir -p gpurun_out/final
python __graft_entry__.py > /dev/null 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/final/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/final/smoke.log
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/final/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/final/pytest_gpu.log
for i in 1 2; do
timeout 600 python bench.py > gpurun_out/final/bench$i.json 2> gpurun_out/final/bench$i.err; echo "bench rc=$?"
python -c "import json; j=json.load(open('gpurun_out/final/bench$i.json')); print('value', round(j['value'],1), 'frac', round(j['roofline']['frac'],3), 'e2e', round(j['e2e']['value'],2), 'e2e_roof', round(j['e2e_roofline']['frac'],3), 'hidden', round(j['overlap']['hidden_frac'],3), 'h2d', round(j['e2e_roofline']['pcie_gbs']['h2d'],1), 'clk', j['clocks']['sm_mhz'], j['clocks']['reasons'])"
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/final/launches.csv python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-extras \
  > gpurun_out/final/ncu_launch_bench.log 2>&1; echo "launch list rc=$?"
STEPS=4 timeout 900 ncu --set full --clock-control none --import-source on -k regex:heat7_fixed -s 8 -c 1 \
  -o gpurun_out/final/heat7_persistent_full -f python tools/prof_heat.py > gpurun_out/final/ncu_full.log 2>&1; echo "full rc=$?"; tail -1 gpurun_out/final/ncu_full.log
