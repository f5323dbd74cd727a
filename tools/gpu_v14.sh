#!/bin/bash
mkdir -p gpurun_out/v14
python __graft_entry__.py > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/v14/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/v14/pytest_gpu.log
for i in 1 2; do
timeout 600 python bench.py > gpurun_out/v14/bench$i.json 2> gpurun_out/v14/bench$i.err; echo "bench rc=$?"
python -c "import json; j=json.load(open('gpurun_out/v14/bench$i.json')); print('value', round(j['value'],1), 'frac', round(j['roofline']['frac'],3), 'e2e', round(j['e2e']['value'],2), 'e2e_roof', round(j['e2e_roofline']['frac'],3), 'hidden', round(j['overlap']['hidden_frac'],3), 'h2d', round(j['e2e_roofline']['pcie_gbs']['h2d'],1), 'clk', j['clocks']['sm_mhz'], j['clocks']['reasons'], j['clocks_e2e']['reasons'])"
done
timeout 900 python bench.py --config c5 --steps 6 --no-cpu-baseline > gpurun_out/v14/c5.json 2>/dev/null; echo "c5 rc=$?"
python -c "import json;j=json.load(open('gpurun_out/v14/c5.json'));print('C5 value',round(j['value'],1),'frac',round(j['roofline']['frac'],3),'e2e',round(j['e2e']['value'],1))"
