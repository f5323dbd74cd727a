#!/bin/bash
# persistent multi-step heat7: GPU tests, A/B bench (TILES_PERSIST=1/0)
mkdir -p gpurun_out/pers
python __graft_entry__.py > /dev/null 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/pers/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/pers/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pers/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pers/pytest_gpu.log
for v in 1 0 1 0; do
TILES_PERSIST=$v timeout 600 python bench.py --no-cpu-baseline --no-extras > gpurun_out/pers/bench_p$v.json 2>gpurun_out/pers/bench_p$v.err
python -c "import json;d=json.load(open('gpurun_out/pers/bench_p$v.json'));print('persist=$v', round(d['value'],1), round(d['roofline']['frac'],4), round(d['roofline']['avg_launch_ms'],3), d['gpu_launches'], 'e2e', round(d['e2e']['value'],2))"
done
