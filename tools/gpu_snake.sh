#!/bin/bash
# snake order across the steps of a persistent launch: parity, then C2 value A/B
mkdir -p gpurun_out/snake
python __graft_entry__.py > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q -k "resident or c2 or c1 or runs_continue or edge or shapes or stream_counts or dirichlet or sine or zero_work or kernel_timing" > gpurun_out/snake/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/snake/pytest.log
for cfg in "1 16" "0 0" "1 0" "1 32" "1 16" "0 0" "1 8" "1 48"; do
  set -- $cfg
  TILES_SNAKE=$1 TILES_SNAKE_KEEP=$2 timeout 300 python bench.py --no-cpu-baseline --no-extras --steps 20 > gpurun_out/snake/s$1_k$2.json 2>/dev/null
  python -c "import json;j=json.load(open('gpurun_out/snake/s$1_k$2.json'));print('snake',$1,'keep',$2,'value',round(j['value'],1),'frac',round(j['roofline']['frac'],4),'ms',round(j['roofline']['avg_launch_ms'],4))"
done
