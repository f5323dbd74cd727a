#!/bin/bash
# after persistent launch: GPU tests, launch list of the bench, full captures of one
# whole-domain step (TILES_PERSIST=0) and of a persistent 4-step launch
mkdir -p gpurun_out/prof2
python __graft_entry__.py > /dev/null 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/prof2/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/prof2/pytest_gpu.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/prof2/launches.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-extras \
  > gpurun_out/prof2/ncu_launch_bench.log 2>&1; echo "launch list rc=$?"
TILES_PERSIST=0 timeout 900 ncu --set full --clock-control none --import-source on -k regex:heat7 -s 10 -c 1 \
  -o gpurun_out/prof2/heat7_full -f python tools/prof_heat.py > gpurun_out/prof2/ncu_full.log 2>&1; echo "full rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:heat7 -s 9 -c 1 \
  -o gpurun_out/prof2/heat7_persistent_full -f python tools/prof_heat.py > gpurun_out/prof2/ncu_full_p.log 2>&1; echo "full persistent rc=$?"
