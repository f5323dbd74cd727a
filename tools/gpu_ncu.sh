#!/bin/bash
# ncu: launch list of the bench command + one full capture of a whole-domain heat7_tma launch.
mkdir -p gpurun_out
python __graft_entry__.py > /dev/null 2>&1
if [ "${LAUNCHES:-1}" = "1" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv \
  --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-extras \
  > gpurun_out/ncu_launch_bench.log 2>&1; echo "launch list rc=$?"
fi
timeout 900 ncu --set full --clock-control none --import-source on -k regex:heat7 -s 10 -c 1 \
  -o gpurun_out/heat7_full -f python tools/prof_heat.py > gpurun_out/ncu_full.log 2>&1; echo "full rc=$?"; tail -2 gpurun_out/ncu_full.log
