#!/bin/bash
# racecheck + C2 value with per-warp (0) vs per-thread (1) stage hand-off arrives
mkdir -p gpurun_out/arrive
for v in 1 0; do
  TILES_NVCC_DEFS="-DTILES_ARRIVE_PER_THREAD=$v" python paper_conf_icpp_bastemuzas17_b200/build.py --force > /dev/null 2>&1
  timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python tools/sanitize.py > gpurun_out/arrive/race_$v.log 2>&1
  echo "v=$v racecheck rc=$?"; grep -E "SUMMARY" gpurun_out/arrive/race_$v.log; grep -o "heat7[a-z0-9_]*<[^>]*>" gpurun_out/arrive/race_$v.log | sort | uniq -c
  for i in 1 2 3; do timeout 300 python bench.py --no-extras --no-cpu-baseline > gpurun_out/arrive/bench_$v.$i.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/arrive/bench_$v.$i.json'));print('v=$v value',d['value'],d['roofline']['frac'],d['clocks']['sm_mhz'])"; done
  for i in 1 2; do timeout 300 python bench.py --no-extras --no-cpu-baseline --ghost 2 --two-step 1 > gpurun_out/arrive/x2_$v.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/arrive/x2_$v.json'));print('v=$v x2 value',d['value'])"; done
done
python paper_conf_icpp_bastemuzas17_b200/build.py --force > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/arrive/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/arrive/pytest_gpu.log
