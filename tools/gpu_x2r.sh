#!/bin/bash
mkdir -p gpurun_out/x2r
timeout 900 python -m pytest tests -m gpu -x -q -k "two_step or x2 or ghost" > gpurun_out/x2r/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/x2r/pytest.log
for v in 1 0; do
  TILES_X2_ROWS=$v timeout 300 python bench.py --no-extras --no-cpu-baseline --ghost 2 --two-step 1 > gpurun_out/x2r/x2_$v.json 2>gpurun_out/x2r/x2_$v.err; python -c "import json;d=json.load(open('gpurun_out/x2r/x2_$v.json'));print('rows=$v value',d['value'], d['roofline']['avg_launch_ms'], d['roofline'].get('kernel'))"
done
timeout 300 python bench.py --no-extras --no-cpu-baseline > gpurun_out/x2r/base.json 2>/dev/null; python -c "import json;d=json.load(open('gpurun_out/x2r/base.json'));print('single value',d['value'])"
GHOST=2 STEPS=4 timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat7x2r -s 2 -c 1 -o gpurun_out/x2r/x2r_full -f python tools/prof_heat.py > gpurun_out/x2r/ncu.log 2>&1; echo "ncu rc=$?"; tail -2 gpurun_out/x2r/ncu.log
