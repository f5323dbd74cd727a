#!/bin/bash
# full check: smoke, GPU tests, sanitizers, headline bench
mkdir -p gpurun_out/full
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/full/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/full/smoke.log
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/full/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/full/pytest_gpu.log
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize.py > gpurun_out/full/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY" gpurun_out/full/sanitize_$tool.log | tail -1
done
timeout 900 python bench.py > gpurun_out/full/bench.json 2> gpurun_out/full/bench.err; echo "bench rc=$?"; python -c "import json;d=json.load(open('gpurun_out/full/bench.json'));print(d['value'], d['e2e']['value'], d['roofline']['frac'], d['clocks'])"
timeout 900 python bench.py --config fig8 > gpurun_out/full/fig8.json 2> gpurun_out/full/fig8.err; echo "fig8 rc=$?"; head -c 1500 gpurun_out/full/fig8.json
