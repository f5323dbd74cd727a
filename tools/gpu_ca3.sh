#!/bin/bash
mkdir -p gpurun_out/full
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/full/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/full/pytest_gpu.log
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize.py > gpurun_out/full/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY" gpurun_out/full/sanitize_$tool.log | tail -1
done
timeout 1500 python bench.py --config fig5 --sweep 1,10,16,32,48,64,100,1000 > gpurun_out/full/fig5.json 2>/dev/null; echo "fig5 rc=$?"
python -c "import json;d=json.load(open('gpurun_out/full/fig5.json'));print({T:(round(r['tiled']['ms'],2),round(r['sync']['ms'],2),round(r['sync_pageable']['ms'],1)) for T,r in d['sweep'].items()})"
