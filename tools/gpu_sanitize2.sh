#!/bin/bash
mkdir -p gpurun_out/san
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python tools/sanitize.py 2>&1 | tail -1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize.py > gpurun_out/san/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|sanitize driver ok" gpurun_out/san/sanitize_$tool.log | head -3
done
