#!/bin/bash
mkdir -p gpurun_out
# run the new case alone first: bit-exact vs the oracle
python __graft_entry__.py > /dev/null 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize.py > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|sanitize driver ok|Error" gpurun_out/sanitize_$tool.log | head -3
done
