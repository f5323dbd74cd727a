#!/bin/bash
# sanitizers on every schedule (incl. persistent + direct), then the duplex PCIe probe
mkdir -p gpurun_out/san
python __graft_entry__.py > /dev/null 2>&1
python tools/pcie_dual.py gpurun_out/san/pcie_dual.json 2>&1 | grep -v Warn | tail -18
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 python tools/sanitize.py > gpurun_out/san/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|sanitize driver ok" gpurun_out/san/sanitize_$tool.log | head -3
done
