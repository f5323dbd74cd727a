#!/bin/bash
# Copy-pattern probe + the C2 e2e bench legs on the same box.
O=gpurun_out/s2b
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || { tail -20 $O/build.txt; exit 1; }
timeout 600 python tools/pcie_pattern.py $O/pcie_pattern.json 2>&1 | tail -20
timeout 900 python bench.py --no-extras --no-cpu-baseline > $O/bench.json 2> $O/bench.err
python -c "
import json; d=json.load(open('$O/bench.json')); print('value', d['value'], 'xfer_only', d['overlap']['t_xfer_only_ms'], 'wall', d['overlap']['t_wall_ms'], d['roofline_link']['pcie_gbs'])"
