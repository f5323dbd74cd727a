#!/bin/bash
# (experiment script: the knob it sets was measured and reverted; kept as the record of the A/B)
# heat2_band with the split (mbarrier arrive / wait) barrier: band-kernel parity, then A/B on the resident leg.
O=gpurun_out/s2q
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || { tail -20 $O/build.txt; exit 1; }
TILES_BAND2_SPLIT=1 timeout 240 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "band" 2>&1 | tail -1 | tee -a $O/tests.txt
grep -q passed $O/tests.txt || exit 3
TILES_BAND2_SPLIT=1 timeout 300 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -q -x -k "random or c2_value or split" 2>&1 | tail -1 | tee -a $O/tests.txt
for rnd in 1 2 3 4; do
  for sp in 0 1; do
    TILES_BAND2_SPLIT=$sp timeout 120 python bench.py --no-extras --no-cpu-baseline --steps 20 > $O/sp${sp}_$rnd.json 2>/dev/null
    python -c "
import json; d=json.load(open('$O/sp${sp}_$rnd.json')); r=d['resident']; print('split=$sp', $rnd, 'resident', round(r['value'],1), 'frac', round(r['roofline']['frac'],3), 'launch_ms', round(r['roofline']['avg_launch_ms'],4))"
  done
done
