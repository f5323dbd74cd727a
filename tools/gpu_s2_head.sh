#!/bin/bash
O=gpurun_out/s2n
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || { tail -20 $O/build.txt; exit 1; }
TILES_ST_HEAD=4 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "stream_through" 2>&1 | tail -1 | tee $O/tests.txt
for rnd in 1 2 3 4; do
  for h in 2 3 4 6; do
    TILES_ST_HEAD=$h timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 20 > $O/h${h}_$rnd.json 2>/dev/null
    python -c "
import json; d=json.load(open('$O/h${h}_$rnd.json')); print('head=$h', $rnd, round(d['value'],2), round(d['ms_per_step'],3))"
  done
done
