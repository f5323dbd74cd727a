#!/bin/bash
# A/B of the tile-column sweep's consumer layout (TILES_SWEEP_CS: 1 consecutive rows, 2 + x by shuffle, 3 + 8 rows per thread)
O=gpurun_out/s2w
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || exit 1
for cs in 2 3; do TILES_SWEEP_CS=$cs timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "stream_through or wavefront or random" 2>&1 | tail -1 | tee -a $O/tests.txt; done
for rnd in 1 2 3; do
  for cs in 0 1 2 3; do
    TILES_SWEEP_CS=$cs timeout 120 python bench.py --no-extras --no-cpu-baseline --steps 20 > $O/cs${cs}_$rnd.json 2>/dev/null
    python -c "
import json; d=json.load(open('$O/cs${cs}_$rnd.json')); r=d['roofline']; print('cs=$cs', $rnd, round(d['value'],2), 'frac', round(r['frac'],3), 'launch_us', round(r['avg_launch_ms']*1e3,2))"
  done
done
