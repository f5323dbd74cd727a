#!/bin/bash
# (experiment script: TILES_HEAT_CS was measured and reverted; kept as the record of the A/B)
# heat7_fixed with consecutive consumer rows (TILES_HEAT_CS=1): parity, then A/B on C2 single-step
# resident (--two-step -1) and the C5 per-GPU slab.
O=gpurun_out/s2y
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || exit 1
TILES_HEAT_CS=1 timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_multirank.py -m gpu -q -x 2>&1 | tail -1 | tee $O/tests.txt
grep -q " passed" $O/tests.txt || exit 3
for rnd in 1 2 3; do
  for cs in 0 1; do
    TILES_HEAT_CS=$cs timeout 120 python bench.py --no-extras --no-cpu-baseline --steps 20 --two-step -1 > $O/c2_cs${cs}_$rnd.json 2>/dev/null
    python -c "
import json; d=json.load(open('$O/c2_cs${cs}_$rnd.json')); r=d['resident']; print('c2 cs=$cs', $rnd, 'resident', round(r['value'],1), 'frac', round(r['roofline']['frac'],3), r['roofline'].get('kernel'))"
  done
done
for rnd in 1 2; do
  for cs in 0 1; do
    TILES_HEAT_CS=$cs timeout 300 python bench.py --config c5 --steps 2 --warmup 1 > $O/c5_cs${cs}_$rnd.json 2>/dev/null
    python -c "
import json; d=json.load(open('$O/c5_cs${cs}_$rnd.json')); print('c5 cs=$cs', $rnd, round(d['value'],1), 'frac', round(d['roofline']['frac'],3))"
  done
done
