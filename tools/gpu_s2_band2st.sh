#!/bin/bash
# (experiment script: the knob it sets was measured and reverted; kept as the record of the A/B)
O=gpurun_out/s2l
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || { tail -20 $O/build.txt; exit 1; }
TILES_BAND2_ST=2 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -q -x -k "wavefront or split or band or random" 2>&1 | tail -2 | tee $O/tests.txt
for rnd in 1 2 3; do
  for st in 0 2; do
    echo "ST=$st $rnd $(TILES_BAND2_ST=$st timeout 600 python tools/wave_ab.py 32,48,64,100,200 5)" | tee -a $O/ab.txt
  done
done
