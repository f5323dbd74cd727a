#!/bin/bash
O=gpurun_out/s2f
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || { tail -20 $O/build.txt; exit 1; }
for i in 1 2; do timeout 600 python -m pytest tests/test_errors.py -m gpu -q -rf 2>&1 | tail -40 > $O/errors_$i.txt; tail -12 $O/errors_$i.txt; done
timeout 600 python -m pytest tests/test_errors.py -m gpu -q -x -k "h2d and stream and tile_run" 2>&1 | tail -60 > $O/errors_detail.txt
bash tools/gpu_s2_l2pol.sh
