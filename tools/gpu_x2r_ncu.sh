#!/bin/bash
mkdir -p gpurun_out/x2r
TILES_X2_BAND=32 TILES_X2_STAGES=6 timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat7x2 -s 3 -c 1 -o gpurun_out/x2r/x2r_full -f python bench.py --no-extras --no-cpu-baseline --ghost 2 --two-step 1 --steps 1 --warmup 1 > gpurun_out/x2r/ncu.log 2>&1; echo "ncu rc=$?"; tail -2 gpurun_out/x2r/ncu.log
