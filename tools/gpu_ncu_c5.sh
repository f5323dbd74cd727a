#!/bin/bash
# ncu --set full of the C5-shaped heat7_fixed<256,16> launch (4096^2 x 128 slab, 256^2 x 64 tiles)
mkdir -p gpurun_out/c5ncu
python __graft_entry__.py > /dev/null 2>&1
for rr in 1 0; do
TILES_HEAT_RR=$rr DIMS=4096,4096,128 TD=256,256,64 STEPS=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:heat7_fixed -c 4 \
  -o gpurun_out/c5ncu/c5_rr$rr -f python tools/prof_heat.py > gpurun_out/c5ncu/log_rr$rr.txt 2>&1; echo "rr=$rr rc=$?"; tail -2 gpurun_out/c5ncu/log_rr$rr.txt
done
