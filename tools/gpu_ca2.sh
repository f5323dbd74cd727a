#!/bin/bash
mkdir -p gpurun_out/ca
for sg in 4 5 6; do
TILES_SWEEP_STAGES=$sg T=32 timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:slab_sweep -c 40 --csv --log-file gpurun_out/ca/ncu_sg$sg.csv python tools/prof_st.py > /dev/null 2>&1
echo "sg=$sg"; python tools/ncu_csv.py gpurun_out/ca/ncu_sg$sg.csv 0 | tail -1
done
TILES_SWEEP_STAGES=6 timeout 600 python -m pytest tests -m gpu -x -q -k "stream_through" 2>&1 | tail -1
