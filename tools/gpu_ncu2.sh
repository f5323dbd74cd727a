#!/bin/bash
bash tools/gpu_ncu.sh
T=10 timeout 900 ncu --set full --clock-control none --import-source on -k regex:slab_sweep -s 3 -c 1 \
  -o gpurun_out/slab_sweep_full -f python tools/prof_st.py > gpurun_out/ncu_full_st.log 2>&1; echo "full st rc=$?"; tail -2 gpurun_out/ncu_full_st.log
