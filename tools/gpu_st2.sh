#!/bin/bash
mkdir -p gpurun_out/st
timeout 900 python -m pytest tests -m gpu -x -q -k stream_through > gpurun_out/st/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/st/pytest_gpu.log
for by in 4 2; do
TILES_SWEEP_BY=$by T=32 timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,sm__warps_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:slab_sweep -c 40 --csv --log-file gpurun_out/st/ncu_st_by$by.csv python tools/prof_st.py > gpurun_out/st/ncu_st.log 2>&1; echo "ncu rc=$?"
python tools/ncu_csv.py gpurun_out/st/ncu_st_by$by.csv 3
TILES_SWEEP_BY=$by timeout 900 python bench.py --config fig5 --sweep 10,32,48 --stream-through 1 > gpurun_out/st/fig5_by$by.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/st/fig5_by$by.json'));print('by=$by', {T:(round(r['tiled']['ms'],2),round(r['sync']['ms'],2)) for T,r in d['sweep'].items()})"
done
