#!/bin/bash
mkdir -p gpurun_out/ca
timeout 900 python -m pytest tests -m gpu -x -q -k "stream_through" > gpurun_out/ca/pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/ca/pytest.log
for ca in 1 0; do
TILES_SWEEP_CA=$ca T=32 timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:slab_sweep -c 40 --csv --log-file gpurun_out/ca/ncu_$ca.csv python tools/prof_st.py > /dev/null 2>&1; echo "ncu rc=$?"
python tools/ncu_csv.py gpurun_out/ca/ncu_$ca.csv 2 | tail -3
TILES_SWEEP_CA=$ca timeout 900 python bench.py --config fig5 --sweep 10,32,48,64 --stream-through 1 > gpurun_out/ca/fig5_$ca.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/ca/fig5_$ca.json'));print('ca=$ca', {T:(round(r['tiled']['ms'],2),round(r['sync']['ms'],2)) for T,r in d['sweep'].items()})"
done
