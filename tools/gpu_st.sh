#!/bin/bash
# stream-through cost model check: T sweep with never / auto / forced
mkdir -p gpurun_out/st
timeout 900 python -m pytest tests -m gpu -x -q -k "stream_through" > gpurun_out/st/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/st/pytest_gpu.log
for st in -1 0 1; do
  timeout 900 python bench.py --config fig5 --sweep 1,10,16,32,48,64 --stream-through $st > gpurun_out/st/fig5_st$st.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/st/fig5_st$st.json'));print('st=$st', {T:(round(r['tiled']['ms'],2),round(r['sync']['ms'],2)) for T,r in d['sweep'].items()})"
done
