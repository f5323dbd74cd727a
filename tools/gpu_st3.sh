#!/bin/bash
mkdir -p gpurun_out/st
timeout 900 python -m pytest tests -m gpu -x -q -k "stream_through" > gpurun_out/st/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/st/pytest_gpu.log
timeout 900 python bench.py --config fig5 --sweep 1,10,16,32 > gpurun_out/st/fig5_v.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/st/fig5_v.json'));print({T:(round(r['tiled']['ms'],2),round(r['sync']['ms'],2)) for T,r in d['sweep'].items()})"
