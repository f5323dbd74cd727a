#!/bin/bash
mkdir -p gpurun_out/zc
python __graft_entry__.py > /dev/null 2>&1
TILES_HEAT_ZCHUNK=8 timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x -k "resident or c2 or banded or shapes or runs_continue" 2>&1 | tail -1
TILES_HEAT_ZCHUNK=16 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "resident or banded or shapes" 2>&1 | tail -1
for zc in 0 8 16 32 64 0 8 16; do
  TILES_HEAT_ZCHUNK=$zc timeout 300 python bench.py --no-cpu-baseline --no-extras --steps 20 > gpurun_out/zc/z$zc.json 2>/dev/null
  python -c "import json;j=json.load(open('gpurun_out/zc/z$zc.json'));print('zchunk',$zc,'value',round(j['value'],1),'frac',round(j['roofline']['frac'],4))"
done
