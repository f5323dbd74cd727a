#!/bin/bash
# stream-through with the z-march sweep: tests, T sweep (never / auto / forced)
mkdir -p gpurun_out/st
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/st/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/st/pytest_gpu.log
for st in 0 1; do
  timeout 900 python bench.py --config fig5 --sweep 1,10,16,32,48,64 --stream-through $st > gpurun_out/st/fig5_st$st.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/st/fig5_st$st.json'));print('st=$st', {T:(round(r['tiled']['ms'],2),round(r['sync']['ms'],2)) for T,r in d['sweep'].items()})"
done
timeout 300 python tools/sanitize.py > /dev/null 2>&1 && timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python tools/sanitize.py > gpurun_out/st/memcheck.log 2>&1; echo "memcheck rc=$?"
timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python tools/sanitize.py > gpurun_out/st/racecheck.log 2>&1; echo "racecheck rc=$?"
