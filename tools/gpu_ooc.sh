#!/bin/bash
mkdir -p gpurun_out/ooc
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/ooc/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/ooc/pytest_gpu.log
timeout 900 python bench.py --config c3 --steps 5 --warmup 3 > gpurun_out/ooc/c3.json 2> gpurun_out/ooc/c3.err; echo "c3 rc=$?"; cat gpurun_out/ooc/c3.json | head -c 3000; echo; tail -3 gpurun_out/ooc/c3.err
timeout 900 python bench.py --config c3 --steps 1 --warmup 1 --stream-through -1 > gpurun_out/ooc/c3_perstep.json 2> gpurun_out/ooc/c3_perstep.err; echo "c3 perstep rc=$?"; python -c "import json;d=json.load(open('gpurun_out/ooc/c3_perstep.json'));print(d['value'], d['ms_per_step'], d['roofline']['frac'])"
