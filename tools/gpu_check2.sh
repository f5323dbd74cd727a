#!/bin/bash
# re-entry check: smoke, GPU tests, headline bench, reference arm
mkdir -p gpurun_out/chk
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/chk/smi.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/chk/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 gpurun_out/chk/smoke.log
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/chk/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/chk/pytest_gpu.log
timeout 900 python bench.py > gpurun_out/chk/bench.json 2> gpurun_out/chk/bench.err; echo "bench rc=$?"; python -c "import json;d=json.load(open('gpurun_out/chk/bench.json'));print(d['value'], d['e2e']['value'], d['roofline'], d['clocks'], d['overlap'])"
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/chk/ref.json 2> gpurun_out/chk/ref.err; echo "ref rc=$?"; head -c 800 gpurun_out/chk/ref.json
