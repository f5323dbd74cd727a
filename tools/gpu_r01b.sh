#!/bin/bash
# sanitizers (incl. stream-through), C2 e2e timeline, C5 bench
mkdir -p gpurun_out/timeline
bash tools/gpu_sanitize.sh
timeout 300 python tools/timeline.py c2 gpurun_out/timeline/c2 > gpurun_out/timeline/c2.log 2>&1; echo "tl rc=$?"; tail -2 gpurun_out/timeline/c2.log
rm -f gpurun_out/timeline/c2.trace.json.gz; gzip -f gpurun_out/timeline/c2.trace.json
timeout 600 python bench.py --config c5 --no-cpu-baseline > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err; echo "c5 rc=$?"; cat gpurun_out/bench_c5.json; tail -3 gpurun_out/bench_c5.err
