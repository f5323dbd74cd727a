#!/bin/bash
# Extra bench legs: FP64 peak, C4 sincos sweep, C3 out-of-core; ncu of sincos.
mkdir -p gpurun_out
python __graft_entry__.py > /dev/null 2>&1
nvcc -gencode arch=compute_100a,code=sm_100a -O3 tools/dfma_peak.cu -o /tmp/dfma_peak && /tmp/dfma_peak | tee gpurun_out/dfma_peak.json
timeout 900 python bench.py --config c4 --steps 2 --warmup 1 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err; echo "c4 rc=$?"; cat gpurun_out/bench_c4.json; tail -3 gpurun_out/bench_c4.err
timeout 600 ncu --metrics gpu__time_duration.sum,smsp__inst_executed_pipe_fp64.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,smsp__sass_thread_inst_executed_op_dfma_pred_on.sum,smsp__sass_thread_inst_executed_op_dadd_pred_on.sum,smsp__sass_thread_inst_executed_op_dmul_pred_on.sum,smsp__inst_executed.sum \
  -k regex:sincos -c 1 --csv --log-file gpurun_out/ncu_sincos.csv python bench.py --config c4 --n 256 --steps 1 --warmup 0 --sweep 1 > /dev/null 2>&1; echo "ncu sincos rc=$?"
timeout 1500 python bench.py --config c3 --steps 2 --warmup 1 > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; echo "c3 rc=$?"; cat gpurun_out/bench_c3.json; tail -3 gpurun_out/bench_c3.err
