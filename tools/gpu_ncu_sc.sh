#!/bin/bash
mkdir -p gpurun_out
timeout 600 ncu --metrics gpu__time_duration.sum,smsp__inst_executed_pipe_fp64.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,smsp__sass_thread_inst_executed_op_dfma_pred_on.sum,smsp__sass_thread_inst_executed_op_dadd_pred_on.sum,smsp__sass_thread_inst_executed_op_dmul_pred_on.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__thread_inst_executed_pipe_fp64.sum \
  -k regex:sincos -c 1 --csv --log-file gpurun_out/ncu_sincos_v2.csv python bench.py --config c4 --n 256 --steps 1 --warmup 0 --sweep 1 > gpurun_out/ncu_sc.log 2>&1; echo "ncu sincos rc=$?"
python tools/ncu_csv.py gpurun_out/ncu_sincos_v2.csv 3
