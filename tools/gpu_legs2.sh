#!/bin/bash
mkdir -p gpurun_out
python __graft_entry__.py > /dev/null 2>&1
timeout 900 python bench.py --config c4 --steps 2 --warmup 1 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err; echo "c4 rc=$?"; cat gpurun_out/bench_c4.json; tail -3 gpurun_out/bench_c4.err
timeout 600 ncu --metrics gpu__time_duration.sum,smsp__inst_executed_pipe_fp64.sum,sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active,smsp__sass_thread_inst_executed_op_dfma_pred_on.sum,smsp__sass_thread_inst_executed_op_dadd_pred_on.sum,smsp__sass_thread_inst_executed_op_dmul_pred_on.sum,smsp__inst_executed.sum,sm__warps_active.avg.pct_of_peak_sustained_active \
  -k regex:sincos -s 2 -c 1 --csv --log-file gpurun_out/ncu_sincos_c4.csv python bench.py --config c4 --steps 1 --warmup 0 --sweep 4 > /dev/null 2>&1; echo "ncu sincos rc=$?"
for ns in 2 8; do
timeout 900 python bench.py --config c3 --steps 1 --warmup 1 --nstreams $ns > gpurun_out/bench_c3_s$ns.json 2> gpurun_out/bench_c3.err; echo "c3 ns=$ns rc=$?"; python -c "import json; j=json.load(open('gpurun_out/bench_c3_s$ns.json')); print(j['value'], j['roofline']['frac'], j['overlap'])"
done
