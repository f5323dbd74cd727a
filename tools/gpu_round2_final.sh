#!/bin/bash
# Round-2 evidence: GPU tests, sanitizers, the default bench line, the ncu
# launch list of the same command, and the sweep kernel's DRAM traffic.
mkdir -p gpurun_out/r2
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1800 python -m pytest tests -m gpu -q 2>&1 | tail -3 > gpurun_out/r2/gputests.txt
cat gpurun_out/r2/gputests.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2/smoke.txt 2>&1; tail -1 gpurun_out/r2/smoke.txt
bash tools/gpu_sanitize.sh > gpurun_out/r2/sanitize_summary.txt 2>&1; cp gpurun_out/sanitize_*.log gpurun_out/r2/ 2>/dev/null
cat gpurun_out/r2/sanitize_summary.txt
timeout 900 python bench.py > gpurun_out/r2/bench.json 2> gpurun_out/r2/bench.err
# launch list of the bench command (cost-model ratio fixed: under ncu the calibration would time replayed kernels)
TILES_ST_R=0.021 timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2/launches_bench.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu-baseline > /dev/null 2>&1
python tools/ncu_csv.py gpurun_out/r2/launches_bench.csv 0 | tail -6 > gpurun_out/r2/launches_summary.txt
SCHED=stream T=10 timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --cache-control none -k regex:slab_sweep --csv --log-file gpurun_out/r2/st_sweeps.csv python tools/prof_sweep.py > /dev/null 2>&1
python tools/sweep_traffic.py gpurun_out/r2/st_sweeps.csv stream 10 gpurun_out/r2/slab_sweep_tile_ncu_traffic.json
SCHED=wave T=64 timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --cache-control none -k regex:slab_sweep --csv --log-file gpurun_out/r2/wave_sweeps.csv python tools/prof_sweep.py > /dev/null 2>&1
python tools/sweep_traffic.py gpurun_out/r2/wave_sweeps.csv wave 64 gpurun_out/r2/slab_sweep_tile_wave_traffic.json
SCHED=stream T=10 timeout 900 ncu --set full --clock-control none --import-source on -k regex:slab_sweep -s 60 -c 1 -o gpurun_out/r2/st_sweep_full python tools/prof_sweep.py > /dev/null 2>&1
ncu -i gpurun_out/r2/st_sweep_full.ncu-rep --page raw --csv > gpurun_out/r2/st_sweep_full.raw.csv 2>/dev/null
ls gpurun_out/r2
