python -c "import __graft_entry__ as g; g.build()" || exit 1
bash tools/gpu_sanitize.sh
mkdir -p gpurun_out/san2 && cp gpurun_out/sanitize_*.log gpurun_out/san2/ 2>/dev/null
# launch list of the bench's default command, and the e2e step's sweep traffic (warm L2)
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 2000 --csv --log-file gpurun_out/launches_r2.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu-baseline > gpurun_out/bench_under_ncu.log 2>&1
SCHED=stream T=10 timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --cache-control none -k regex:slab_sweep --csv --log-file gpurun_out/st_sweeps_warm.csv python tools/prof_sweep.py > /dev/null 2>&1
SCHED=stream T=10 timeout 600 ncu --set full --clock-control none --import-source on -k regex:slab_sweep -s 150 -c 1 -o gpurun_out/st_sweep_full python tools/prof_sweep.py > /dev/null 2>&1
ncu -i gpurun_out/st_sweep_full.ncu-rep --page raw --csv > gpurun_out/st_sweep_full.raw.csv 2>/dev/null
timeout 1200 python bench.py --config fig8 --T 1000 --sweep 32,256 > gpurun_out/fig8_T1000.json 2>gpurun_out/fig8.err
tail -2 gpurun_out/fig8.err
