python -c "import __graft_entry__ as g; g.build()" || exit 1
SCHED=wave T=64 TILES_WAVE_C=32 timeout 600 ncu --set full --clock-control none --import-source on -k regex:slab_sweep -s 300 -c 2 -o gpurun_out/sweep_wave_cfg1 python tools/prof_sweep.py > /dev/null 2>&1
ncu -i gpurun_out/sweep_wave_cfg1.ncu-rep --page raw --csv > gpurun_out/sweep_wave_cfg1.raw.csv 2>/dev/null
SCHED=wave T=64 TILES_WAVE_C=32 timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --cache-control none -k regex:slab_sweep -s 200 -c 200 --csv --log-file gpurun_out/sweep_wave_list.csv python tools/prof_sweep.py > /dev/null 2>&1
