python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k wavefront 2>&1 | tail -3
SCHED=wave T=64 timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --cache-control none -k regex:slab_sweep2 -s 100 -c 20 --csv --log-file gpurun_out/sweep2d_list.csv python tools/prof_sweep.py > /dev/null 2>&1
python tools/ncu_csv.py gpurun_out/sweep2d_list.csv 2 | tail -3
for f in 1 0; do TILES_WAVE_FUSE=$f timeout 900 python bench.py --config fig5 --steps 3 --warmup 3 2>&1 | tail -1 > gpurun_out/fig5_fuse$f.json; echo fuse=$f; python -c "import json;d=json.load(open('gpurun_out/fig5_fuse$f.json'));print({k:v for k,v in d.items() if k in ('ms_by_T','by_T','value')})"; done
