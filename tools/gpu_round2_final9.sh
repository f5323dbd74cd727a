#!/bin/bash
# Round-2 final evidence (second session: consecutive-row sweep consumers): GPU tests, smoke,
# sanitizers, the default bench line, the ncu launch list of the same
# command, per-kernel DRAM traffic, --set full captures of the band kernels,
# the Fig. 5 sweep and CUPTI timelines.
O=gpurun_out/r2f9
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -3 > $O/gputests.txt; cat $O/gputests.txt
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1; tail -1 $O/smoke.txt
# compute-sanitizer is closed on the pool (late round 2): the last sanitizer logs are profiles/r02/final4
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
timeout 900 python bench.py --impl reference > $O/bench_reference.json 2> $O/bench_reference.err
TILES_BENCH_ONE_GPU=1 timeout 900 python bench.py --gpus 2 --steps 5 --warmup 3 --no-extras --no-cpu-baseline > $O/bench_n2_one_gpu.json 2> $O/bench_n2.err
TILES_ST_R=0.021 timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $O/launches_bench.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu-baseline > /dev/null 2>&1
python tools/ncu_csv.py $O/launches_bench.csv 0 | tail -8 > $O/launches_summary.txt
SCHED=stream T=10 timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --cache-control none -k regex:slab_sweep --csv --log-file $O/st_sweeps.csv python tools/prof_sweep.py > /dev/null 2>&1
python tools/sweep_traffic.py $O/st_sweeps.csv stream 10 $O/slab_sweep_tile_ncu_traffic.json
SCHED=wave T=64 timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --cache-control none -k regex:heat2_band_slab --csv --log-file $O/wave_band.csv python tools/prof_sweep.py > /dev/null 2>&1
python tools/sweep_traffic.py $O/wave_band.csv wave 64 $O/heat2_band_slab_ncu_traffic.json heat2_band_slab
cat > /tmp/b2one.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, synth
from paper_conf_icpp_bastemuzas17_b200 import tiles as T
n = 512
u = np.empty((n, n, n)); synth.fill_uniform_native(u.ctypes.data, n, n, n, 0, n, 0, n, 0, n, 42)
d = T.Domain((n, n, n), (64, 64, 64), sweep_link_ratio=0.021)
d.load(u); d.run(T.heat7(), 1, 4); d.sync()
d.run(T.heat7(), 10, 4); d.sync()
PY
timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat2_band -s 2 -c 1 -o $O/heat2_band_full python /tmp/b2one.py > /dev/null 2>&1
ncu -i $O/heat2_band_full.ncu-rep --page raw --csv > $O/heat2_band_full.raw.csv 2>/dev/null
SCHED=wave T=64 timeout 900 ncu --set full --clock-control none --import-source on -k regex:heat2_band_slab -s 200 -c 1 -o $O/heat2_band_slab_full python tools/prof_sweep.py > /dev/null 2>&1
ncu -i $O/heat2_band_slab_full.ncu-rep --page raw --csv > $O/heat2_band_slab_full.raw.csv 2>/dev/null
rm -f $O/*.ncu-rep
timeout 1200 python bench.py --config fig5 --steps 3 --warmup 3 --sweep 1,10,32,48,64,100,200,1000 > $O/fig5.json 2>/dev/null
for c in c2 wave; do T=64 python tools/timeline.py $c $O/timeline_$c > /dev/null 2>&1; rm -f $O/timeline_$c.trace.json; done
ls $O
