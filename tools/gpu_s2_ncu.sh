#!/bin/bash
# --set full capture of one stream-through sweep (slab_sweep_tile, evict-last stores) mid-run.
O=gpurun_out/s2u
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || exit 1
SCHED=stream T=10 timeout 900 ncu --set full --clock-control none --import-source on -k regex:slab_sweep_tile -s 200 -c 1 -o $O/st_sweep_full python tools/prof_sweep.py > $O/ncu.log 2>&1
ncu -i $O/st_sweep_full.ncu-rep --page raw --csv > $O/st_sweep_full.raw.csv 2>/dev/null
ncu -i $O/st_sweep_full.ncu-rep --page details --csv > $O/st_sweep_full.details.csv 2>/dev/null
rm -f $O/st_sweep_full.ncu-rep
ls -la $O
