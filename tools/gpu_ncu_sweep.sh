#!/bin/bash
# ncu --set full of one mid-run sweep launch, TMA and cp.async variants, stream-through and wavefront
python -c "import __graft_entry__ as g; g.build()" || exit 1
NCU=ncu
for v in 1 0; do
  for sc in stream wave; do
    TILES_SWEEP_TMA=$v SCHED=$sc T=10 TILES_WAVE_C=32 timeout 600 $NCU --set full --clock-control none --import-source on \
      -k regex:slab_sweep -s 40 -c 1 -o gpurun_out/sweep_${sc}_tma$v python tools/prof_sweep.py > gpurun_out/ncu_${sc}_tma$v.log 2>&1
    ncu -i gpurun_out/sweep_${sc}_tma$v.ncu-rep --page raw --csv > gpurun_out/sweep_${sc}_tma$v.raw.csv 2>/dev/null
  done
done
ls -la gpurun_out/*.ncu-rep
