python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
for rep in 1 2; do
for gm in 0 1; do
v=$(TILES_SWEEP_GRID=$gm timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 20 --warmup 3 2>/dev/null | tail -1 | python -c "import json,sys;d=json.load(sys.stdin);r=d['roofline'];print(round(d['ms_per_step'],3), r['kernel'], round(r['frac'],3), round(r['avg_launch_ms']*1e3,1))")
echo "grid=$gm : $v"
done; done
