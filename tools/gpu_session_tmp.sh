python -c "import __graft_entry__ as g; g.build()" || exit 1
for rep in 1 2 3 4; do
for two in 1 0; do
v=$(TILES_ST_TWO=$two timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 30 --warmup 3 2>/dev/null | tail -1 | python -c "import json,sys;d=json.load(sys.stdin);r=d['roofline'];print(round(d['ms_per_step'],3), r['kernel'], round(r['frac'],3), d['clocks']['sm_mhz'])")
echo "two=$two : $v"
done; done
