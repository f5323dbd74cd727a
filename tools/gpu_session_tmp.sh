python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "band2 or wavefront or stream_through" 2>&1 | tail -4
for two in 1 0 1 0; do
v=$(TILES_ST_TWO=$two timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 20 --warmup 3 2>/dev/null | tail -1 | python -c "import json,sys;d=json.load(sys.stdin);r=d['roofline'];print(round(d['ms_per_step'],3), round(d['value'],2), r['kernel'], round(r['frac'],3), round(r['avg_launch_ms']*1e3,1), r['launches_per_step'])")
echo "two=$two : $v"
done
