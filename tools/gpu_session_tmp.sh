python -c "import __graft_entry__ as g; g.build()" || exit 1
for mu in 16 32 64 16 32; do TILES_ST_MINUNIT=$mu timeout 600 python bench.py --no-cpu-baseline --no-extras --steps 20 > gpurun_out/bench_mu$mu.json 2>/dev/null
python -c "import json;j=json.loads(open('gpurun_out/bench_mu$mu.json').read().strip().splitlines()[-1]);print($mu, round(j['value'],2), round(j['ms_per_step'],2), 'sweep', round(j['roofline']['achieved']), round(j['roofline']['frac'],3), round(j['roofline']['avg_launch_ms']*1e3,1), j['roofline']['launches_per_step'])"; done
