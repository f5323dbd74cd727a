python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_host_regions.py tests/test_errors.py -m gpu -x -q 2>&1 | tail -3
for pdl in 1 0 1; do
  TILES_SWEEP_PDL=$pdl timeout 600 python bench.py --no-cpu-baseline --no-extras --steps 10 > gpurun_out/bench_pdl$pdl.json 2>/dev/null
  python -c "import json;j=json.loads(open('gpurun_out/bench_pdl$pdl.json').read().strip().splitlines()[-1]);print('pdl',$pdl, round(j['value'],2), round(j['roofline']['achieved']), round(j['roofline']['frac'],3), round(j['roofline']['avg_launch_ms']*1e3,1))"
  TILES_SWEEP_PDL=$pdl timeout 600 python bench.py --config fig5 --steps 1 --sweep 32,48,64,100 > gpurun_out/fig5_pdl$pdl.json 2>/dev/null
  python -c "import json;j=json.loads(open('gpurun_out/fig5_pdl$pdl.json').read().strip().splitlines()[-1]);print({T:(round(r['tiled']['ms'],1), round(r['tiled_frac_of_bound'],3), r['tiled']['schedule'][:5]) for T,r in j['sweep'].items()})"
done
