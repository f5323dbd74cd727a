python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -x -q -k "wavefront" 2>&1 | tail -2
for bg in 4 1 2 8; do TILES_WAVE_BIG=$bg timeout 600 python bench.py --config fig5 --steps 1 --sweep 32,48,64,100 --wavefront 1 > gpurun_out/fig5_big$bg.json 2>/dev/null
python -c "import json;j=json.loads(open('gpurun_out/fig5_big$bg.json').read().strip().splitlines()[-1]);print($bg, {T:(round(r['tiled']['ms'],1), round(r['tiled_frac_of_bound'],3)) for T,r in j['sweep'].items()})"; done
