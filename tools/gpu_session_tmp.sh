python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -x -q -k "wavefront or stream_through" 2>&1 | tail -2
timeout 600 python bench.py --config fig5 --steps 1 --sweep 10,32,48,64,100 > gpurun_out/fig5_boot.json 2>/dev/null
python -c "import json;j=json.loads(open('gpurun_out/fig5_boot.json').read().strip().splitlines()[-1]);print({T:(round(r['tiled']['ms'],1), round(r['tiled_frac_of_bound'],3), r['tiled']['schedule'][:5], round(r['speedup_tiled_vs_sync'],2)) for T,r in j['sweep'].items()})"
for c in 16 64; do TILES_WAVE_C=$c timeout 600 python bench.py --config fig5 --steps 1 --sweep 48,64,100 --wavefront 1 > gpurun_out/fig5_boot_c$c.json 2>/dev/null
python -c "import json;j=json.loads(open('gpurun_out/fig5_boot_c$c.json').read().strip().splitlines()[-1]);print($c, {T:(round(r['tiled']['ms'],1), round(r['tiled_frac_of_bound'],3)) for T,r in j['sweep'].items()})"; done
