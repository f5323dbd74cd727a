python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "wavefront or stream_through" 2>&1 | tail -1
timeout 900 python bench.py --config fig5 --steps 1 > gpurun_out/fig5_final2.json 2>/dev/null
python -c "import json;j=json.loads(open('gpurun_out/fig5_final2.json').read().strip().splitlines()[-1]);print({T:(round(r['tiled']['ms'],1), round(r['tiled_frac_of_bound'],3), round(r['tiled_frac_of_causal_bound'],3), round(r['speedup_tiled_vs_sync'],2)) for T,r in j['sweep'].items()})"
mkdir -p gpurun_out/tl
timeout 600 python tools/timeline.py wave gpurun_out/tl/timeline_wave64 > /dev/null 2>&1; cat gpurun_out/tl/timeline_wave64.summary.json
timeout 600 python tools/timeline.py c2 gpurun_out/tl/timeline_c2 > /dev/null 2>&1; cat gpurun_out/tl/timeline_c2.summary.json
rm -f gpurun_out/tl/*.trace.json
