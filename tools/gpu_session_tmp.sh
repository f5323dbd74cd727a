python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "band2 or wavefront" 2>&1 | tail -4
for wf in 1 2; do
timeout 900 python bench.py --config fig5 --steps 3 --warmup 3 --wavefront $wf 2>/dev/null | tail -1 > gpurun_out/fig5_b2s_wf$wf.json
python -c "
import json;d=json.load(open('gpurun_out/fig5_b2s_wf$wf.json'));print('wf=$wf', {T:(round(v['tiled']['ms'],1), v['tiled']['schedule'][:12]) for T,v in d['sweep'].items()})"
done
