python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "split or band2 or wavefront_bit" 2>&1 | tail -2
for sp in 1 0; do
TILES_WAVE_SPLIT=$sp timeout 1200 python bench.py --config fig5 --steps 3 --warmup 3 --sweep 100,150,200,300,1000 2>/dev/null | tail -1 > gpurun_out/fig5_split$sp.json
python -c "
import json;d=json.load(open('gpurun_out/fig5_split$sp.json'));print('split=$sp', {T:(round(v['tiled']['ms'],1), v['tiled']['schedule'][:14]) for T,v in d['sweep'].items()})"
done
