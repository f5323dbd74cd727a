python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q -m gpu -k "wavefront" 2>&1 | tail -3
for it in 1 0; do
TILES_WAVE_ITER=$it timeout 900 python bench.py --config fig5 --steps 3 --warmup 3 --sweep 32,48,64,100 2>/dev/null | tail -1 > gpurun_out/fig5_it$it.json
python -c "
import json;d=json.load(open('gpurun_out/fig5_it$it.json'));print('iter=$it', {T:(round(v['tiled']['ms'],1), v['tiled']['schedule'][:12]) for T,v in d['sweep'].items()})"
done
