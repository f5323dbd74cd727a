python -c "import __graft_entry__ as g; g.build()" || exit 1
for c in 32 64 128 16; do
TILES_WAVE_C=$c timeout 900 python bench.py --config fig5 --steps 3 --warmup 3 --sweep 32,64,100,200 2>/dev/null | tail -1 > gpurun_out/fig5_c$c.json
python -c "
import json;d=json.load(open('gpurun_out/fig5_c$c.json'));print('c=$c', {T:(round(v['tiled']['ms'],1), v['tiled']['schedule'][:12]) for T,v in d['sweep'].items()})"
done
