python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "timing or wavefront or stream" 2>&1 | tail -3
timeout 900 python bench.py 2>&1 | tail -1 > gpurun_out/bench_iv.json
python -c "
import json;d=json.load(open('gpurun_out/bench_iv.json'));r=d['roofline'];print(d['value'], {k:r.get(k) for k in ('frac','frac_in_pipeline','avg_launch_ms','launches_per_step','kernel')}, d['resident']['roofline']['frac'])"
