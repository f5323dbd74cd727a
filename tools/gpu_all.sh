#!/bin/bash
# Full GPU pass: tests, headline bench, Fig.5 sweep, C3 out-of-core.
mkdir -p gpurun_out
python __graft_entry__.py > /dev/null 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
python -c "import json; j=json.load(open('gpurun_out/bench.json')); print('value', j['value'], 'frac', j['roofline']['frac'], 'e2e', j['e2e']['value'], 'sync', j.get('sync_baseline_e2e',{}).get('value'), 'e2e_roof', j.get('e2e_roofline',{}).get('frac'), 'hidden', j.get('overlap',{}).get('hidden_frac'))"
if [ "${FIG5:-1}" = "1" ]; then
timeout 900 python bench.py --config fig5 > gpurun_out/bench_fig5.json 2>gpurun_out/fig5.err; echo "fig5 rc=$?"
python -c "
import json; j=json.load(open('gpurun_out/bench_fig5.json'))
for k,v in j['sweep'].items(): print('T',k, round(v['tiled']['ms'],2), round(v['sync']['ms'],2), round(v['speedup_tiled_vs_sync'],3), round(v['tiled_frac_of_bound'],3))"
fi
if [ "${C3:-0}" = "1" ]; then
timeout 1200 python bench.py --config c3 --steps 2 --warmup 1 --nstreams ${C3NS:-4} > gpurun_out/bench_c3.json 2> gpurun_out/bench_c3.err; echo "c3 rc=$?"
python -c "import json; j=json.load(open('gpurun_out/bench_c3.json')); print(j['value'], j['roofline']['frac'], j['overlap'], j['residency'])"
fi
