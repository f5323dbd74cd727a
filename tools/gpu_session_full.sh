python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.txt 2>&1; tail -2 gpurun_out/smoke.txt
timeout 1800 python -m pytest tests -x -q -m gpu 2>&1 | tail -4 > gpurun_out/gputests.txt; cat gpurun_out/gputests.txt
timeout 900 python bench.py 2>/dev/null | tail -1 > gpurun_out/bench_default.json
python -c "
import json;d=json.load(open('gpurun_out/bench_default.json'));print(d['value'], d['roofline']['frac'], d['resident']['value'], d['resident']['roofline']['frac'], d['resident']['roofline']['kernel'])"
timeout 900 python bench.py --config fig5 --steps 3 --warmup 3 2>/dev/null | tail -1 > gpurun_out/fig5_default.json
python -c "
import json;d=json.load(open('gpurun_out/fig5_default.json'));print({T:(round(v['tiled']['ms'],1), v['tiled']['schedule'][:12]) for T,v in d['sweep'].items()})"
