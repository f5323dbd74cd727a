#!/bin/bash
# Last check of the session: build, every GPU test, smoke, the default bench line.
O=gpurun_out/r2f7
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || { tail -20 $O/build.txt; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q 2>&1 | tail -3 > $O/gputests.txt; cat $O/gputests.txt
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1; tail -1 $O/smoke.txt
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
python -c "
import json; d=json.load(open('$O/bench.json')); print('value', round(d['value'],2), 'frac', round(d['roofline']['frac'],3), 'resident', round(d['resident']['value'],1), 'link', round(d['roofline_link']['frac'],3))"
