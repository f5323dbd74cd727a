#!/bin/bash
O=gpurun_out/s2s
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || exit 1
s=$(date +%s); timeout 900 python bench.py > $O/bench.json 2> $O/bench.err; e=$(date +%s); echo "default bench secs $((e-s))"
python -c "
import json; d=json.load(open('$O/bench.json')); print('value', round(d['value'],2), 'c3', d['c3'].get('value'), 'c4', d['c4'].get('value'), 'c5', json.dumps(d.get('c5'))[:600])"
tail -3 $O/bench.err
timeout 300 python bench.py --config c5 --steps 2 --warmup 1 > $O/c5.json 2>/dev/null; head -c 300 $O/c5.json
