#!/bin/bash
O=gpurun_out/s2r
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || exit 1
s=$(date +%s); timeout 600 python bench.py --config c5 --steps 2 --warmup 1 > $O/c5.json 2> $O/c5.err; e=$(date +%s); echo "c5 secs $((e-s))"
head -c 1500 $O/c5.json; echo
s=$(date +%s); timeout 900 python bench.py > $O/bench.json 2> $O/bench.err; e=$(date +%s); echo "default bench secs $((e-s))"
