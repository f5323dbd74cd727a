#!/bin/bash
# Re-entry check: build, GPU tests, smoke, default bench line.
O=gpurun_out/s2a
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || { tail -20 $O/build.txt; exit 1; }
timeout 2400 python -m pytest tests -m gpu -q -x 2>&1 | tail -15 > $O/gputests.txt; cat $O/gputests.txt
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.txt 2>&1; tail -1 $O/smoke.txt
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err; cat $O/bench.json | head -c 3000
