#!/bin/bash
O=gpurun_out/s2t
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.txt 2>&1 || exit 1
timeout 600 python -m pytest tests/test_host_regions.py tests/test_errors.py -m gpu -q 2>&1 | tail -3 | tee $O/tests.txt
