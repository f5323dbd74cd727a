python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "band2" 2>&1 | tail -3
timeout 300 python tools/band2_probe.py 2>&1 | tail -4
