python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "wavefront" 2>&1 | grep -E "^E|FAILED|Error" | head -20
