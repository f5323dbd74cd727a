python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -m gpu -k "band2_resident or split or band2_middle" 2>&1 | tail -2
for rr in 1 0 1 0; do echo "runs=$rr"; TILES_BAND2_RUNS=$rr timeout 300 python tools/band2_probe.py 2>&1 | grep "two_step= 0" | head -1; done
