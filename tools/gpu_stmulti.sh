#!/bin/bash
# multi-rank stream-through: parity (processes on one GPU), then the regression suite
mkdir -p gpurun_out
python __graft_entry__.py > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_multirank.py -x -q -k "stream_through" > gpurun_out/pytest_stmulti.log 2>&1; echo "st-multi rc=$?"; tail -15 gpurun_out/pytest_stmulti.log
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_gpu.log
