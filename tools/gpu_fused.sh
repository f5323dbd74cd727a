#!/bin/bash
# fused peer halo push: GPU tests (one process per rank on the one GPU) + bench N=2 hook
mkdir -p gpurun_out/fused
python __graft_entry__.py > /dev/null 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/fused/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/fused/pytest_gpu.log
for tr in peer peer-copy; do
TILES_BENCH_ONE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --no-cpu-baseline --no-extras --transport $tr > gpurun_out/fused/bench2_$tr.json 2> gpurun_out/fused/bench2_$tr.err
echo "bench2 $tr rc=$?"; tail -c 600 gpurun_out/fused/bench2_$tr.json
done
