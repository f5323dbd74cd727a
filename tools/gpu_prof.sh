#!/bin/bash
# round profile set: tests, headline bench (x2), 2-rank hook bench, ncu launch list + full heat7 capture
mkdir -p gpurun_out/prof
python __graft_entry__.py > /dev/null 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/prof/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/prof/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/prof/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/prof/pytest_gpu.log
for i in 1 2; do
timeout 900 python bench.py > gpurun_out/prof/bench_$i.json 2> gpurun_out/prof/bench_$i.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/prof/bench_$i.json'));print(round(d['value'],1), round(d['roofline']['frac'],4), 'e2e', round(d['e2e']['value'],2), 'hidden', round(d['overlap']['hidden_frac'],3), 'e2e_roof', round(d['e2e_roofline']['frac'],3), d['clocks'])"
done
for tr in peer peer-copy; do
TILES_BENCH_ONE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --no-cpu-baseline --no-extras --transport $tr > gpurun_out/prof/bench2_$tr.json 2> gpurun_out/prof/bench2_$tr.err
python -c "import json;d=json.load(open('gpurun_out/prof/bench2_$tr.json'));print('2 ranks on 1 GPU $tr', round(d['value'],1), round(d['ms_per_step'],2))"
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/prof/launches.csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --no-extras \
  > gpurun_out/prof/ncu_launch_bench.log 2>&1; echo "launch list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:heat7 -s 10 -c 1 \
  -o gpurun_out/prof/heat7_full -f python tools/prof_heat.py > gpurun_out/prof/ncu_full.log 2>&1; echo "full rc=$?"
