#!/bin/bash
# bench N=2/4 through torchrun with both ranks on the pool's one GPU (functional check of the
# multi-rank e2e path, not a performance number), then N=1 merge A/B
mkdir -p gpurun_out/n2st
python __graft_entry__.py > /dev/null 2>&1
for n in 2 4; do
TILES_BENCH_ONE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 2953$n bench.py --gpus $n --steps 4 --warmup 3 --no-cpu-baseline > gpurun_out/n2st/bench$n.json 2> gpurun_out/n2st/bench$n.err; echo "n=$n rc=$?"
python -c "import json;j=json.load(open('gpurun_out/n2st/bench$n.json'));print('value',round(j['value'],1),'e2e',round(j['e2e']['value'],1), j['e2e'], j.get('overlap'), j['config']['parallelism'])"
done
for m in 1 2 1 2; do
  TILES_ST_H2D_MERGE=$m timeout 300 python bench.py --no-cpu-baseline --steps 10 > gpurun_out/n2st/m$m.json 2>/dev/null
  python -c "import json;j=json.load(open('gpurun_out/n2st/m$m.json'));print('merge',$m,'e2e ms',round(j['e2e']['ms_per_step'],3),'hidden',round(j['overlap']['hidden_frac'],3),'xo',round(j['overlap']['t_xfer_only_ms'],2),'frac',round(j['e2e_roofline']['frac'],3),'h2d',round(j['e2e_roofline']['pcie_gbs']['h2d'],1))"
done
