#!/bin/bash
mkdir -p gpurun_out/c5tile
python __graft_entry__.py > /dev/null 2>&1
for t in 64,64,64 128,128,64 256,256,64; do
  timeout 900 python bench.py --config c5 --steps 6 --no-cpu-baseline --tile $t > gpurun_out/c5tile/c5_$t.json 2> gpurun_out/c5tile/c5_$t.err; echo "rc=$?"
  python -c "import json;j=json.load(open('gpurun_out/c5tile/c5_$t.json'));print('C5 tile $t value',round(j['value'],1),'frac',round(j['roofline']['frac'],3),'e2e',round(j['e2e']['value'],1),'setup',round(j['config']['setup_s'],1), j['config']['host_cpus'] if 'host_cpus' in j['config'] else '')"
done
timeout 300 python bench.py --no-cpu-baseline --no-extras --steps 10 > gpurun_out/c5tile/c2.json 2>/dev/null; python -c "import json;j=json.load(open('gpurun_out/c5tile/c2.json'));print('C2', round(j['value'],1), j['config'].get('host_cpus'))"
