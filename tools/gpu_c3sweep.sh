#!/bin/bash
python __graft_entry__.py > /dev/null 2>&1
for cfg in "8 2 2" "16 2 2" "8 4 2" "4 4 2"; do
  set -- $cfg
  timeout 900 python bench.py --config c3 --steps 1 --warmup 1 --nstreams $1 --T $2 --ghost $3 > gpurun_out/c3.json 2> gpurun_out/c3.err
  python -c "import json; j=json.load(open('gpurun_out/c3.json')); print('ns=$1 T=$2 g=$3', round(j['value'],2), round(j['roofline']['frac'],3), round(j['roofline']['achieved'],1), j['overlap']['hidden_frac'])"
done
