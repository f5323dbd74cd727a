#!/bin/bash
# Tuning sweep of heat7 specialisations (band rows x ring stages) on C2.
python __graft_entry__.py >/dev/null
for cfg in "${@:-64_4}"; do
  cfg=${cfg//_/ }
  set -- $cfg
  for i in 1 2; do
    r=$(TILES_HEAT_CACHE=${3:-0} TILES_HEAT_BAND=$1 TILES_HEAT_STAGES=$2 python bench.py --no-extras --no-cpu-baseline --steps 30 | python -c "import json,sys; j=json.load(sys.stdin); print(round(j['value'],1), round(j['roofline']['frac'],3))")
    echo "band=$1 stages=$2 cache=${3:-0} : $r"
  done
done
