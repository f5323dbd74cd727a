python -c "import __graft_entry__ as g; g.build()" || exit 1
for rep in 1 2; do
for cfg in "1 1 2" "2 1 2" "1 2 2" "2 2 2" "2 2 1" "4 4 2"; do
set -- $cfg
v=$(TILES_ST_IN=$1 TILES_ST_OUT=$2 TILES_ST_H2D_MERGE=$3 timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 20 --warmup 3 2>/dev/null | tail -1 | python -c "import json,sys;d=json.load(sys.stdin);print(round(d['ms_per_step'],3), round(d['value'],2))")
echo "in=$1 out=$2 merge=$3 : $v"
done; done
