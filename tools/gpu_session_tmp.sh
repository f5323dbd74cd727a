python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q -m gpu -k "stream" 2>&1 | tail -2
for rep in 1 2; do
for cfg in "0 2" "1 2" "1 1" "1 3" "0 1"; do
set -- $cfg
v=$(TILES_ST_OFFSET=$1 TILES_ST_H2D_MERGE=$2 timeout 300 python bench.py --no-extras --no-cpu-baseline --steps 20 --warmup 3 2>/dev/null | tail -1 | python -c "import json,sys;d=json.load(sys.stdin);print(round(d['ms_per_step'],3), round(d['value'],2))")
echo "offset=$1 merge=$2 : $v"
done; done
TILES_ST_OFFSET=1 python tools/timeline.py c2 gpurun_out/tl_c2o > /dev/null 2>&1; rm -f gpurun_out/tl_c2o.trace.json
