python -c "import __graft_entry__ as g; g.build()" || exit 1
cat > /tmp/b2one.py <<'PY'
import os, sys
sys.path.insert(0, os.getcwd())
import numpy as np, synth
from paper_conf_icpp_bastemuzas17_b200 import tiles as T
n = 512
u = np.empty((n, n, n)); synth.fill_uniform_native(u.ctypes.data, n, n, n, 0, n, 0, n, 0, n, 42)
d = T.Domain((n, n, n), (64, 64, 64), sweep_link_ratio=0.021)
d.load(u); d.run(T.heat7(), 1, 4); d.sync()
d.run(T.heat7(), 10, 4); d.sync()
PY
timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat2_band -s 2 -c 1 -o gpurun_out/band2d_full python /tmp/b2one.py > /dev/null 2>&1
ncu -i gpurun_out/band2d_full.ncu-rep --page raw --csv > gpurun_out/band2d_full.raw.csv 2>/dev/null
ncu -i gpurun_out/band2d_full.ncu-rep --page source --csv --print-source sass > gpurun_out/band2d_full.sass.csv 2>/dev/null
ncu -i gpurun_out/band2d_full.ncu-rep --page details --csv > gpurun_out/band2d_full.details.csv 2>/dev/null
