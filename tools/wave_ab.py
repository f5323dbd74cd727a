"""Fresh-upload C2 runs at the given Ts (the Fig. 5 tiled leg), several
repetitions: min / median ms per T as one JSON line. Env knobs pass through
(A/B runs of kernel variants).   python tools/wave_ab.py 32,48,64,100 [reps]"""
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import synth  # noqa: E402
from paper_conf_icpp_bastemuzas17_b200 import tiles as T  # noqa: E402

Ts = [int(v) for v in sys.argv[1].split(",")]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
n = 512
u = np.empty((n, n, n))
synth.fill_uniform_native(u.ctypes.data, n, n, n, 0, n, 0, n, 0, n, 42)
d = T.Domain((n, n, n), (64, 64, 64), device=0)
d.load(u)
k = T.heat7(0.125)
out = {}
for t in Ts:
    d.invalidate()
    d.run(k, t, 4)
    d.sync()
    ms = []
    for _ in range(reps):
        d.invalidate()
        d.timer_start()
        d.run(k, t, 4)
        d.sync()
        ms.append(d.timer_stop())
    out[t] = {"min": round(min(ms), 2), "median": round(statistics.median(ms), 2)}
print(json.dumps(out))
