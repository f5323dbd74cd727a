"""Profiling driver for the sweep kernels: one C2 (512^3, 64^3 tiles)
fresh-upload run of T steps (env T, default 10) on the schedule env SCHED
(stream = stream-through forced, wave = wavefront forced, wave2 = two
levels per pass; TILES_WAVE_C sets
the wavefront chunk), then a resident run, for ncu -k regex:slab_sweep."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import synth
from paper_conf_icpp_bastemuzas17_b200 import tiles as T
n = int(os.environ.get("N", "512")); steps = int(os.environ.get("T", "10"))
sched = os.environ.get("SCHED", "wave")
u = np.empty((n, n, n)); synth.fill_uniform_native(u.ctypes.data, n, n, n, 0, n, 0, n, 0, n, 42)
kw = {"wavefront": 2 if sched == "wave2" else 1} if sched.startswith("wave") else \
    {"stream_through": 1, "wavefront": -1}
kw["sweep_link_ratio"] = 0.021  # fixed: the device calibration under ncu would see replayed kernels
d = T.Domain((n, n, n), (64, 64, 64), **kw)
d.load(u); d.run(T.heat7(), steps, 4); d.sync()
print("prof ok", d.get_info()["last_schedule"], d.stats()["n_kernels"])
