"""Profiling driver: one C2 (512^3, 64^3 tiles) stream-through run of T steps
(env T, default 10; forced stream-through) from a fresh upload, for ncu."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import synth
from paper_conf_icpp_bastemuzas17_b200 import tiles as T
n = int(os.environ.get("N", "512")); t = int(os.environ.get("TILE", "64")); steps = int(os.environ.get("T", "10"))
u = np.empty((n, n, n)); synth.fill_uniform_native(u.ctypes.data, n, n, n, 0, n, 0, n, 0, n, 42)
d = T.Domain((n, n, n), (t, t, t), stream_through=1)
d.load(u); d.run(T.heat7(), steps, 4); d.sync()
print("prof ok", d.stats()["n_kernels"])
