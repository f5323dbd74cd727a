"""C2-shaped resident run (512^3, 64^3 tiles, T = 10) with the heat update as
a user stencil (NVRTC, face ghosts, one thread per cell) vs the built-in
heat7_fixed: Gcell-updates/s from the library's device timer, median of 5."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import synth
from paper_conf_icpp_bastemuzas17_b200 import tiles as T

n = 512
u = np.empty((n, n, n))
synth.fill_uniform_native(u.ctypes.data, n, n, n, 0, n, 0, n, 0, n, 42)
fs = T.UserFn("__device__ double hu(double c, double xm, double xp, double ym, double yp, double zm, double zp)"
              " { return c + 0.125 * ((((xm + xp) + (ym + yp)) + (zm + zp)) - 6.0 * c); }", "hu", stencil=True)
with T.Domain((n, n, n), (64, 64, 64)) as d:
    d.load(u)
    d.run(T.heat7(), 1, 4)
    d.sync()
    for name, k in (("heat7_fixed (built-in)", T.heat7()), ("user stencil (NVRTC)", T.user_stencil(fs))):
        d.run(k, 10, 4)
        d.sync()
        ts = []
        for _ in range(5):
            d.timer_start()
            d.run(k, 10, 4)
            ts.append(d.timer_stop())
        ms = float(np.median(ts))
        print(f"{name}: {n ** 3 * 10 / (ms / 1e3) / 1e9:.1f} Gcell/s ({ms:.2f} ms per 10 steps, "
              f"{16 * n ** 3 * 10 / (ms / 1e3) / 1e9:.0f} GB/s algorithmic)", flush=True)
