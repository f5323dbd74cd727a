"""C2 resident rate: heat2_band (two steps per kernel) vs the persistent
single-step launch (two_step=-1), T = 10 per run, CUDA events."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import synth
from paper_conf_icpp_bastemuzas17_b200 import tiles as T
n = 512
u = np.empty((n, n, n)); synth.fill_uniform_native(u.ctypes.data, n, n, n, 0, n, 0, n, 0, n, 42)
for ts in (0, -1, 0, -1):
    d = T.Domain((n, n, n), (64, 64, 64), two_step=ts)
    d.load(u); d.run(T.heat7(), 1, 4); d.sync()
    for _ in range(3):
        d.run(T.heat7(), 10, 4)
    d.sync()
    d.set_kernel_timing(True); d.reset_stats()
    d.timer_start()
    for _ in range(10):
        d.run(T.heat7(), 10, 4)
    ms = d.timer_stop()
    st = d.stats()
    print(f"two_step={ts:2d} sched={d.get_info()['last_schedule']} {ms/10:.3f} ms/10 steps "
          f"{n**3*100/ms/1e6:.1f} Gcell/s  kernels={st['n_kernels']} sweep_ms={st['sweep_ms']:.2f} "
          f"alg={16*st['sweep_cells']/st['sweep_ms']/1e6:.0f} GB/s", flush=True)
    d.free()
