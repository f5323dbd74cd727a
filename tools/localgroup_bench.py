"""Multi-rank resident schedule overhead on ONE GPU: G z-slab ranks of a
512^3 grid as threads of one process (in-process transport, tile_local_group),
all sharing cuda:0 concurrently (one context, no time-slicing), vs the same
grid as one rank. Aggregate Gcell-updates/s of T = 10 resident steps, median
of 5 runs. A proxy for the per-step halo schedule's cost, not a scaling number.

  python tools/localgroup_bench.py [G ...]
"""
import os
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import synth
from paper_conf_icpp_bastemuzas17_b200 import tiles as T

n, td, steps = 512, (64, 64, 64), 10


def run(G):
    u = np.empty((n, n, n))
    synth.fill_uniform_native(u.ctypes.data, n, n, n, 0, n, 0, n, 0, n, 42)
    nzl = n // G
    g = T.LocalGroup(G) if G > 1 else None
    doms = [T.Domain((n, n, n), td, nranks=G, rank=r, device=0, local_group=g) if G > 1
            else T.Domain((n, n, n), td, device=0) for r in range(G)]
    for r, d in enumerate(doms):
        d.load(u[r * nzl:(r + 1) * nzl])
    times = []
    for rep in range(7):
        bar = threading.Barrier(G)
        out = [0.0] * G

        def work(r):
            d = doms[r]
            if rep == 0:  # the first run after the upload is the stream-through e2e path
                d.run(T.heat7(0.125), 1, 4)
                d.sync()
            bar.wait()
            d.timer_start()  # device time of this rank's streams (no host write-back)
            d.run(T.heat7(0.125), steps, 4)
            out[r] = d.timer_stop() / 1e3
        th = [threading.Thread(target=work, args=(r,)) for r in range(G)]
        [t.start() for t in th]
        [t.join() for t in th]
        if rep >= 2:
            times.append(max(out))
    for d in doms:
        d.free()
    if g:
        g.free()
    t = float(np.median(times))
    return n ** 3 * steps / t / 1e9, t * 1e3


if __name__ == "__main__":
    torch.cuda.set_device(0)
    for G in [int(a) for a in sys.argv[1:]] or [1, 2, 4]:
        v, ms = run(G)
        print(f"G={G}: {v:.1f} Gcell/s aggregate ({ms:.2f} ms per {steps} steps)", flush=True)
