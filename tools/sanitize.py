"""Small runs of every schedule for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck): resident heat (layered + whole-domain phases),
streaming heat with a tiny budget, Dirichlet, sincos, the generic kernel, the
persistent multi-step launch (direct ghosts, grid counter, snake order; banded tiles in round-robin order), a ranged NVRTC user kernel, a user stencil and
the stream-through schedule, the wavefront (tile-column TMA sweeps with
tensor-map x halos), the band kernels (heat2_band, heat2_band_slab) and the
in-process multi-rank transport."""
import os
import sys
import threading

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np

import synth
from paper_conf_icpp_bastemuzas17_b200 import tiles as T


def budget(dims, td, n, **kw):
    lo, hi = 1, 1 << 36
    while lo < hi:
        mid = (lo + hi) // 2
        try:
            k = T.Domain(dims, td, dry_run=True, sched="stream", device_budget_bytes=mid, **kw).info["nslots"]
        except T.TileError:
            k = -1
        lo, hi = (lo, mid) if k >= n else (mid + 1, hi)
    return lo


u = synth.uniform_grid(64, 32, 32, 42)
with T.Domain((64, 32, 32), (32, 16, 8)) as d:          # fixed kernel (32,16), 4 layers -> phases
    d.load(u); d.run(T.heat7(), 6, 2); d.store()
    d.run(T.heat7(), 5, 2); d.store()                    # resident: one persistent multi-step launch
ext0 = synth.uniform_grid(66, 34, 34, 6)
with T.Domain((64, 32, 32), (32, 16, 8), bc="dirichlet") as d:   # direct ghosts + Dirichlet, persistent
    d.load(ext0); d.run(T.heat7(), 2, 2); d.sync(); d.run(T.heat7(), 4, 2); d.store()
with T.Domain((48, 40, 20), (24, 20, 5)) as d:          # generic kernel
    d.load(synth.uniform_grid(48, 40, 20, 1)); d.run(T.heat7(), 3, 2); d.store()
with T.Domain((64, 32, 32), (32, 16, 8), sched="stream", device_budget_bytes=budget((64, 32, 32), (32, 16, 8), 3)) as d:
    d.load(u); d.run(T.heat7(), 3, 2); d.store()
ext = synth.uniform_grid(66, 34, 34, 5)
with T.Domain((64, 32, 32), (32, 16, 16), bc="dirichlet") as d:
    d.load(ext); d.run(T.heat7(), 3, 2); d.store()
with T.Domain((64, 32, 32), (32, 16, 16)) as d:
    d.load(u); d.run(T.sincos(2), 2, 2); d.store()
us = synth.uniform_grid(64, 64, 256, 3)                   # stream-through (units of 16 planes)
with T.Domain((64, 64, 256), (64, 64, 32)) as d:
    d.load(us); d.run(T.heat7(), 2, 2); d.store(); d.run(T.heat7(), 1, 2); d.store()
with T.Domain((64, 64, 256), (32, 32, 32)) as d:          # stream-through, unit = tile layer
    d.load(us); d.run(T.heat7(), 10, 2); d.store()
with T.Domain((128, 64, 64), (64, 64, 16), ghost=2, two_step=1) as d:   # heat7x2 (two steps per pass)
    d.load(synth.uniform_grid(128, 64, 64, 9)); d.run(T.heat7(), 6, 2); d.store()
uo = synth.uniform_grid(64, 64, 256, 4)                   # out-of-core stream-through (unit ring)
bo = budget((64, 64, 256), (32, 32, 32), 30)
with T.Domain((64, 64, 256), (32, 32, 32), sched="stream", device_budget_bytes=bo) as d:
    d.load(uo); d.run(T.heat7(), 5, 3); d.store()
with T.Domain((128, 64, 64), (64, 64, 16), ghost=2, two_step=1) as d:   # heat7x2r (band 32)
    d.load(synth.uniform_grid(128, 64, 64, 11)); d.run(T.heat7(), 4, 2); d.store()
ub = synth.uniform_grid(512, 512, 16, 12)                 # banded tiles: round-robin columns,
with T.Domain((512, 512, 16), (32, 64, 8)) as d:          # snake-ordered persistent launch
    d.load(ub); d.run(T.heat7(), 1, 2); d.sync(); d.run(T.heat7(), 4, 2); d.store()
fu = T.UserFn("__device__ double aff(double u, long long g) { return 2.0 * u + 1.0; }", "aff")
with T.Domain((64, 32, 32), (32, 16, 16)) as d:           # user pointwise kernel (NVRTC), ranged
    d.load(u); d.run(T.user(fu, 2, box=((5, 3, 7), (40, 16, 32))), 2, 2); d.store()
fs = T.UserFn("__device__ double hu(double c, double xm, double xp, double ym, double yp, double zm, double zp)"
              " { return c + 0.125 * ((((xm + xp) + (ym + yp)) + (zm + zp)) - 6.0 * c); }", "hu", stencil=True)
with T.Domain((64, 32, 32), (32, 16, 16)) as d:           # user stencil (NVRTC, face ghosts)
    d.load(u); d.run(T.user_stencil(fs), 3, 2); d.run(T.heat7(), 2, 2); d.store()
uw = synth.uniform_grid(128, 64, 256, 13)                 # wavefront (T > tz: scratch layers, bootstrap),
with T.Domain((128, 64, 256), (64, 64, 32), wavefront=1) as d:   # tile-column TMA sweeps
    d.load(uw); d.run(T.heat7(), 40, 2); d.store(); d.run(T.heat7(), 2, 2); d.store()
    d.invalidate(); d.run(T.heat7(), 7, 3); d.store()
with T.Domain((128, 64, 256), (64, 64, 32), stream_through=1, wavefront=-1) as d:  # stream-through, tile kernel
    d.load(uw); d.run(T.heat7(), 12, 2); d.store()
ub2 = synth.uniform_grid(512, 16, 32, 14)                # heat2_band (resident, 512 wide, two steps per kernel)
with T.Domain((512, 16, 32), (64, 16, 16)) as d:
    d.load(ub2); d.run(T.heat7(), 1, 2); d.sync(); d.run(T.heat7(), 4, 2); d.store(); d.run(T.heat7(), 3, 2); d.store()
uw2 = synth.uniform_grid(512, 16, 128, 15)               # wavefront, two-level band passes (heat2_band_slab)
with T.Domain((512, 16, 128), (64, 16, 16), wavefront=1) as d:
    d.load(uw2); d.run(T.heat7(), 12, 2); d.store()
with T.Domain((512, 8, 128), (64, 4, 8), stream_through=1, wavefront=-1, two_step=1) as d:  # two sweeps per kernel
    d.load(synth.uniform_grid(512, 8, 128, 16)); d.run(T.heat7(), 5, 2); d.store()
g = T.LocalGroup(2)
def rank(r):
    with T.Domain((64, 32, 64), (32, 16, 16), nranks=2, rank=r, local_group=g) as d:
        d.load(synth.uniform_grid(64, 32, 64, 42)[r * 32:(r + 1) * 32]); d.run(T.heat7(), 4, 2); d.store()
th = [threading.Thread(target=rank, args=(r,)) for r in range(2)]
[t.start() for t in th]; [t.join() for t in th]
g.free()
print("sanitize driver ok")
