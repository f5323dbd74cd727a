"""Profiling driver: C2 resident heat steps (for ncu). Launch order:
8 layer-batched launches (first run loads the grid), then whole-domain launches."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import synth
from paper_conf_icpp_bastemuzas17_b200 import tiles as T
n = int(os.environ.get("N", "512")); t = int(os.environ.get("TILE", "64"))
# DIMS="nx,ny,nz" / TD="tx,ty,tz" override the cube (e.g. a C5 slab: 4096,4096,128 / 256,256,64)
dims = tuple(int(v) for v in os.environ["DIMS"].split(",")) if "DIMS" in os.environ else (n, n, n)
td = tuple(int(v) for v in os.environ["TD"].split(",")) if "TD" in os.environ else (t, t, t)
u = np.empty(dims[::-1]); synth.fill_uniform_native(u.ctypes.data, *dims, 0, dims[2], 0, dims[1], 0, dims[0], 42)
d = T.Domain(dims, td, ghost=int(os.environ.get("GHOST", "1")), stream_through=-1,
             two_step=int(os.environ.get("TWO_STEP", "0")))
d.load(u); d.run(T.heat7(), 1, 4); d.sync()
d.run(T.heat7(), int(os.environ.get("STEPS", "4")), 4); d.sync()
print("prof ok")
print("steps_per_pass", d.info["steps_per_pass"], "kernels", d.stats()["n_kernels"])
