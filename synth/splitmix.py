"""Counter-based splitmix64 generator (NumPy) + structured fields for closed forms.

See synth/__init__.py for the recipe. Nothing here computes the heat update or
the compute-intensive kernel; the structured fields (constant, linear, sine
modes) are inputs whose exact evolution is known in closed form.
"""
import ctypes
import os
import numpy as np

GOLDEN_GAMMA = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)


def splitmix64(z):
    """splitmix64 finaliser of (z + gamma); z is a uint64 array or scalar."""
    z = np.asarray(z, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = z + GOLDEN_GAMMA
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
    return z ^ (z >> np.uint64(31))


def uniform_at(gidx, seed):
    """U[0,1) value of global linear index gidx (uint64 array)."""
    gidx = np.asarray(gidx, dtype=np.uint64)
    with np.errstate(over="ignore"):
        key = gidx + np.uint64(seed) * GOLDEN_GAMMA
    r = splitmix64(key) >> np.uint64(11)
    return r.astype(np.float64) * (2.0 ** -53)


def uniform_block(nx, ny, nz, seed, z0=0, y0=0, x0=0, bz=None, by=None, bx=None,
                  wrap=True):
    """Sub-block [z0,z0+bz) x [y0,..) x [x0,..) of the global (nz,ny,nx) grid.

    Coordinates may lie outside the grid; with wrap=True they wrap periodically
    (used by the cone oracle to regenerate neighbourhoods across seams).
    """
    bz = nz if bz is None else bz
    by = ny if by is None else by
    bx = nx if bx is None else bx
    zz = np.arange(z0, z0 + bz, dtype=np.int64)
    yy = np.arange(y0, y0 + by, dtype=np.int64)
    xx = np.arange(x0, x0 + bx, dtype=np.int64)
    if wrap:
        zz %= nz; yy %= ny; xx %= nx
    g = ((zz[:, None, None] * ny + yy[None, :, None]) * nx + xx[None, None, :])
    return uniform_at(g.astype(np.uint64), seed)


def uniform_grid(nx, ny, nz, seed=42):
    """Whole (nz, ny, nx) grid, C-order, x fastest."""
    return uniform_block(nx, ny, nz, seed)


def constant_grid(nx, ny, nz, c=0.3):
    return np.full((nz, ny, nx), c, dtype=np.float64)


def linear_grid(nx, ny, nz, g=0, coeff=(1.0, 2.0, 3.0)):
    """u = a*x + b*y + c*z on [-g, n+g) per axis (halo included when g>0)."""
    x = np.arange(-g, nx + g, dtype=np.float64)
    y = np.arange(-g, ny + g, dtype=np.float64)
    z = np.arange(-g, nz + g, dtype=np.float64)
    a, b, c = coeff
    return (a * x[None, None, :] + b * y[None, :, None] + c * z[:, None, None])


def sine_grid(nx, ny, nz, m=(1, 1, 1)):
    """Periodic mode prod_d sin(2*pi*m_d*i_d/n_d)."""
    x = np.sin(2 * np.pi * m[0] * np.arange(nx) / nx)
    y = np.sin(2 * np.pi * m[1] * np.arange(ny) / ny)
    z = np.sin(2 * np.pi * m[2] * np.arange(nz) / nz)
    return z[:, None, None] * y[None, :, None] * x[None, None, :]


def sine_grid_dirichlet(nx, ny, nz, m=(1, 1, 1), g=1):
    """Dirichlet-zero mode prod_d sin(pi*m_d*(i_d+1)/(n_d+1)) on [-g, n+g).

    The halo cells i=-1 and i=n evaluate to sin(0)=0 and sin(pi*m)~0; they are
    forced to exact zeros (fixed Dirichlet boundary).
    """
    def ax(n, md):
        i = np.arange(-g, n + g)
        v = np.sin(np.pi * md * (i + 1) / (n + 1))
        v[(i < 0) | (i >= n)] = 0.0
        return v
    x, y, z = ax(nx, m[0]), ax(ny, m[1]), ax(nz, m[2])
    return z[:, None, None] * y[None, :, None] * x[None, None, :]


_native = None


def _load_native():
    global _native
    if _native is None:
        here = os.path.dirname(os.path.abspath(__file__))
        path = os.path.join(here, "libsynth.so")
        if not os.path.exists(path):
            import subprocess
            subprocess.check_call(["gcc", "-O2", "-fPIC", "-shared", "-fopenmp",
                                   os.path.join(here, "splitmix.c"), "-o", path])
        lib = ctypes.CDLL(path)
        lib.synth_fill_uniform.argtypes = [ctypes.c_void_p] + [ctypes.c_int64] * 9 + [ctypes.c_uint64]
        lib.synth_fill_uniform.restype = None
        _native = lib
    return _native


def fill_uniform_native(out_ptr, nx, ny, nz, z0, bz, y0, by, x0, bx, seed):
    """Fill a C-order (bz,by,bx) float64 buffer at out_ptr with the generator
    (C twin of uniform_block, multi-threaded; for grids of tens of GB)."""
    _load_native().synth_fill_uniform(ctypes.c_void_p(out_ptr), nx, ny, nz, z0, bz,
                                      y0, by, x0, bx, ctypes.c_uint64(seed))
