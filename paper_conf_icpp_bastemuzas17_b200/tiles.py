"""Thin ctypes binding of libtiles (include/tiles.h): argument marshalling only.

Every step of the hot path runs inside libtiles' CUDA kernels; this module
only converts Python/NumPy arguments and raises on error codes. The function
names mirror the C ABI (tile_domain_create, tile_load, tile_run, tile_sync,
tile_store, tile_free, ...); `Domain` is a convenience wrapper around them.

There is no fallback: if libtiles.so is missing, importing this module
raises ImportError (build it with `python paper_conf_icpp_bastemuzas17_b200/build.py`).
"""
import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libtiles.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        "libtiles.so not built: run `python paper_conf_icpp_bastemuzas17_b200/build.py` "
        "(there is no CPU fallback)")
_lib = ctypes.CDLL(LIB_PATH, mode=ctypes.RTLD_GLOBAL)

# ----------------------------------------------------------------- constants
TILE_OK, TILE_EINVAL, TILE_ENOMEM_HOST, TILE_ENOMEM_DEVICE, TILE_ECUDA, TILE_ENCCL, \
    TILE_ESTATE, TILE_ENOSYS = range(8)
STATUS_NAMES = {0: "OK", 1: "EINVAL", 2: "ENOMEM_HOST", 3: "ENOMEM_DEVICE", 4: "ECUDA",
                5: "ENCCL", 6: "ESTATE", 7: "ENOSYS"}
TILE_BC_PERIODIC, TILE_BC_DIRICHLET = 0, 1
TILE_KERNEL_HEAT7, TILE_KERNEL_SINCOS, TILE_KERNEL_USER, TILE_KERNEL_USER_STENCIL = 1, 2, 3, 4
TILE_SCHED_AUTO, TILE_SCHED_RESIDENT, TILE_SCHED_STREAM, TILE_SCHED_SYNC = 0, 1, 2, 3
TILE_MEASURE_NORMAL, TILE_MEASURE_XFER_ONLY, TILE_MEASURE_COMP_ONLY = 0, 1, 2
OP_NAMES = {1: "h2d", 2: "d2h", 3: "kernel", 4: "record", 5: "wait", 6: "faces_h2d",
            7: "extract", 8: "halo", 9: "drop", 10: "hit", 11: "pointwise", 12: "kernel2",
            13: "gather", 14: "sweep", 15: "scatter", 16: "copy", 17: "h2d_part", 18: "d2h_part",
            19: "copy_part", 20: "h2d_pack", 21: "sweep_u", 22: "kerneld", 23: "halo_signal",
            24: "st_halo", 25: "sync", 26: "wsweep", 27: "d2h_planes", 28: "copy_planes",
            29: "wsweep2", 30: "wsweep2_dst", 31: "band2",
            32: "sweep2s"}
SCHEDS = {"auto": 0, "resident": 1, "stream": 2, "sync": 3}
BCS = {"periodic": 0, "dirichlet": 1}


class TileOptions(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int32), ("bc", ctypes.c_int), ("device_budget_bytes", ctypes.c_uint64),
                ("device_pool", ctypes.c_void_p), ("device_pool_bytes", ctypes.c_uint64),
                ("streams", ctypes.POINTER(ctypes.c_void_p)), ("nstreams_provided", ctypes.c_int32),
                ("nranks", ctypes.c_int32), ("rank", ctypes.c_int32),
                ("nccl_unique_id", ctypes.c_void_p), ("sched", ctypes.c_int),
                ("dry_run", ctypes.c_int32), ("fuse_pointwise_steps", ctypes.c_int32),
                ("local_group", ctypes.c_void_p), ("pageable_host", ctypes.c_int32),
                ("stream_through", ctypes.c_int32), ("peer_transport", ctypes.c_int32),
                ("two_step", ctypes.c_int32), ("wavefront", ctypes.c_int32),
                ("sweep_link_ratio", ctypes.c_double)]


class TileKernel(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int), ("alpha", ctypes.c_double), ("inner_iters", ctypes.c_int32),
                ("user", ctypes.c_void_p), ("box", ctypes.POINTER(ctypes.c_int64))]


class TileStats(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in ("bytes_h2d", "bytes_d2h", "bytes_halo", "n_h2d", "n_d2h",
                                               "n_kernels", "n_halo", "hits", "misses", "evictions",
                                               "writebacks", "steps_done")] + [
        ("last_run_ms", ctypes.c_double), ("kernel_ms", ctypes.c_double), ("kernel_timed", ctypes.c_uint64),
        ("sweep_ms", ctypes.c_double), ("sweep_cells", ctypes.c_uint64), ("sweep_timed", ctypes.c_uint64)]

    def as_dict(self):
        return {n: getattr(self, n) for n, _ in self._fields_}


class TileInfo(ctypes.Structure):
    _fields_ = [("dims", ctypes.c_int64 * 3), ("local_dims", ctypes.c_int64 * 3),
                ("tile_dims", ctypes.c_int64 * 3), ("tiles", ctypes.c_int64 * 3),
                ("ntiles", ctypes.c_int64), ("z_offset", ctypes.c_int64), ("ghost", ctypes.c_int32),
                ("nslots", ctypes.c_int32), ("sched", ctypes.c_int32), ("resident", ctypes.c_int32),
                ("device_bytes", ctypes.c_uint64), ("host_bytes", ctypes.c_uint64),
                ("steps_per_pass", ctypes.c_int32), ("last_schedule", ctypes.c_int32),
                ("sweep_link_ratio", ctypes.c_double)]

    def as_dict(self):
        out = {}
        for n, _ in self._fields_:
            v = getattr(self, n)
            out[n] = tuple(v) if hasattr(v, "__len__") else v
        return out


class TileOp(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int32), ("stream", ctypes.c_int32), ("a", ctypes.c_int64),
                ("b", ctypes.c_int64), ("c", ctypes.c_int64), ("d", ctypes.c_int64)]


_P = ctypes.c_void_p
_I64P = ctypes.POINTER(ctypes.c_int64)
_sig = {
    "tile_domain_create": ([_I64P, _I64P, ctypes.c_int32, ctypes.POINTER(TileOptions), ctypes.POINTER(_P)], ctypes.c_int),
    "tile_load": ([_P, _P], ctypes.c_int),
    "tile_host_tile": ([_P, ctypes.c_int64, ctypes.POINTER(_P)], ctypes.c_int),
    "tile_mark_host_dirty": ([_P], ctypes.c_int),
    "tile_host_region": ([_P, ctypes.c_int64, ctypes.c_int32, ctypes.POINTER(_P)], ctypes.c_int),
    "tile_host_ghosts": ([_P, ctypes.c_int64, _P, ctypes.c_int64], ctypes.c_int),
    "tile_host_compute": ([_P, _I64P, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32, _P, _P], ctypes.c_int),
    "tile_run": ([_P, ctypes.POINTER(TileKernel), ctypes.c_int32, ctypes.c_int32], ctypes.c_int),
    "tile_sync": ([_P], ctypes.c_int),
    "tile_store": ([_P, _P], ctypes.c_int),
    "tile_invalidate": ([_P], ctypes.c_int),
    "tile_ghost_map": ([_P, ctypes.c_int64, _I64P, ctypes.c_int64], ctypes.c_int),
    "tile_face_sources": ([_P, ctypes.c_int64, _I64P], ctypes.c_int),
    "tile_get_info": ([_P, ctypes.POINTER(TileInfo)], ctypes.c_int),
    "tile_get_stats": ([_P, ctypes.POINTER(TileStats)], ctypes.c_int),
    "tile_reset_stats": ([_P], ctypes.c_int),
    "tile_set_measure": ([_P, ctypes.c_int32], ctypes.c_int),
    "tile_timer_start": ([_P], ctypes.c_int),
    "tile_timer_stop": ([_P, ctypes.POINTER(ctypes.c_double)], ctypes.c_int),
    "tile_set_kernel_timing": ([_P, ctypes.c_int32], ctypes.c_int),
    "tile_trace": ([_P, ctypes.POINTER(TileOp), ctypes.c_int64, _I64P], ctypes.c_int),
    "tile_trace_clear": ([_P], ctypes.c_int),
    "tile_free": ([_P], ctypes.c_int),
    "tile_last_error": ([], ctypes.c_char_p),
    "tile_nccl_unique_id": ([_P], ctypes.c_int),
    "tile_peer_handle": ([_P, _P], ctypes.c_int),
    "tile_peer_connect": ([_P, _P, ctypes.c_int32], ctypes.c_int),
    "tile_local_group_create": ([ctypes.c_int32, ctypes.POINTER(_P)], ctypes.c_int),
    "tile_local_group_free": ([_P], ctypes.c_int),
    "tile_version": ([], ctypes.c_char_p),
    "tile_user_fn_create": ([ctypes.c_char_p, ctypes.c_char_p, ctypes.POINTER(_P)], ctypes.c_int),
    "tile_user_fn_free": ([_P], ctypes.c_int),
    "tile_user_stencil_create": ([ctypes.c_char_p, ctypes.c_char_p, ctypes.POINTER(_P)], ctypes.c_int),
}
EXPORTED = tuple(_sig)
# tile_host_fn(ctx, tile_id, tile, shell, tile_dims, origin, ghost)
HOST_FN = ctypes.CFUNCTYPE(None, _P, ctypes.c_int64, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double),
                           _I64P, _I64P, ctypes.c_int32)
for _name, (_args, _res) in _sig.items():
    _f = getattr(_lib, _name)
    _f.argtypes = _args
    _f.restype = _res
    globals()[_name] = _f


class TileError(RuntimeError):
    def __init__(self, code, where):
        self.code = code
        msg = tile_last_error().decode()
        super().__init__(f"{where}: {STATUS_NAMES.get(code, code)}: {msg}")


def _check(code, where):
    if code != TILE_OK:
        raise TileError(code, where)


def nccl_unique_id():
    buf = ctypes.create_string_buffer(128)
    _check(tile_nccl_unique_id(buf), "tile_nccl_unique_id")
    return buf.raw


class LocalGroup:
    """In-process multi-rank transport (tile_local_group_create): one domain
    per rank, each driven by its own thread, ranks may share one GPU."""

    def __init__(self, nranks):
        h = ctypes.c_void_p()
        _check(tile_local_group_create(nranks, ctypes.byref(h)), "tile_local_group_create")
        self.handle = h
        self.nranks = nranks

    def free(self):
        if self.handle is not None:
            tile_local_group_free(self.handle)
            self.handle = None


def heat7(alpha=0.125):
    """Heat kernel descriptor (reading R1)."""
    return TileKernel(TILE_KERNEL_HEAT7, alpha, 0)


def sincos(inner_iters=32):
    """Compute-intensive kernel descriptor."""
    return TileKernel(TILE_KERNEL_SINCOS, 0.0, inner_iters)


class UserFn:
    """A user pointwise function compiled by libtiles (tile_user_fn_create):
    `source` defines ``__device__ double <name>(double u, long long gidx)``."""

    def __init__(self, source, name, stencil=False):
        h = ctypes.c_void_p()
        create = tile_user_stencil_create if stencil else tile_user_fn_create
        _check(create(source.encode(), name.encode(), ctypes.byref(h)), create.__name__)
        self._h = h
        self.stencil = stencil

    def free(self):
        if self._h is not None:
            tile_user_fn_free(self._h)
            self._h = None

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass


def user_stencil(fn):
    """Kernel descriptor of a user 7-point stencil (UserFn(..., stencil=True))."""
    k = TileKernel(TILE_KERNEL_USER_STENCIL, 0.0, 0)
    k.user = fn._h.value
    k._fn = fn
    return k


def user(fn, inner_iters=1, box=None):
    """Kernel descriptor applying UserFn `fn` inner_iters times per step;
    box = ((x0, y0, z0), (x1, y1, z1)) restricts it to global cells
    x0 <= x < x1 etc. (ranged compute)."""
    k = TileKernel(TILE_KERNEL_USER, 0.0, inner_iters)
    k.user = fn._h.value
    k._fn = fn  # keep the function alive as long as the descriptor
    if box is not None:
        k._box = (ctypes.c_int64 * 6)(*[int(v) for v in tuple(box[0]) + tuple(box[1])])
        k.box = ctypes.cast(k._box, ctypes.POINTER(ctypes.c_int64))
    return k


class Domain:
    """Tiled domain (tile_domain_create ... tile_free). dims and tile_dims are
    (nx, ny, nz); arrays are NumPy float64 in [z][y][x] order."""

    def __init__(self, dims, tile_dims, ghost=1, bc="periodic", device=-1, device_budget_bytes=0,
                 sched="auto", nranks=1, rank=0, nccl_id=None, dry_run=False,
                 fuse_pointwise_steps=True, device_pool=None, streams=None, local_group=None,
                 pageable_host=False, two_step=0, stream_through=0, peer_transport=False, wavefront=0,
                 sweep_link_ratio=0.0):
        self._h = None
        self._inflight = []  # kernel descriptors (user functions) of unsynchronised runs
        self.dims = tuple(int(v) for v in dims)
        self.tile_dims = tuple(int(v) for v in tile_dims)
        self.bc = BCS[bc] if isinstance(bc, str) else int(bc)
        o = TileOptions()
        o.device = device
        o.bc = self.bc
        o.device_budget_bytes = int(device_budget_bytes)
        self._pool = device_pool  # keep the borrowed (torch) pool alive
        if device_pool is not None:
            o.device_pool = ctypes.c_void_p(device_pool.data_ptr())
            o.device_pool_bytes = device_pool.numel() * device_pool.element_size()
        self._streams = None
        if streams:
            arr = (ctypes.c_void_p * len(streams))(*[s.cuda_stream if hasattr(s, "cuda_stream") else s
                                                     for s in streams])
            self._streams = (streams, arr)
            o.streams = ctypes.cast(arr, ctypes.POINTER(ctypes.c_void_p))
            o.nstreams_provided = len(streams)
        o.nranks, o.rank = nranks, rank
        self._nccl_id = None
        if nccl_id is not None:
            self._nccl_id = ctypes.create_string_buffer(bytes(nccl_id), 128)
            o.nccl_unique_id = ctypes.cast(self._nccl_id, ctypes.c_void_p)
        o.sched = SCHEDS[sched] if isinstance(sched, str) else int(sched)
        o.dry_run = 1 if dry_run else 0
        o.fuse_pointwise_steps = 1 if fuse_pointwise_steps else 0
        o.pageable_host = 1 if pageable_host else 0
        o.two_step = int(two_step)
        o.stream_through = int(stream_through)
        o.wavefront = int(wavefront)
        o.sweep_link_ratio = float(sweep_link_ratio)
        o.peer_transport = int(peer_transport)  # True/1: copy pushes; 2: fused kernel pushes
        self._group = local_group
        if local_group is not None:
            o.local_group = local_group.handle
        d = (ctypes.c_int64 * 3)(*self.dims)
        t = (ctypes.c_int64 * 3)(*self.tile_dims)
        h = ctypes.c_void_p()
        _check(tile_domain_create(d, t, ghost, ctypes.byref(o), ctypes.byref(h)), "tile_domain_create")
        self._h = h
        self.info = self.get_info()

    # -- lifecycle --------------------------------------------------------
    def free(self):
        if self._h is not None:
            h, self._h = self._h, None
            _check(tile_free(h), "tile_free")
            self._inflight.clear()

    def __del__(self):
        try:
            self.free()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.free()

    # -- data -------------------------------------------------------------
    def _shape(self):
        nx, ny, nz = self.info["local_dims"]
        h = 2 if self.bc == TILE_BC_DIRICHLET else 0
        return (nz + h, ny + h, nx + h)

    def load(self, arr):
        a = np.ascontiguousarray(arr, dtype=np.float64)
        if a.shape != self._shape():
            raise ValueError(f"expected shape {self._shape()}, got {a.shape}")
        _check(tile_load(self._h, a.ctypes.data), "tile_load")
        self._inflight.clear()

    def store(self, out=None):
        if out is None:
            out = np.zeros(self._shape(), dtype=np.float64)
        if out.shape != self._shape() or out.dtype != np.float64 or not out.flags.c_contiguous:
            raise ValueError("bad output array")
        _check(tile_store(self._h, out.ctypes.data), "tile_store")
        self._inflight.clear()
        return out

    def host_tile(self, tile_id):
        """Writable NumPy view of a tile in the pinned host store."""
        p = ctypes.c_void_p()
        _check(tile_host_tile(self._h, tile_id, ctypes.byref(p)), "tile_host_tile")
        tx, ty, tz = self.tile_dims
        buf = (ctypes.c_double * (tx * ty * tz)).from_address(p.value)
        return np.frombuffer(buf, dtype=np.float64).reshape(tz, ty, tx)

    def mark_host_dirty(self):
        _check(tile_mark_host_dirty(self._h), "tile_mark_host_dirty")

    # -- execution --------------------------------------------------------
    def host_region(self, tile_id, write=False):
        """GPU-disabled request of one region: the tile's current data
        as a writable NumPy view of the pinned store; write=True drops the
        device copy (CPU code will change it)."""
        p = ctypes.c_void_p()
        _check(tile_host_region(self._h, tile_id, 1 if write else 0, ctypes.byref(p)), "tile_host_region")
        tx, ty, tz = self.tile_dims
        buf = (ctypes.c_double * (tx * ty * tz)).from_address(p.value)
        return np.frombuffer(buf, dtype=np.float64).reshape(tz, ty, tx)

    def host_ghosts(self, tile_id):
        """Tile with its ghost shell gathered on the host (P:L96 host update)."""
        g = self.info["ghost"]
        tx, ty, tz = self.tile_dims
        out = np.empty((tz + 2 * g, ty + 2 * g, tx + 2 * g))
        _check(tile_host_ghosts(self._h, tile_id, out.ctypes.data, out.size), "tile_host_ghosts")
        return out

    def host_compute(self, fn, tiles=None, write=False, ghosted=False):
        """GPU-disabled iteration (P:L92 compute(tile, lambda) on the CPU;
        P:L90): calls fn(tile_id, tile, shell, origin) for each tile
        (default: all) with `tile` a NumPy view (tz, ty, tx) of the tile in the
        pinned host store (writable with write=True) and `shell` the tile plus
        its ghost shell gathered on the host before the first call
        (ghosted=True; else None). fn is the caller's CPU code: the library
        itself only moves data."""
        err = []

        def tramp(_ctx, tid, tp, sp, dims, origin, g):
            try:
                tx, ty, tz = dims[0], dims[1], dims[2]
                tile = np.ctypeslib.as_array(tp, shape=(tz, ty, tx))
                if not write:
                    tile = tile.view()
                    tile.flags.writeable = False
                shell = None
                if sp:
                    shell = np.ctypeslib.as_array(sp, shape=(tz + 2 * g, ty + 2 * g, tx + 2 * g)).view()
                    shell.flags.writeable = False
                fn(tid, tile, shell, (origin[0], origin[1], origin[2]))
            except BaseException as e:  # noqa: BLE001  (re-raised after the C call returns)
                if not err:
                    err.append(e)

        cb = HOST_FN(tramp)
        ids = None if tiles is None else np.ascontiguousarray(tiles, dtype=np.int64)
        n = 0 if ids is None else ids.size
        ptr = None if ids is None else ids.ctypes.data_as(_I64P)
        _check(tile_host_compute(self._h, ptr, n, 1 if write else 0, 1 if ghosted else 0,
                                 ctypes.cast(cb, _P), None), "tile_host_compute")
        if err:
            raise err[0]

    def run(self, kernel, steps, nstreams=4):
        _check(tile_run(self._h, ctypes.byref(kernel), steps, nstreams), "tile_run")
        # a user function's module must outlive the launches queued with it
        # (tiles.h: free it only after tile_sync): keep the descriptor until
        # the next call that synchronises
        if getattr(kernel, "_fn", None) is not None:
            self._inflight.append(kernel)

    def sync(self):
        _check(tile_sync(self._h), "tile_sync")
        self._inflight.clear()

    def invalidate(self):
        _check(tile_invalidate(self._h), "tile_invalidate")
        self._inflight.clear()

    def set_measure(self, mode):
        _check(tile_set_measure(self._h, mode), "tile_set_measure")

    def timer_start(self):
        _check(tile_timer_start(self._h), "tile_timer_start")

    def timer_stop(self):
        ms = ctypes.c_double()
        _check(tile_timer_stop(self._h, ctypes.byref(ms)), "tile_timer_stop")
        return ms.value

    def set_kernel_timing(self, on=True):
        _check(tile_set_kernel_timing(self._h, 1 if on else 0), "tile_set_kernel_timing")

    # -- introspection ----------------------------------------------------
    def ghost_map(self, tile_id):
        tx, ty, tz = self.tile_dims
        g = self.info["ghost"]
        out = np.empty((tz + 2 * g, ty + 2 * g, tx + 2 * g), dtype=np.int64)
        _check(tile_ghost_map(self._h, tile_id, out.ctypes.data_as(_I64P), out.size), "tile_ghost_map")
        return out

    def face_sources(self, tile_id):
        out = np.empty(12, dtype=np.int64)
        _check(tile_face_sources(self._h, tile_id, out.ctypes.data_as(_I64P)), "tile_face_sources")
        return out.reshape(6, 2)

    def get_info(self):
        i = TileInfo()
        _check(tile_get_info(self._h, ctypes.byref(i)), "tile_get_info")
        return i.as_dict()

    def stats(self):
        s = TileStats()
        _check(tile_get_stats(self._h, ctypes.byref(s)), "tile_get_stats")
        return s.as_dict()

    def reset_stats(self):
        _check(tile_reset_stats(self._h), "tile_reset_stats")

    def peer_handle(self):
        """64-byte CUDA IPC handle of this rank's halo window (peer transport)."""
        buf = ctypes.create_string_buffer(64)
        _check(tile_peer_handle(self._h, buf), "tile_peer_handle")
        return buf.raw

    def peer_connect(self, handles):
        """Map the z-neighbours' windows; `handles` = every rank's peer_handle()
        in rank order."""
        blob = b"".join(bytes(h) for h in handles)
        buf = ctypes.create_string_buffer(blob, len(blob))
        _check(tile_peer_connect(self._h, buf, len(handles)), "tile_peer_connect")

    def trace(self):
        n = ctypes.c_int64()
        _check(tile_trace(self._h, None, 0, ctypes.byref(n)), "tile_trace")
        buf = (TileOp * max(1, n.value))()
        _check(tile_trace(self._h, buf, n.value, ctypes.byref(n)), "tile_trace")
        return [(OP_NAMES[o.kind], o.stream, o.a, o.b, o.c, o.d) for o in buf[:n.value]]

    def clear_trace(self):
        _check(tile_trace_clear(self._h), "tile_trace_clear")
