"""The boundary's error contract (include/tiles.h "Conventions"; SURVEY.md
§8(b)): a CUDA failure returns TILE_ECUDA and poisons the domain — every
later call except tile_free returns TILE_ESTATE —; a failed pinned host
allocation returns TILE_ENOMEM_HOST; a device budget below the minimum slot
count returns TILE_ENOMEM_DEVICE; TILE_EINVAL has no side effects.

Failures are forced with the library's fault hook, TILES_FAULT=<kind>:<n>
(the n-th h2d / d2h / kernel / sync / host_alloc operation of a domain
fails). In a dry run the executor reports TILE_ECUDA itself; on a GPU the
CUDA executor queues an invalid copy, so the error comes back from the CUDA
runtime through the same path as any other CUDA error.
"""
import ctypes

import numpy as np
import pytest

import synth
from tests.conftest import cuda_available, import_tiles
from tests.test_schedule import _budget_for

T = import_tiles()

DIMS, TD = (32, 16, 16), (16, 8, 8)   # 8 tiles


def _every_call_is_estate(d):
    """Each exported call that takes the domain, except tile_free."""
    h = d._h
    arr = np.zeros((16, 16, 32))
    k = T.heat7()
    info, stats = T.TileInfo(), T.TileStats()
    gm = (ctypes.c_int64 * (18 * 10 * 10))()  # also a large-enough double buffer
    fs = (ctypes.c_int64 * 12)()
    p = ctypes.c_void_p()
    ms = ctypes.c_double()
    n = ctypes.c_int64()
    blob = ctypes.create_string_buffer(64)
    called = []
    noop = T.HOST_FN(lambda *a: called.append(a))
    calls = {
        "tile_load": lambda: T.tile_load(h, arr.ctypes.data),
        "tile_host_tile": lambda: T.tile_host_tile(h, 0, ctypes.byref(p)),
        "tile_mark_host_dirty": lambda: T.tile_mark_host_dirty(h),
        "tile_host_region": lambda: T.tile_host_region(h, 0, 0, ctypes.byref(p)),
        "tile_host_ghosts": lambda: T.tile_host_ghosts(h, 0, gm, len(gm)),
        "tile_host_compute": lambda: T.tile_host_compute(h, None, 0, 0, 0, ctypes.cast(noop, T._P), None),
        "tile_run": lambda: T.tile_run(h, ctypes.byref(k), 1, 2),
        "tile_sync": lambda: T.tile_sync(h),
        "tile_store": lambda: T.tile_store(h, arr.ctypes.data),
        "tile_invalidate": lambda: T.tile_invalidate(h),
        "tile_ghost_map": lambda: T.tile_ghost_map(h, 0, gm, len(gm)),
        "tile_face_sources": lambda: T.tile_face_sources(h, 0, fs),
        "tile_get_info": lambda: T.tile_get_info(h, ctypes.byref(info)),
        "tile_get_stats": lambda: T.tile_get_stats(h, ctypes.byref(stats)),
        "tile_reset_stats": lambda: T.tile_reset_stats(h),
        "tile_set_measure": lambda: T.tile_set_measure(h, 0),
        "tile_timer_start": lambda: T.tile_timer_start(h),
        "tile_timer_stop": lambda: T.tile_timer_stop(h, ctypes.byref(ms)),
        "tile_set_kernel_timing": lambda: T.tile_set_kernel_timing(h, 1),
        "tile_trace": lambda: T.tile_trace(h, None, 0, ctypes.byref(n)),
        "tile_trace_clear": lambda: T.tile_trace_clear(h),
        "tile_peer_handle": lambda: T.tile_peer_handle(h, blob),
        "tile_peer_connect": lambda: T.tile_peer_connect(h, blob, 1),
    }
    domain_calls = {name for name, (args, _) in T._sig.items()
                    if args and args[0] is T._P and name.startswith("tile_") and name not in
                    ("tile_free", "tile_local_group_free", "tile_user_fn_free", "tile_nccl_unique_id")}
    assert domain_calls == set(calls), domain_calls ^ set(calls)
    for name, call in calls.items():
        rc = call()
        assert rc == T.TILE_ESTATE, (name, rc)
        assert "poisoned" in T.tile_last_error().decode()
    assert not called  # a poisoned domain calls no host function


def _run_to_fault(d, u):
    """load + two runs + sync; returns (call, status) of the first failure."""
    h = d._h
    k = T.heat7()
    steps = [("tile_load", lambda: T.tile_load(h, u.ctypes.data)),
             ("tile_run", lambda: T.tile_run(h, ctypes.byref(k), 3, 2)),
             ("tile_run", lambda: T.tile_run(h, ctypes.byref(k), 2, 2)),
             ("tile_sync", lambda: T.tile_sync(h))]
    for name, call in steps:
        rc = call()
        if rc != T.TILE_OK:
            return name, rc
    return None, T.TILE_OK


@pytest.mark.parametrize("fault,sched,where", [("h2d:1", "resident", "tile_run"),
                                               ("h2d:5", "stream", "tile_run"),
                                               ("kernel:2", "resident", "tile_run"),
                                               ("kernel:7", "stream", "tile_run"),
                                               ("d2h:1", "resident", "tile_sync"),
                                               ("d2h:3", "stream", "tile_run"),
                                               ("sync:1", "resident", "tile_sync")])
def test_cuda_error_poisons_domain_dry(monkeypatch, fault, sched, where):
    monkeypatch.setenv("TILES_FAULT", fault)
    kw = {"sched": sched, "stream_through": -1, "wavefront": -1}
    if sched == "stream":
        kw["device_budget_bytes"] = _budget_for(DIMS, TD, 4, sched="stream", stream_through=-1)
    d = T.Domain(DIMS, TD, dry_run=True, **kw)
    name, rc = _run_to_fault(d, synth.uniform_grid(*DIMS, 1))
    assert (name, rc) == (where, T.TILE_ECUDA), (name, rc, T.tile_last_error())
    assert "injected" in T.tile_last_error().decode()
    _every_call_is_estate(d)
    h, d._h = d._h, None
    assert T.tile_free(h) == T.TILE_OK


def test_no_fault_without_the_hook_dry(monkeypatch):
    monkeypatch.delenv("TILES_FAULT", raising=False)
    d = T.Domain(DIMS, TD, dry_run=True)
    assert _run_to_fault(d, synth.uniform_grid(*DIMS, 1)) == (None, T.TILE_OK)
    monkeypatch.setenv("TILES_FAULT", "h2d:1000000")   # never reached
    d = T.Domain(DIMS, TD, dry_run=True)
    assert _run_to_fault(d, synth.uniform_grid(*DIMS, 1)) == (None, T.TILE_OK)
    d.free()


def test_host_allocation_failure_dry(monkeypatch):
    monkeypatch.setenv("TILES_FAULT", "host_alloc:1")
    with pytest.raises(T.TileError) as e:
        T.Domain(DIMS, TD, dry_run=True)
    assert e.value.code == T.TILE_ENOMEM_HOST


def test_device_budget_below_minimum_slots_dry():
    for sched in ("auto", "stream"):
        with pytest.raises(T.TileError) as e:
            T.Domain(DIMS, TD, dry_run=True, sched=sched, device_budget_bytes=4096)
        assert e.value.code == T.TILE_ENOMEM_DEVICE
    # the smallest budget that works streams with 2 slots (fewer
    # regions than tiles share device pointers)
    lo, hi = 1, 1 << 36
    while lo < hi:
        mid = (lo + hi) // 2
        try:
            T.Domain(DIMS, TD, dry_run=True, device_budget_bytes=mid)
            hi = mid
        except T.TileError as e:
            assert e.code == T.TILE_ENOMEM_DEVICE
            lo = mid + 1
    d = T.Domain(DIMS, TD, dry_run=True, device_budget_bytes=lo)
    assert d.info["nslots"] == 2 and d.info["sched"] == T.TILE_SCHED_STREAM


@pytest.mark.gpu
@pytest.mark.parametrize("fault,sched,where", [("h2d:1", "resident", "tile_run"),
                                               ("kernel:2", "resident", "tile_run"),
                                               ("d2h:1", "resident", "tile_sync"),
                                               ("sync:1", "resident", "tile_sync"),
                                               ("h2d:5", "stream", "tile_run"),
                                               ("d2h:3", "stream", "tile_run")])
def test_cuda_error_poisons_domain_gpu(monkeypatch, fault, sched, where):
    if not cuda_available():
        pytest.skip("no CUDA device")
    monkeypatch.setenv("TILES_FAULT", fault)
    kw = {"sched": sched, "stream_through": -1, "wavefront": -1, "device": 0}
    if sched == "stream":
        kw["device_budget_bytes"] = _budget_for(DIMS, TD, 4, sched="stream", stream_through=-1)
    d = T.Domain(DIMS, TD, **kw)
    name, rc = _run_to_fault(d, synth.uniform_grid(*DIMS, 1))
    assert (name, rc) == (where, T.TILE_ECUDA), (name, rc, T.tile_last_error())
    assert "cudaMemcpyAsync" in T.tile_last_error().decode()   # the CUDA runtime's own error
    _every_call_is_estate(d)
    h, d._h = d._h, None
    assert T.tile_free(h) == T.TILE_OK
    # the device is still usable by a fresh domain
    monkeypatch.delenv("TILES_FAULT")
    u = synth.uniform_grid(*DIMS, 1)
    with T.Domain(DIMS, TD, device=0) as d2:
        d2.load(u)
        d2.run(T.heat7(), 2, 2)
        assert np.isfinite(d2.store()).all()


@pytest.mark.gpu
def test_pinned_host_allocation_failure_gpu(monkeypatch):
    if not cuda_available():
        pytest.skip("no CUDA device")
    monkeypatch.setenv("TILES_FAULT", "host_alloc:1")
    with pytest.raises(T.TileError) as e:
        T.Domain(DIMS, TD, device=0)
    assert e.value.code == T.TILE_ENOMEM_HOST
    assert "cudaHostAlloc" in str(e.value)


@pytest.mark.gpu
def test_device_budget_below_minimum_gpu():
    if not cuda_available():
        pytest.skip("no CUDA device")
    with pytest.raises(T.TileError) as e:
        T.Domain(DIMS, TD, device=0, device_budget_bytes=4096)
    assert e.value.code == T.TILE_ENOMEM_DEVICE
