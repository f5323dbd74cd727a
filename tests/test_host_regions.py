"""The paper's CPU side of the uniform API (CPU half):
a GPU-disabled request of one region (§IV.B.4: the region is copied
back if its newest data is on the device, then the host pointer is returned,
P:L86) and the host-side ghost update (§III, §IV.B.6: ghost cells
of a region on the host are filled on the host). CPU tests use dry runs (the
host logic and the op trace); GPU tests check the data against the oracle."""
import numpy as np
import pytest

import oracle
import synth
from tests.conftest import cuda_available, import_tiles
from tests.test_schedule import _budget_for

T = import_tiles()
ALPHA = 0.125


def _gather(u, m):
    flat = u.ravel()
    out = np.full(m.shape, np.nan)
    ok = m >= 0
    out[ok] = flat[m[ok]]
    return out


@pytest.mark.parametrize("dims,td,g", [((16, 8, 12), (8, 4, 4), 1), ((12, 8, 8), (4, 4, 4), 2)])
def test_host_ghosts_equal_the_ghost_map_gather_dry(dims, td, g):
    u = synth.uniform_grid(*dims, 21)
    d = T.Domain(dims, td, ghost=g, dry_run=True)
    d.load(u)
    for k in range(d.info["ntiles"]):
        m = oracle.ghost_map(dims, td, g, k)
        assert np.array_equal(d.host_ghosts(k), _gather(u, m))


def test_host_ghosts_dirichlet_faces_dry():
    dims, td = (16, 8, 8), (8, 4, 4)
    ext = synth.uniform_grid(18, 10, 10, 3)
    d = T.Domain(dims, td, bc="dirichlet", dry_run=True)
    d.load(ext)
    for k in range(d.info["ntiles"]):
        got = d.host_ghosts(k)
        ix, iy, iz = k % 2, (k // 2) % 2, k // 4
        exp = ext[iz * 4:iz * 4 + 6, iy * 4:iy * 4 + 6, ix * 8:ix * 8 + 10].copy()
        # shell cells outside the domain in two or three axes are not stored
        zz, yy, xx = np.meshgrid(np.arange(6) + iz * 4 - 1, np.arange(6) + iy * 4 - 1, np.arange(10) + ix * 8 - 1,
                                 indexing="ij")
        outside = (xx < 0) | (xx >= 16)
        nout = outside.astype(int) + ((yy < 0) | (yy >= 8)).astype(int) + ((zz < 0) | (zz >= 8)).astype(int)
        exp[nout >= 2] = np.nan
        assert np.array_equal(got, exp, equal_nan=True), k


def test_host_region_read_copies_back_only_that_tile_dry():
    """Resident dry run: a READ of one device-newer tile issues one D2H of
    that tile and a host sync; the device copy stays (the next run is
    resident, no H2D)."""
    dims, td = (16, 16, 16), (8, 8, 8)
    d = T.Domain(dims, td, dry_run=True, wavefront=-1, stream_through=-1)
    d.load(np.zeros((16, 16, 16)))
    d.run(T.heat7(ALPHA), 2, 2)
    d.clear_trace()
    d.host_region(5)
    ops = [(op[0], op[2]) for op in d.trace() if op[0] in ("d2h", "sync", "h2d")]
    assert ops == [("d2h", 5), ("sync", 0)]
    d.clear_trace()
    d.run(T.heat7(ALPHA), 1, 2)
    assert not [op for op in d.trace() if op[0] == "h2d"]


def test_host_region_write_drops_the_device_copy_dry():
    """WRITE: stream mode frees the tile's slot (its next visit is a miss with
    an H2D); resident mode writes every device-newer tile back and the next
    run re-uploads the domain."""
    dims, td = (16, 16, 16), (8, 8, 4)
    b = _budget_for(dims, td, 20, sched="stream", stream_through=-1)
    d = T.Domain(dims, td, dry_run=True, sched="stream", device_budget_bytes=b, stream_through=-1)
    d.load(np.zeros((16, 16, 16)))
    d.run(T.heat7(ALPHA), 1, 2)
    d.sync()
    d.host_region(15, write=True)
    d.clear_trace()
    d.run(T.heat7(ALPHA), 1, 2)
    h2d = {op[2] for op in d.trace() if op[0] == "h2d"}
    assert 15 in h2d
    r = T.Domain(dims, td, dry_run=True, wavefront=-1, stream_through=-1)
    r.load(np.zeros((16, 16, 16)))
    r.run(T.heat7(ALPHA), 2, 2)
    r.host_region(3, write=True)
    assert not r.get_info()["resident"]
    r.clear_trace()
    r.run(T.heat7(ALPHA), 1, 2)
    assert sum(op[4] for op in r.trace() if op[0] == "h2d") == r.info["ntiles"]


@pytest.mark.gpu
@pytest.mark.parametrize("sched", ["resident", "stream"])
def test_host_region_and_ghosts_gpu(sched):
    """After device runs, one region read on the host equals the oracle's
    tile (no full tile_sync), its host ghost shell equals the oracle grid's
    shell, and a region changed on the host (WRITE) is what the next device
    steps start from."""
    if not cuda_available():
        pytest.skip("no CUDA device")
    dims, td = (64, 32, 48), (32, 16, 16)
    u = synth.uniform_grid(*dims, 42)
    kw = {"stream_through": -1}
    if sched == "stream":
        kw.update(sched="stream", device_budget_bytes=_budget_for(dims, td, 5, sched="stream", stream_through=-1))
    with T.Domain(dims, td, **kw) as d:
        d.load(u)
        d.run(T.heat7(ALPHA), 3, 2)
        ref = oracle.heat_c(u, ALPHA, 3)
        k = 7
        ix, iy, iz = k % 2, (k // 2) % 2, k // 4
        sl = np.s_[iz * 16:(iz + 1) * 16, iy * 16:(iy + 1) * 16, ix * 32:(ix + 1) * 32]
        assert np.array_equal(d.host_region(k), ref[sl])
        assert np.array_equal(d.host_ghosts(k), _gather(ref, oracle.ghost_map(dims, td, 1, k)))
        v = d.host_region(k, write=True)
        v[:] = 0.25                      # CPU code changes the region
        mod = ref.copy()
        mod[sl] = 0.25
        d.run(T.heat7(ALPHA), 2, 2)
        out = d.store()
    assert np.array_equal(out, oracle.heat_c(mod, ALPHA, 2))


def _cpu_heat_step(alpha):
    """The caller's CPU code (the paper's lambda in a GPU-disabled iteration,
    P:L92): one 7-point Jacobi update of a tile from its host shell, written
    in place, in the oracle's order of operations (heat_np)."""
    def fn(tid, tile, shell, origin):
        g = (shell.shape[0] - tile.shape[0]) // 2
        c = shell[g:-g, g:-g, g:-g]
        xm, xp = shell[g:-g, g:-g, g - 1:-g - 1], shell[g:-g, g:-g, g + 1:shell.shape[2] - g + 1]
        ym, yp = shell[g:-g, g - 1:-g - 1, g:-g], shell[g:-g, g + 1:shell.shape[1] - g + 1, g:-g]
        zm, zp = shell[g - 1:-g - 1, g:-g, g:-g], shell[g + 1:shell.shape[0] - g + 1, g:-g, g:-g]
        s = ((xm + xp) + (ym + yp)) + (zm + zp)
        tile[:] = c + alpha * (s - 6.0 * c)
    return fn


@pytest.mark.parametrize("dims,td,g", [((16, 8, 12), (8, 4, 4), 1), ((12, 8, 8), (4, 4, 4), 2)])
def test_host_compute_jacobi_step_equals_the_oracle_dry(dims, td, g):
    """GPU-disabled iteration over every tile with ghosted shells: the shells
    are gathered before the first call, so a CPU update written in place
    still reads only old values — the result is the oracle's heat step
    (P:L92 compute on the CPU, P:L96 host ghost update)."""
    u = synth.uniform_grid(*dims, 5)
    d = T.Domain(dims, td, ghost=g, dry_run=True)
    d.load(u)
    d.host_compute(_cpu_heat_step(ALPHA), write=True, ghosted=True)
    assert np.array_equal(d.store(), oracle.heat_c(u, ALPHA, 1))


def test_host_compute_jacobi_step_dirichlet_dry():
    """Dirichlet: the shells carry the fixed boundary faces."""
    dims, td = (16, 8, 8), (8, 4, 4)
    ext = synth.uniform_grid(18, 10, 10, 7)
    d = T.Domain(dims, td, bc="dirichlet", dry_run=True)
    d.load(ext)
    d.host_compute(_cpu_heat_step(ALPHA), write=True, ghosted=True)
    ref = oracle.heat_c(ext, ALPHA, 1, oracle.BC_DIRICHLET)[1:-1, 1:-1, 1:-1]
    assert np.array_equal(d.store()[1:-1, 1:-1, 1:-1], ref)


def test_host_compute_calls_origins_subset_and_read_only_dry():
    dims, td = (16, 8, 12), (8, 4, 4)
    u = synth.uniform_grid(*dims, 6)
    d = T.Domain(dims, td, dry_run=True)
    d.load(u)
    seen = []

    def look(tid, tile, shell, origin):
        x, y, z = origin
        assert np.array_equal(tile, u[z:z + 4, y:y + 4, x:x + 8])
        assert shell is None and not tile.flags.writeable
        seen.append((tid, origin))

    d.host_compute(look, tiles=[5, 2])
    assert [s[0] for s in seen] == [5, 2]
    assert seen[0][1] == (8, 0, 4) and seen[1][1] == (0, 4, 0)

    def add_one(tid, tile, shell, origin):
        tile += 1.0

    d.host_compute(add_one, tiles=[1], write=True)
    exp = u.copy()
    exp[0:4, 0:4, 8:16] += 1.0
    assert np.array_equal(d.store(), exp)


def test_host_compute_read_shells_one_at_a_time_dry():
    """READ with shells: each call sees its tile's ghost-map gather (the shells
    are gathered one at a time: nothing changes between the calls)."""
    dims, td, g = (12, 8, 8), (4, 4, 4), 2
    u = synth.uniform_grid(*dims, 9)
    d = T.Domain(dims, td, ghost=g, dry_run=True)
    d.load(u)
    seen = []

    def check(tid, tile, shell, origin):
        assert np.array_equal(shell, _gather(u, oracle.ghost_map(dims, td, g, tid)), equal_nan=True)
        seen.append(tid)

    d.host_compute(check, ghosted=True)
    assert seen == list(range(d.info["ntiles"]))


def test_host_compute_errors_dry():
    d = T.Domain((16, 8, 12), (8, 4, 4), dry_run=True)
    d.load(np.zeros((12, 8, 16)))
    with pytest.raises(T.TileError) as e:
        d.host_compute(lambda *a: None, tiles=[99])
    assert e.value.code == 1  # TILE_EINVAL
    with pytest.raises(ZeroDivisionError):  # the caller's exception comes back
        d.host_compute(lambda *a: 1 / 0, tiles=[0])
    calls = []
    with pytest.raises(T.TileError):
        d.host_compute(lambda *a: calls.append(a), tiles=[0, -1])
    assert calls == []  # EINVAL has no side effects


@pytest.mark.gpu
@pytest.mark.parametrize("sched", ["resident", "stream"])
@pytest.mark.parametrize("bc", ["periodic", "dirichlet"])
def test_host_compute_interleaved_with_gpu_steps(sched, bc):
    """The uniform API's two sides in one run: T1 steps on the GPU, one step
    by the caller's CPU code in a GPU-disabled iteration (newest data
    brought to the host first; ghosts on the host), T2 more on
    the GPU — bit-exact against the oracle's T1 + 1 + T2 steps."""
    if not cuda_available():
        pytest.skip("no CUDA device")
    dims, td = (64, 32, 48), (32, 16, 16)
    ext = bc == "dirichlet"
    u = synth.uniform_grid(*((66, 34, 50) if ext else dims), 43)
    kw = {"stream_through": -1, "bc": bc}
    if sched == "stream":
        kw.update(sched="stream",
                  device_budget_bytes=_budget_for(dims, td, 5, sched="stream", stream_through=-1, bc=bc))
    with T.Domain(dims, td, **kw) as d:
        d.load(u)
        d.run(T.heat7(ALPHA), 3, 2)
        d.host_compute(_cpu_heat_step(ALPHA), write=True, ghosted=True)
        d.run(T.heat7(ALPHA), 2, 2)
        out = d.store()
    if ext:
        ref = oracle.heat_c(u, ALPHA, 6, oracle.BC_DIRICHLET)[1:-1, 1:-1, 1:-1]
        assert np.array_equal(out[1:-1, 1:-1, 1:-1], ref)
    else:
        assert np.array_equal(out, oracle.heat_c(u, ALPHA, 6))


def test_host_compute_z_slab_rank_shells_dry():
    """z-slab ranks: ghosted host compute of a middle tile layer works (its
    shell is inside the rank's slab: the oracle's step there); an end layer's
    shell lives on another rank — TILE_EINVAL before any call."""
    G, dims, td = 2, (16, 8, 24), (8, 4, 4)
    u = synth.uniform_grid(*dims, 11)
    nzl = dims[2] // G
    d = T.Domain(dims, td, nranks=G, rank=1, dry_run=True)
    d.load(u[nzl:])
    mid = [k for k in range(d.info["ntiles"]) if 0 < k // 4 < nzl // 4 - 1]
    d.host_compute(_cpu_heat_step(ALPHA), tiles=mid, write=True, ghosted=True)
    ref = oracle.heat_c(u, ALPHA, 1)[nzl:]
    got = d.store()
    assert np.array_equal(got[4:8], ref[4:8])          # the middle layer updated
    assert np.array_equal(got[:4], u[nzl:][:4])        # the end layers untouched
    calls = []
    with pytest.raises(T.TileError) as e:
        d.host_compute(lambda *a: calls.append(a), tiles=[0], ghosted=True)
    assert e.value.code == 1 and calls == []
