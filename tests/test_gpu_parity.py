"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle.

Heat is compared BIT-EXACTLY (the kernels use explicit round-to-nearest
intrinsics in the order of reading R1, like the no-FMA oracle), which is
stricter than the north star's 1e-12 relative max-norm. The compute-intensive
kernel is compared within 1e-12 relative (CUDA libdevice sin/cos vs glibc,
DESIGN.md reading R17) plus its closed form x_T ~ x_0 + K*T.
"""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu

from tests.conftest import import_tiles

T = import_tiles()
T_ = T
ALPHA = 0.125


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.init()


def _heat(dims, td, steps, ns=2, bc="periodic", seed=42, alpha=ALPHA, runs=None, **kw):
    nx, ny, nz = dims
    if bc == "periodic":
        u0 = synth.uniform_grid(nx, ny, nz, seed)
        inp = u0
    else:
        inp = synth.uniform_grid(nx + 2, ny + 2, nz + 2, seed)
    with T.Domain(dims, td, bc=bc, **kw) as d:
        d.load(inp)
        for s in (runs or [steps]):
            d.run(T.heat7(alpha), s, ns)
        out = d.store()
        info, st = d.info, d.stats()
    if bc == "periodic":
        ref = oracle.heat_c(inp, alpha, steps)
    else:
        ref = oracle.heat_c(inp, alpha, steps, oracle.BC_DIRICHLET)[1:-1, 1:-1, 1:-1]
        out = out[1:-1, 1:-1, 1:-1]
    return out, ref, info, st


def test_c1_bit_exact_and_survey_hash(golden_dir):
    import hashlib
    import os
    out, ref, info, st = _heat((64, 64, 64), (32, 32, 32), 10, ns=2)
    assert np.array_equal(out, ref)
    rows = [l.split() for l in open(os.path.join(golden_dir, "c1_survey_values.txt"))
            if l.strip() and not l.startswith("#")]
    sha = [r[4] for r in rows if r[0] == "sha_u10"][0]
    assert hashlib.sha256(out.tobytes()).hexdigest() == sha
    assert info["sched"] == T.TILE_SCHED_RESIDENT and st["n_kernels"] > 0


@pytest.mark.parametrize("dims,td", [((64, 32, 48), (32, 16, 16)), ((128, 64, 32), (64, 32, 8)),
                                     ((32, 32, 32), (32, 32, 32)), ((48, 40, 20), (24, 20, 5)),
                                     ((256, 32, 16), (128, 16, 16)), ((64, 64, 64), (16, 64, 64)),
                                     ((512, 8, 8), (512, 8, 8))])
def test_tile_shapes_bit_exact(dims, td):
    out, ref, _, _ = _heat(dims, td, 7, ns=3)
    assert np.array_equal(out, ref)


@pytest.mark.parametrize("ns", [1, 2, 4, 8])
def test_stream_counts_bit_exact(ns):
    out, ref, _, _ = _heat((64, 64, 64), (32, 16, 16), 6, ns=ns)
    assert np.array_equal(out, ref)


@pytest.mark.parametrize("dims,td,steps,ns", [((8, 8, 8), (2, 2, 2), 4, 2),        # 64 tiny tiles, generic kernel
                                              ((16, 8, 9), (8, 4, 3), 5, 3),      # odd tile depth
                                              ((64, 64, 64), (32, 16, 16), 6, 64), # the maximum stream count
                                              ((16, 16, 8), (16, 16, 8), 3, 1),   # one tile, wraps onto itself
                                              ((32, 16, 256), (32, 16, 8), 4, 4)]) # 32 thin layers
def test_edge_shapes_and_counts(dims, td, steps, ns):
    """Degenerate decompositions: tiles of 2 cells per axis, odd depths, a
    single tile whose ghosts are its own faces, many thin layers, 64 streams."""
    out, ref, _, _ = _heat(dims, td, steps, ns=ns)
    assert np.array_equal(out, ref)


def test_zero_work_runs_are_identity():
    """tile_run with 0 steps, and SINCOS with 0 inner iterations, change nothing."""
    nx, ny, nz = 64, 32, 32
    u0 = synth.uniform_grid(nx, ny, nz, 3)
    with T.Domain((nx, ny, nz), (32, 16, 16)) as d:
        d.load(u0)
        d.run(T.heat7(ALPHA), 0, 2)
        assert np.array_equal(d.store(), u0)
        d.run(T.sincos(0), 3, 2)
        assert np.array_equal(d.store(), u0)
    with T.Domain((nx, ny, nz), (32, 16, 16), sched="stream", device_budget_bytes=_budget((nx, ny, nz), (32, 16, 16), 3)) as d:
        d.load(u0)
        d.run(T.heat7(ALPHA), 0, 2)
        assert np.array_equal(d.store(), u0)


def test_runs_continue_state():
    out, ref, _, _ = _heat((64, 64, 64), (32, 32, 16), 9, runs=[4, 1, 0, 4])
    assert np.array_equal(out, ref)


@pytest.mark.parametrize("direct,persist", [("1", "1"), ("1", "0"), ("0", "0")])
@pytest.mark.parametrize("bc", ["periodic", "dirichlet"])
@pytest.mark.parametrize("dims,td", [((128, 64, 64), (64, 32, 16)), ((64, 96, 48), (32, 32, 8))])
def test_resident_paths_bit_exact(monkeypatch, direct, persist, bc, dims, td):
    """The resident single-step variants give the same bits: direct y/z ghosts
    + persistent multi-step launch (default), direct ghosts with one launch
    per step, and every ghost from exported faces. Several runs, so a run
    starts from the state (and the stale y/z exports) a direct run left."""
    monkeypatch.setenv("TILES_DIRECT", direct)
    monkeypatch.setenv("TILES_PERSIST", persist)
    out, ref, _, st = _heat(dims, td, 13, bc=bc, runs=[3, 6, 1, 3])
    assert np.array_equal(out, ref), np.abs(out - ref).max()


def test_sync_baseline_bit_exact():
    out, ref, info, _ = _heat((64, 64, 64), (32, 32, 32), 5, sched="sync")
    assert np.array_equal(out, ref) and info["sched"] == T.TILE_SCHED_SYNC


@pytest.mark.parametrize("alpha", [0.1, 1.0 / 6.0])
def test_other_alphas(alpha):
    out, ref, _, _ = _heat((64, 32, 32), (32, 16, 16), 5, alpha=alpha)
    assert np.array_equal(out, ref)


def test_dirichlet_random_and_linear():
    out, ref, _, _ = _heat((64, 32, 32), (32, 16, 16), 6, bc="dirichlet", seed=5)
    assert np.array_equal(out, ref)
    ue = synth.linear_grid(32, 32, 32, g=1)
    with T.Domain((32, 32, 32), (16, 16, 16), bc="dirichlet") as d:
        d.load(ue)
        d.run(T.heat7(), 5, 2)
        out = d.store()
    assert np.array_equal(out[1:-1, 1:-1, 1:-1], ue[1:-1, 1:-1, 1:-1])


def test_sine_mode_decay():
    import math
    n = 64
    u = synth.sine_grid(n, n, n)
    with T.Domain((n, n, n), (32, 32, 32)) as d:
        d.load(u)
        d.run(T.heat7(), 10, 2)
        out = d.store()
    lam = 1 - 6 * ALPHA * (1 - math.cos(2 * math.pi / n))
    assert np.abs(out - lam ** 10 * u).max() / np.abs(u).max() <= 1e-12


def _budget(dims, td, nslots, bc="periodic"):
    # the same plan in dry-run tells the persistent bytes; add nslots tiles
    lo, hi = 1, 1 << 40
    while lo < hi:
        mid = (lo + hi) // 2
        try:
            n = T.Domain(dims, td, dry_run=True, sched="stream", bc=bc,
                         device_budget_bytes=mid).info["nslots"]
        except T.TileError:
            n = -1
        lo, hi = (lo, mid) if n >= nslots else (mid + 1, hi)
    return lo


@pytest.mark.parametrize("nslots,ns", [(2, 1), (3, 2), (6, 4), (17, 3)])
def test_out_of_core_capped_bit_exact(nslots, ns):
    dims, td = (64, 64, 64), (32, 16, 16)   # 32 tiles
    b = _budget(dims, td, nslots)
    out, ref, info, st = _heat(dims, td, 5, ns=ns, sched="stream", device_budget_bytes=b, runs=[3, 2])
    assert info["sched"] == T.TILE_SCHED_STREAM and info["nslots"] == nslots
    assert np.array_equal(out, ref)
    assert st["misses"] > 0 and st["writebacks"] > 0


@pytest.mark.parametrize("dims,td,nslots,runs", [((64, 64, 256), (32, 32, 32), 30, [5, 3]),
                                                 ((64, 64, 256), (32, 32, 32), 30, [13]),
                                                 ((64, 32, 192), (32, 32, 16), 20, [40]),
                                                 ((128, 64, 128), (64, 64, 8), 40, [6, 1, 2])])
def test_out_of_core_stream_through_bit_exact(dims, td, nslots, runs):
    """Out-of-core heat with temporal blocking: passes of k steps over units
    of planes (ring of input units, fused first/last sweeps), one H2D and one
    D2H per cell per pass; bit-identical to the oracle; a following per-step
    run (stream_through off) continues from the host data."""
    b = _budget(dims, td, nslots)
    out, ref, info, st = _heat(dims, td, sum(runs), ns=3, sched="stream", device_budget_bytes=b, runs=runs)
    assert info["sched"] == T.TILE_SCHED_STREAM and info["nslots"] == nslots
    assert np.array_equal(out, ref)
    cells = dims[0] * dims[1] * dims[2]
    assert st["bytes_h2d"] < sum(runs) * cells * 8   # fewer link passes than steps
    nx, ny, nz = dims
    u0 = synth.uniform_grid(nx, ny, nz, 42)
    with T.Domain(dims, td, sched="stream", device_budget_bytes=b) as d:
        d.load(u0)
        d.run(T.heat7(ALPHA), 4, 2)                       # stream-through pass(es)
        d.run(T.heat7(ALPHA), 1, 2)                       # per-step (T = 1)
        d.run(T.sincos(2), 1, 2)                          # pointwise after it
        out2 = d.store()
    assert np.allclose(out2, oracle.sincos_c(oracle.heat_c(u0, ALPHA, 5), 2, 1), rtol=1e-12, atol=0)


def test_out_of_core_dirichlet():
    dims, td = (64, 32, 32), (32, 16, 16)
    b = _budget(dims, td, 4, bc="dirichlet")
    out, ref, _, _ = _heat(dims, td, 4, bc="dirichlet", sched="stream", device_budget_bytes=b)
    assert np.array_equal(out, ref)


def test_invalidate_restreams_from_host():
    u0 = synth.uniform_grid(64, 64, 64, 42)
    with T.Domain((64, 64, 64), (32, 32, 32)) as d:
        d.load(u0)
        d.run(T.heat7(), 3, 2)
        d.sync()
        d.invalidate()
        d.reset_stats()
        d.run(T.heat7(), 2, 2)
        out = d.store()
        st = d.stats()
    assert np.array_equal(out, oracle.heat_c(u0, ALPHA, 5))
    assert st["bytes_h2d"] == 64 ** 3 * 8 and st["bytes_d2h"] == 64 ** 3 * 8


def test_measure_modes_run():
    u0 = synth.uniform_grid(64, 64, 64, 1)
    with T.Domain((64, 64, 64), (32, 32, 32)) as d:
        d.load(u0)
        for m in (T.TILE_MEASURE_XFER_ONLY, T.TILE_MEASURE_COMP_ONLY, T.TILE_MEASURE_NORMAL):
            d.set_measure(m)
            d.invalidate()
            d.run(T.heat7(), 2, 2)
            d.sync()


def test_kernel_timing_and_device_timer():
    u0 = synth.uniform_grid(128, 128, 128, 1)
    with T.Domain((128, 128, 128), (64, 64, 64)) as d:
        d.load(u0)
        d.run(T.heat7(), 1, 1)
        d.sync()
        d.set_kernel_timing(True)
        d.reset_stats()
        d.timer_start()
        d.run(T.heat7(), 4, 1)
        ms = d.timer_stop()
        st = d.stats()
    # 4 steps: one persistent multi-step launch (default) or 4 launches
    # (TILES_PERSIST=0), plus one face extraction when the first run took a
    # fresh-upload schedule that leaves the faces to the next resident run
    assert st["n_kernels"] in (1, 2, 4, 5) and st["kernel_timed"] == st["n_kernels"]
    assert ms > 0 and 0 < st["kernel_ms"] <= ms * 1.01


# ----------------------------------------------------------- large configs
def test_c2_full_size_cone_samples():
    """C2 (512^3, 8^3 tiles of 64^3, resident, 4 streams) at BASELINE size,
    in the launch configuration bench.py times; sampled blocks vs the cone
    oracle (bit-exact), including tile seams and the periodic corner."""
    n, steps = 512, 10
    u0 = np.empty((n, n, n))
    synth.fill_uniform_native(u0.ctypes.data, n, n, n, 0, n, 0, n, 0, n, 42)
    with T.Domain((n, n, n), (64, 64, 64)) as d:
        d.load(u0)
        del u0
        d.run(T.heat7(), steps, 4)
        out = d.store()
    rng = np.random.default_rng(1234)
    blocks = [(0, 0, 0), (n - 2, n - 2, n - 2), (62, 63, 64), (127, 190, 255), (448, 0, 511)]
    blocks += [tuple(int(v) for v in rng.integers(0, n, 3)) for _ in range(6)]
    for z0, y0, x0 in blocks:
        ref = oracle.cone_block(n, n, n, 42, ALPHA, steps, z0, y0, x0, 2, synth.uniform_block)
        got = out[np.ix_([(z0 + i) % n for i in range(2)], [(y0 + i) % n for i in range(2)],
                         [(x0 + i) % n for i in range(2)])]
        assert np.array_equal(got, ref), (z0, y0, x0)
    # invariant at any size: periodic heat conserves the sum (to rounding)
    assert out.min() >= 0.0 and out.max() <= 1.0


def test_sincos_parity_and_closed_form():
    x0 = synth.uniform_grid(64, 64, 32, 7)
    K, steps = 32, 3
    for sched, fuse in (("auto", True), ("auto", False)):
        with T.Domain((64, 64, 32), (32, 32, 16), sched=sched, fuse_pointwise_steps=fuse) as d:
            d.load(x0)
            d.run(T.sincos(K), steps, 4)
            out = d.store()
        ref = oracle.sincos_c(x0, K, steps)
        assert np.abs(out - ref).max() / np.abs(ref).max() <= 1e-12
        s = x0.copy()
        for _ in range(K * steps):
            s = s + 1.0
        assert np.all(np.abs(out - s) <= 4 * np.spacing(out))


def test_sincos_out_of_core_step_major():
    dims, td = (64, 64, 32), (32, 32, 16)
    b = _budget(dims, td, 3)
    x0 = synth.uniform_grid(*dims, 7)
    with T.Domain(dims, td, sched="stream", device_budget_bytes=b, fuse_pointwise_steps=False) as d:
        d.load(x0)
        d.run(T.sincos(4), 3, 2)
        out = d.store()
        st = d.stats()
    ref = oracle.sincos_c(x0, 4, 3)
    assert np.abs(out - ref).max() / np.abs(ref).max() <= 1e-12
    assert st["misses"] >= 8 * 3 - 2 * 3


def test_torch_pool_and_streams():
    import torch
    u0 = synth.uniform_grid(64, 64, 64, 42)
    pool = torch.empty(64 << 20, dtype=torch.uint8, device="cuda")
    streams = [torch.cuda.Stream() for _ in range(2)]
    with T.Domain((64, 64, 64), (32, 32, 32), device_pool=pool, streams=streams) as d:
        d.load(u0)
        d.run(T.heat7(), 4, 2)
        out = d.store()
    assert np.array_equal(out, oracle.heat_c(u0, ALPHA, 4))


def test_sincos_single_iteration_accuracy_wide_range():
    """One iteration of the listing on arguments spanning small, negative,
    medium and huge (1e9..1e15, multi-word reduction) values, against the
    glibc oracle per cell."""
    rng = np.random.default_rng(3)
    x = np.concatenate([rng.uniform(0, 2000, 1 << 16), rng.uniform(-400, 0, 1 << 14),
                        rng.uniform(1e6, 2e6, 1 << 12), rng.uniform(1e9, 1e15, 1 << 12),
                        np.array([0.0, 1048575.9, 1048576.0, np.pi / 4, np.pi / 2, np.pi, -np.pi / 4])])
    x = np.concatenate([x, np.full((-x.size) % 4096, 0.5)])
    n = x.size
    grid = x.reshape(n // 512, 8, 64)
    with T.Domain((64, 8, n // 512), (64, 8, 8)) as d:
        d.load(grid)
        d.run(T.sincos(1), 1, 1)
        out = d.store().ravel()
    ref = oracle.sincos_c(x, 1, 1)
    # sqrt(s^2+c^2) is 1 within an ulp on both sides, so per cell the
    # results may differ by ulp(1) (absolute) plus the final rounding
    err = np.abs(out - ref)
    assert np.all(err <= np.spacing(1.0) + 2 * np.spacing(np.abs(ref))), x[np.argmax(err)]


def test_pageable_host_baseline_bit_exact():
    out, ref, _, _ = _heat((64, 64, 64), (32, 32, 32), 5, sched="sync", pageable_host=True)
    assert np.array_equal(out, ref)


@pytest.mark.parametrize("bc,td", [("periodic", (32, 16, 16)), ("dirichlet", (32, 16, 8)),
                                   ("periodic", (48, 40, 10)), ("periodic", (64, 64, 16))])
def test_ghost2_faces_bit_exact(bc, td):
    """ghost = 2: faces are exported 2 layers deep."""
    dims = (64 if td[0] != 48 else 96, 64 if td[1] != 40 else 80, 32 if td[2] != 10 else 20)
    out, ref, info, _ = _heat(dims, td, 7, bc=bc, ghost=2, runs=[4, 3])
    assert info["ghost"] == 2
    assert np.array_equal(out, ref)
    b = _budget(dims, td, 3, bc=bc)
    out, ref, _, _ = _heat(dims, td, 5, bc=bc, ghost=2, sched="stream", device_budget_bytes=b * 2)
    assert np.array_equal(out, ref)


@pytest.mark.parametrize("bc,dims,td,runs", [("periodic", (128, 64, 64), (64, 64, 16), [6, 3]),
                                             ("dirichlet", (128, 64, 64), (64, 32, 16), [4, 5]),
                                             ("periodic", (64, 64, 32), (32, 32, 8), [7]),
                                             ("periodic", (256, 64, 16), (128, 16, 8), [4]),
                                             ("dirichlet", (64, 32, 32), (32, 16, 8), [2, 2, 3])])
def test_two_step_passes_bit_exact(bc, dims, td, runs):
    """ghost = 2 runs two Jacobi steps per pass (heat7x2): bit-identical to
    single steps and to the oracle, resident and out-of-core."""
    out, ref, info, st = _heat(dims, td, sum(runs), bc=bc, ghost=2, runs=runs, two_step=1)
    assert np.array_equal(out, ref)
    assert info["steps_per_pass"] == 2
    b = _budget(dims, td, 4, bc=bc)
    out, ref, info, _ = _heat(dims, td, sum(runs), bc=bc, ghost=2, runs=runs, sched="stream",
                              device_budget_bytes=b * 2)
    assert np.array_equal(out, ref) and info["steps_per_pass"] == 2


@pytest.mark.parametrize("dims,td,T", [((128, 64, 256), (64, 32, 32), 5), ((64, 64, 192), (32, 32, 64), 10),
                                       ((64, 64, 256), (64, 64, 32), 1), ((64, 64, 512), (64, 64, 32), 20),
                                       ((64, 32, 1024), (32, 32, 64), 64)])
def test_stream_through_bit_exact(dims, td, T):
    """Fresh-upload runs with T <= tz take the stream-through schedule
    (units of planes, T sweeps reading the resident array first and writing
    packed sub-tiles last, D2H, write-back); the host
    result and the kept device copy (a following resident run) are exact."""
    nx, ny, nz = dims
    u0 = synth.uniform_grid(nx, ny, nz, 42)
    with T_.Domain(dims, td, stream_through=1) as d:   # forced (the default is cost-model driven)
        d.load(u0)
        d.run(T_.heat7(), T, 2)
        out1 = d.store()
        st = d.stats()
        d.run(T_.heat7(), 3, 2)   # continues from the device copy
        out2 = d.store()
    assert np.array_equal(out1, oracle.heat_c(u0, ALPHA, T))
    assert np.array_equal(out2, oracle.heat_c(u0, ALPHA, T + 3))
    assert st["bytes_h2d"] == nx * ny * nz * 8 and st["bytes_d2h"] == nx * ny * nz * 8


@pytest.mark.parametrize("dims,td,T", [((64, 32, 128), (32, 16, 16), 20), ((128, 64, 256), (64, 64, 32), 48),
                                       ((64, 64, 64), (32, 32, 8), 7), ((96, 64, 160), (32, 32, 32), 1),
                                       ((64, 32, 512), (32, 32, 64), 100), ((512, 64, 128), (64, 64, 64), 16),
                                       ((512, 32, 256), (64, 32, 32), 20), ((512, 64, 384), (64, 64, 64), 48),
                                       ((512, 16, 512), (64, 16, 64), 100), ((512, 32, 256), (64, 32, 32), 21),
                                       ((512, 4, 128), (64, 4, 16), 10), ((512, 12, 192), (64, 4, 32), 33)])
@pytest.mark.parametrize("wave", [1, 2, 3])
def test_wavefront_bit_exact(dims, td, T, wave):
    """Fresh-upload runs on the time-skewed wavefront (forced): chunks of
    planes, level s of chunk i on planes [c*i - s, c*i + c - s), the seam's
    bootstrap trapezoid in the scratch layers, each chunk's final planes
    back to the host as soon as it ends; the host result, the kept device
    copy (a following resident run) and a second wavefront run are exact,
    and every cell crossed the link once per direction. wave = 1: the default
    (two levels per pass on grids 512 wide, heat2_band_slab); 2: two levels
    per pass everywhere (slab_sweep2_tile off the band shape); 3: one level
    per pass (slab_sweep_tile)."""
    nx, ny, nz = dims
    u0 = synth.uniform_grid(nx, ny, nz, 42)
    with T_.Domain(dims, td, wavefront=wave) as d:
        d.load(u0)
        d.run(T_.heat7(), T, 2)
        out1 = d.store()
        st = d.stats()
        sched = d.get_info()["last_schedule"]
        d.run(T_.heat7(), 3, 2)   # continues from the device copy
        out2 = d.store()
        d.invalidate()
        d.run(T_.heat7(), T, 4)   # a second fresh upload of u^{T+3}
        out3 = d.store()
    assert sched == 6
    assert np.array_equal(out1, oracle.heat_c(u0, ALPHA, T))
    assert np.array_equal(out2, oracle.heat_c(u0, ALPHA, T + 3))
    assert np.array_equal(out3, oracle.heat_c(u0, ALPHA, 2 * T + 3))
    assert st["bytes_h2d"] == nx * ny * nz * 8 and st["bytes_d2h"] == nx * ny * nz * 8


@pytest.mark.parametrize("dims,td,runs", [((512, 64, 64), (64, 64, 32), [1, 2, 3, 8]),
                                          ((512, 96, 48), (64, 32, 16), [2, 6, 1]),
                                          ((512, 8, 40), (64, 4, 8), [3, 4]),
                                          ((512, 512, 64), (64, 64, 64), [1, 10]),
                                          ((512, 20, 16), (64, 20, 4), [2, 5]),     # one tile row, thin layers
                                          ((512, 12, 6), (64, 4, 3), [4]),          # bands = tile rows, nz = 6
                                          ((512, 40, 9), (64, 8, 9), [1, 6]),       # 5 tile rows, one layer
                                          ((512, 4, 2), (64, 4, 1), [2, 3]),        # one band, nz = 2
                                          ((512, 8, 1), (64, 8, 1), [1, 4])])       # nz = 1 (z neighbours = self)
def test_band2_resident_bit_exact(dims, td, runs):
    """Resident periodic runs 512 cells wide: two steps per kernel over the
    whole grid (heat2_band — full-width bands, 5-D TMA boxes, both levels in
    registers), the odd step on the face-ghost path, bit-exact to the oracle;
    the kernel timing counts one 16-byte pass per cell per two steps."""
    out, ref, info, st = _heat(dims, td, sum(runs), runs=runs)
    assert np.array_equal(out, ref), np.abs(out - ref).max()
    u0 = synth.uniform_grid(*dims, 3)
    with T.Domain(dims, td) as d:
        d.load(u0)
        d.run(T.heat7(), 1, 2)
        d.sync()
        d.set_kernel_timing(True)
        d.reset_stats()
        d.run(T.heat7(), 4, 2)
        d.sync()
        st = d.stats()
        assert d.get_info()["last_schedule"] == 7
        out = d.store()
    assert np.array_equal(out, oracle.heat_c(u0, ALPHA, 5))
    assert st["n_kernels"] == 2 and st["sweep_timed"] == 2
    assert st["sweep_cells"] == 2 * dims[0] * dims[1] * dims[2]


@pytest.mark.parametrize("dims,td,T_", [((512, 64, 256), (64, 64, 32), 10), ((512, 32, 192), (64, 32, 16), 5),
                                         ((512, 4, 128), (64, 4, 16), 7),
                                         ((512, 64, 128), (64, 64, 64), 2), ((512, 128, 256), (64, 64, 64), 13)])
def test_stream_through_two_sweeps_bit_exact(dims, td, T_):
    """Fresh-upload stream-through on grids 512 wide with two_step = 1: two sweeps per kernel
    (heat2_band_slab shrink mode: resident array / dense slabs / packed
    sub-tiles as views), an odd T's last sweep alone; bit-exact, then a
    resident continuation."""
    nx, ny, nz = dims
    u0 = synth.uniform_grid(nx, ny, nz, 8)
    with T.Domain(dims, td, stream_through=1, wavefront=-1, two_step=1) as d:
        d.load(u0)
        d.run(T.heat7(), T_, 3)
        out1 = d.store()
        sched = d.get_info()["last_schedule"]
        d.run(T.heat7(), 2, 2)
        out2 = d.store()
    assert sched == 2
    assert np.array_equal(out1, oracle.heat_c(u0, ALPHA, T_))
    assert np.array_equal(out2, oracle.heat_c(u0, ALPHA, T_ + 2))


def test_wavefront_one_launch_per_iteration_bit_exact():
    """The opt-in one-launch-per-iteration wavefront (heat2_band_iter,
    TILES_WAVE_ITER=1: bands synchronised by progress flags) on the 512-wide
    wavefront parity cases, in a fresh process (the knob is read once)."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    ids = [f"tests/test_gpu_parity.py::test_wavefront_bit_exact[1-dims{k}-td{k}-{t}]"
           for k, t in ((5, 16), (6, 20), (7, 48), (8, 100))]   # the 512-wide cases
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "-p", "no:cacheprovider", *ids],
                       cwd=root, env={**os.environ, "TILES_WAVE_ITER": "1"}, capture_output=True, text=True,
                       timeout=900)
    assert r.returncode == 0, r.stdout[-3000:] + r.stderr[-2000:]
    assert " passed" in r.stdout


@pytest.mark.parametrize("wave", [1, 3])
def test_wavefront_growing_T_on_one_domain_bit_exact(wave):
    """Fresh-upload wavefront runs of growing T on one domain (the Fig. 5
    sweep's pattern): the scratch grows in place between runs and every
    tensor map over it must follow (a stale map read the new part as
    out-of-bounds zeros)."""
    dims, td = (512, 32, 256), (64, 32, 32)
    u0 = synth.uniform_grid(*dims, 31)
    with T.Domain(dims, td, wavefront=wave) as d:
        for T_ in (5, 20, 47, 64):
            d.load(u0)   # the host store holds the previous run's result after store()
            d.run(T.heat7(), T_, 3)
            out = d.store()
            assert d.get_info()["last_schedule"] == 6
            assert np.array_equal(out, oracle.heat_c(u0, ALPHA, T_)), T_


@pytest.mark.parametrize("case", range(40))
def test_band_kernels_random_shapes_bit_exact(case):
    """Seeded random 512-wide shapes and run sequences through the default
    schedules (fresh uploads: stream-through / two-level wavefront / split
    large-T; resident: heat2_band, odd steps on the face-ghost path), every
    stored grid against the oracle, bit-exact."""
    import random
    rng = random.Random(1000 + case)
    ny = rng.choice([4, 8, 12, 16, 24, 32, 64])
    ty = rng.choice([t for t in range(4, ny + 1, 4) if ny % t == 0])
    nz = rng.choice([1, 2, 3, 8, 24, 48, 96, 128, 192])
    tz = rng.choice([t for t in range(1, nz + 1) if nz % t == 0 and t <= 64])
    dims, td = (512, ny, nz), (64, ty, tz)
    u = synth.uniform_grid(*dims, case)
    total = 0
    with T.Domain(dims, td) as d:
        d.load(u)
        for k in range(3):
            steps = rng.choice([1, 2, 3, 5, 8, 13, 21, 34, 40, 70])
            d.run(T.heat7(), steps, rng.choice([1, 2, 4]))
            total += steps
            sched = d.get_info()["last_schedule"]
            out = d.store()
            assert np.array_equal(out, oracle.heat_c(u, ALPHA, total)), (dims, td, total, sched)
            if rng.random() < 0.5:   # the next run starts from the host store again
                d.invalidate()


@pytest.mark.parametrize("case", range(40))
def test_general_shapes_random_bit_exact(case):
    """Seeded random shapes off the band layout (any width, tile shapes,
    ghost 1 or 2, periodic or Dirichlet, stream budgets) and run sequences
    through the default schedules; every stored grid against the oracle."""
    import random
    rng = random.Random(5000 + case)
    def dim():
        n = rng.choice([8, 16, 24, 32, 48, 64, 96, 128])
        t = rng.choice([t for t in (4, 8, 16, 32, 64) if n % t == 0 and t <= n] or [n])
        return n, t
    (nx, tx), (ny, ty), (nz, tz) = dim(), dim(), dim()
    dims, td = (nx, ny, nz), (tx, ty, tz)
    ghost = rng.choice([1, 1, 2])
    bc = rng.choice(["periodic", "periodic", "dirichlet"])
    kw = {"ghost": ghost, "bc": bc}
    if rng.random() < 0.3:   # out of core: a budget of a few tiles
        kw["sched"] = "stream"
        kw["device_budget_bytes"] = int(8 * tx * ty * tz * 8 * rng.choice([3, 5, 9]) + (1 << 20))
    ext = synth.uniform_grid(nx + 2, ny + 2, nz + 2, case) if bc == "dirichlet" else None
    u = ext[1:-1, 1:-1, 1:-1].copy() if ext is not None else synth.uniform_grid(nx, ny, nz, case)
    try:
        d = T.Domain(dims, td, **kw)
    except T.TileError:
        pytest.skip("shape not accepted")
    total = 0
    with d:
        d.load(ext if ext is not None else u)
        for k in range(3):
            steps = rng.choice([1, 2, 3, 5, 8, 13])
            d.run(T.heat7(), steps, rng.choice([1, 2, 3, 4]))
            total += steps
            out = d.store()
            if ext is not None:   # store() returns the extended array: compare the interiors
                ref = oracle.heat_c(ext, ALPHA, total, oracle.BC_DIRICHLET)[1:-1, 1:-1, 1:-1]
                out = out[1:-1, 1:-1, 1:-1]
            else:
                ref = oracle.heat_c(u, ALPHA, total)
            assert np.array_equal(out, ref), (dims, td, kw, total, d.get_info()["last_schedule"])


@pytest.mark.parametrize("two_step", [0, 1])
def test_band2_with_ghost2_domains_bit_exact(two_step):
    """Ghost-2 domains 512 wide: resident runs take heat2_band (faces left
    stale), the next face-reading run (the layered first phase, heat7x2
    passes with two_step = 1, the odd step) re-extracts depth-2 faces."""
    dims, td = (512, 64, 64), (64, 32, 16)
    out, ref, info, st = _heat(dims, td, 12, runs=[3, 4, 5], ghost=2, two_step=two_step)
    assert np.array_equal(out, ref), np.abs(out - ref).max()


@pytest.mark.parametrize("T_", [70, 73])
def test_large_T_split_wavefront_bit_exact(T_):
    """Fresh upload at large T: wavefront during the upload, two-step passes,
    wavefront during the download (last_schedule 8); bit-exact, then a
    resident continuation."""
    dims, td = (512, 64, 128), (64, 64, 16)
    u0 = synth.uniform_grid(*dims, 21)
    with T.Domain(dims, td) as d:
        d.load(u0)
        d.run(T.heat7(), T_, 4)
        out1 = d.store()
        sched = d.get_info()["last_schedule"]
        st = d.stats()
        d.run(T.heat7(), 3, 2)
        out2 = d.store()
    assert sched == 8
    assert np.array_equal(out1, oracle.heat_c(u0, ALPHA, T_))
    assert np.array_equal(out2, oracle.heat_c(u0, ALPHA, T_ + 3))
    assert st["bytes_h2d"] == u0.nbytes and st["bytes_d2h"] == u0.nbytes


@pytest.mark.parametrize("T_", [7, 9, 12, 40])
def test_band2_middle_of_batched_fresh_upload_bit_exact(T_):
    """Fresh upload on the batched schedule: the load-overlapping layer steps,
    the middle steps in pairs on heat2_band, the layered last step(s)."""
    dims, td = (512, 64, 128), (64, 64, 16)
    out, ref, info, st = _heat(dims, td, T_, wavefront=-1, stream_through=-1)
    assert np.array_equal(out, ref), np.abs(out - ref).max()


@pytest.mark.parametrize("td,runs", [((32, 64, 8), [1, 4]), ((32, 128, 8), [2, 5])])
def test_banded_round_robin_snake_bit_exact(td, runs):
    """Banded tiles (ty > band) with enough columns for the round-robin
    column order (HeatParams::rr_rounds >= 1 at 148 CTAs), then a persistent
    multi-step launch in snake order (odd steps reversed): bit-exact."""
    dims = (512, 512, 16)
    out, ref, _, _ = _heat(dims, td, sum(runs), runs=runs)
    assert np.array_equal(out, ref), np.abs(out - ref).max()


def test_cost_model_calibrated_on_device():
    """tile_domain_create measures the fresh-upload cost model's ratio (one
    sweep's time per plane / one plane's duplex host-link time) on the box;
    an explicit tile_options value overrides it."""
    d = T_.Domain((512, 512, 512), (64, 64, 64))
    r = d.get_info()["sweep_link_ratio"]
    d.free()
    assert 0.003 < r < 0.2, r
    d = T_.Domain((512, 512, 512), (64, 64, 64), sweep_link_ratio=0.05)
    assert d.get_info()["sweep_link_ratio"] == 0.05
    d.free()
