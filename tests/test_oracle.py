"""Pins of the oracle against things other than itself (CPU only).

Every pin names what fixes the expected value: the paper's text, a closed
form of the discrete heat equation, an invariant, a hand-derived fixture
under tests/golden/, or an independently computed survey value.
"""
import hashlib
import math
import os
from fractions import Fraction

import numpy as np
import pytest

import oracle
import synth

ALPHA = 0.125


def _read_rows(path):
    rows = []
    for line in open(path):
        line = line.strip()
        if line and not line.startswith("#"):
            rows.append(line.split())
    return rows


# ---------------------------------------------------------------- generator
def test_splitmix64_reference_vectors(golden_dir):
    for k, hexv in _read_rows(os.path.join(golden_dir, "splitmix64_vectors.txt")):
        state = np.uint64((int(k) * 0x9E3779B97F4A7C15) % (1 << 64))
        assert int(synth.splitmix64(state)) == int(hexv, 16)


def test_generator_native_twin_matches_numpy():
    ref = synth.uniform_block(7, 5, 6, 42, -2, 3, 4, 4, 3, 9)
    out = np.empty((4, 3, 9))
    synth.fill_uniform_native(out.ctypes.data, 7, 5, 6, -2, 4, 3, 3, 4, 9, 42)
    assert np.array_equal(out, ref)


# ---------------------------------------------------- survey-computed values
def test_c1_survey_values(golden_dir):
    rows = _read_rows(os.path.join(golden_dir, "c1_survey_values.txt"))
    u0 = synth.uniform_grid(64, 64, 64, 42)
    u10 = oracle.heat_c(u0, ALPHA, 10)
    for kind, z, y, x, val in rows:
        if kind == "u0":
            assert u0[int(z), int(y), int(x)] == float(val)
        elif kind == "u10":
            assert u10[int(z), int(y), int(x)] == float(val)
        elif kind == "min10":
            assert u10.min() == float(val)
        elif kind == "max10":
            assert u10.max() == float(val)
        elif kind == "sha_u0":
            assert hashlib.sha256(u0.tobytes()).hexdigest() == val
        elif kind == "sha_u10":
            assert hashlib.sha256(u10.tobytes()).hexdigest() == val


# ------------------------------------------------------------- closed forms
@pytest.mark.parametrize("impl", [oracle.heat_c, oracle.heat_np])
def test_constant_field_unchanged_bit_exact(impl):
    u = synth.constant_grid(6, 5, 7, 0.3)
    assert np.array_equal(impl(u, ALPHA, 5), u)


@pytest.mark.parametrize("impl", [oracle.heat_c, oracle.heat_np])
def test_linear_field_dirichlet_unchanged(impl):
    # discrete Laplacian of a linear field is zero; integer values are exact
    ue = synth.linear_grid(7, 6, 5, g=1)
    out = impl(ue, ALPHA, 6, oracle.BC_DIRICHLET)
    assert np.array_equal(out, ue)


def test_linear_field_periodic_interior_unchanged():
    T = 2
    u = synth.linear_grid(12, 11, 10)
    out = oracle.heat_c(u, ALPHA, T)
    # cells farther than T from the periodic seam never see the wrap
    sl = (slice(T, 10 - T), slice(T, 11 - T), slice(T, 12 - T))
    assert np.array_equal(out[sl], u[sl])
    assert not np.array_equal(out, u)  # the seam does diffuse


@pytest.mark.parametrize("n,m,alpha,T", [(16, (1, 1, 1), 0.125, 10),
                                         (12, (2, 1, 3), 0.1, 7),
                                         (10, (1, 2, 1), 1.0 / 6.0, 5)])
def test_sine_mode_periodic_eigen_decay(n, m, alpha, T):
    # u = prod_d sin(2 pi m_d i_d / n): u^T = lambda^T u,
    # lambda = 1 - 2 alpha sum_d (1 - cos(2 pi m_d / n))
    u = synth.sine_grid(n, n, n, m)
    lam = 1 - 2 * alpha * sum(1 - math.cos(2 * math.pi * md / n) for md in m)
    out = oracle.heat_c(u, alpha, T)
    err = np.abs(out - lam ** T * u).max() / np.abs(u).max()
    assert err <= 1e-12


@pytest.mark.parametrize("n,T", [(9, 10), (14, 4)])
def test_sine_mode_dirichlet_eigen_decay(n, T):
    # Dirichlet-zero: lambda = 1 - 6 alpha (1 - cos(pi/(n+1))) for m = (1,1,1)
    ue = synth.sine_grid_dirichlet(n, n, n)
    lam = 1 - 6 * ALPHA * (1 - math.cos(math.pi / (n + 1)))
    out = oracle.heat_c(ue, ALPHA, T, oracle.BC_DIRICHLET)
    err = np.abs(out - lam ** T * ue).max() / np.abs(ue).max()
    assert err <= 1e-12
    assert np.array_equal(out[0], ue[0]) and np.array_equal(out[:, :, -1], ue[:, :, -1])


def test_delta_green_function_hand_values(golden_dir):
    for impl in (oracle.heat_c, oracle.heat_np):
        for steps, dz, dy, dx, val in _read_rows(os.path.join(golden_dir, "delta_green.txt")):
            u = np.zeros((8, 8, 8))
            u[4, 4, 4] = 1.0
            out = impl(u, ALPHA, int(steps))
            assert out[4 + int(dz), 4 + int(dy), 4 + int(dx)] == float(val)


def test_delta_green_function_exact_rational():
    # the whole field after T steps equals (L^T delta) computed in exact
    # rational arithmetic by sparse polynomial powers of
    # L = (1-6a) I + a sum_{d,+-} S_d  (independent representation)
    a = Fraction(1, 8)
    field = {(0, 0, 0): Fraction(1)}
    T = 3
    shifts = [(1, 0, 0), (-1, 0, 0), (0, 1, 0), (0, -1, 0), (0, 0, 1), (0, 0, -1)]
    for _ in range(T):
        new = {}
        for p, v in field.items():
            new[p] = new.get(p, 0) + (1 - 6 * a) * v
            for s in shifts:
                q = (p[0] + s[0], p[1] + s[1], p[2] + s[2])
                new[q] = new.get(q, 0) + a * v
        field = new
    u = np.zeros((10, 10, 10))
    u[5, 5, 5] = 1.0
    out = oracle.heat_c(u, 0.125, T)
    exp = np.zeros_like(out)
    for (dz, dy, dx), v in field.items():
        exp[5 + dz, 5 + dy, 5 + dx] = float(v)
    assert np.array_equal(out, exp)


def test_brute_force_python_loops_tiny():
    # pure-Python loops with explicit neighbour indices (not a stencil library)
    nz, ny, nx = 3, 4, 5
    u = synth.uniform_grid(nx, ny, nz, 3)
    ref = [[[float(u[z, y, x]) for x in range(nx)] for y in range(ny)] for z in range(nz)]
    for _ in range(3):
        new = [[[0.0] * nx for _ in range(ny)] for _ in range(nz)]
        for z in range(nz):
            for y in range(ny):
                for x in range(nx):
                    c = ref[z][y][x]
                    xs = ref[z][y][(x - 1) % nx] + ref[z][y][(x + 1) % nx]
                    ys = ref[z][(y - 1) % ny][x] + ref[z][(y + 1) % ny][x]
                    zs = ref[(z - 1) % nz][y][x] + ref[(z + 1) % nz][y][x]
                    new[z][y][x] = c + 0.125 * (((xs + ys) + zs) - 6.0 * c)
        ref = new
    assert np.array_equal(oracle.heat_c(u, 0.125, 3), np.array(ref))


# --------------------------------------------------------------- invariants
def test_numpy_twin_bit_exact_with_c():
    u = synth.uniform_grid(9, 8, 7, 42)
    assert np.array_equal(oracle.heat_c(u, 0.1, 6), oracle.heat_np(u, 0.1, 6))
    ue = synth.uniform_grid(11, 10, 9, 5)
    assert np.array_equal(oracle.heat_c(ue, 0.1, 4, oracle.BC_DIRICHLET),
                          oracle.heat_np(ue, 0.1, 4, oracle.BC_DIRICHLET))


def test_periodic_shift_equivariance():
    u = synth.uniform_grid(10, 9, 8, 42)
    out = oracle.heat_c(u, ALPHA, 4)
    for sh in [(1, 0, 0), (0, 3, 0), (0, 0, 7), (5, 2, 1)]:
        rolled = np.roll(u, sh, axis=(0, 1, 2))
        assert np.array_equal(oracle.heat_c(rolled, ALPHA, 4), np.roll(out, sh, axis=(0, 1, 2)))


def test_reflections_and_xy_transpose():
    u = synth.uniform_grid(8, 8, 6, 11)
    out = oracle.heat_c(u, ALPHA, 3)
    for ax in (0, 1, 2):
        f = np.flip(u, ax)
        assert np.array_equal(oracle.heat_c(f, ALPHA, 3), np.flip(out, ax))
    tr = np.ascontiguousarray(np.swapaxes(u, 1, 2))
    assert np.array_equal(oracle.heat_c(tr, ALPHA, 3), np.swapaxes(out, 1, 2))


def test_conservation_and_max_principle():
    u = synth.uniform_grid(12, 10, 8, 42)
    T = 20
    out = oracle.heat_c(u, 1.0 / 6.0, T)
    eps = np.finfo(np.float64).eps
    assert abs(out.sum() - u.sum()) <= u.size * T * eps * np.abs(u).max() * 8
    assert out.min() >= u.min() and out.max() <= u.max()
    assert out.std() < u.std()


# --------------------------------------------------------------------- tiles
def test_ghost_map_hand_values(golden_dir):
    for bc, k, j, i, exp in _read_rows(os.path.join(golden_dir, "ghost_map_hand.txt")):
        b = oracle.BC_PERIODIC if bc == "periodic" else oracle.BC_DIRICHLET
        m = oracle.ghost_map((4, 2, 2), (2, 2, 2), 1, 1, b)
        assert m[int(k), int(j), int(i)] == int(exp)


def test_ghost_map_interior_identity_and_wrap():
    dims, td, g = (6, 4, 4), (3, 2, 4), 2
    for t in range(2 * 2 * 1):
        m = oracle.ghost_map(dims, td, g, t)
        ox, oy, oz = oracle.oracle.tile_origin(dims, td, t)
        inner = m[g:-g, g:-g, g:-g]
        zz, yy, xx = np.meshgrid(np.arange(oz, oz + 4), np.arange(oy, oy + 2),
                                 np.arange(ox, ox + 3), indexing="ij")
        assert np.array_equal(inner, (zz * 4 + yy) * 6 + xx)
        assert m.min() >= 0 and m.max() < 96


@pytest.mark.parametrize("bc", [oracle.BC_PERIODIC, oracle.BC_DIRICHLET])
@pytest.mark.parametrize("td", [(4, 4, 4), (8, 4, 2), (8, 8, 8), (2, 2, 2)])
def test_tiled_equals_untiled_bit_exact(bc, td):
    T = 4
    if bc == oracle.BC_PERIODIC:
        u = synth.uniform_grid(8, 8, 8, 42)
        ref = oracle.heat_c(u, 0.1, T)
        out = oracle.tiled_heat(u, td, 0.1, T)
        assert np.array_equal(out, ref)
    else:
        ue = synth.uniform_grid(10, 10, 10, 9)
        ref = oracle.heat_c(ue, 0.1, T, bc)
        out = oracle.tiled_heat(ue[1:-1, 1:-1, 1:-1], td, 0.1, T, bc, halo=ue)
        assert np.array_equal(out, ref[1:-1, 1:-1, 1:-1])


def test_cone_block_matches_full_run():
    nx, ny, nz, T = 16, 12, 10, 3
    full = oracle.heat_c(synth.uniform_grid(nx, ny, nz, 42), ALPHA, T)
    for (z0, y0, x0) in [(0, 0, 0), (8, 10, 14), (4, 5, 6)]:
        blk = oracle.cone_block(nx, ny, nz, 42, ALPHA, T, z0, y0, x0, 2, synth.uniform_block)
        ref = full[np.ix_([(z0 + i) % nz for i in range(2)], [(y0 + i) % ny for i in range(2)],
                          [(x0 + i) % nx for i in range(2)])]
        assert np.array_equal(blk, ref)


# ------------------------------------------------------------------ sincos
def test_sincos_special_values():
    # sin(0)=0, cos(0)=1, sqrt(1)=1: one iteration maps 0 -> 1 exactly
    assert oracle.sincos_c(np.zeros(3), 1)[0] == 1.0
    x = synth.uniform_grid(4, 2, 1, 7)
    assert np.array_equal(oracle.sincos_c(x, 0, 5), x)  # K = 0: no iteration


def test_sincos_closed_form_and_py_twin():
    # sqrt(sin^2 + cos^2) == 1 up to one rounding, so x_T ~ x_0 + K*T
    x0 = synth.uniform_grid(8, 8, 8, 7).ravel()
    K, T = 32, 10
    out = oracle.sincos_c(x0, K, T)
    s = x0.copy()
    for _ in range(K * T):
        s = s + 1.0
    ulp = np.spacing(out)
    assert np.all(np.abs(out - s) <= 4 * ulp)
    assert np.array_equal(oracle.sincos_py(x0[:16], K, T), out[:16])


def test_sincos_survey_values():
    # seed 7, first 4 cells of an 8^3 grid, K*T = 320
    x0 = synth.uniform_grid(8, 8, 8, 7).ravel()[:4]
    assert np.allclose(x0, [0.771546556331567, 0.5230671798509814,
                            0.7390873243475791, 0.8887184341115442], rtol=0, atol=1e-15)
    out = oracle.sincos_c(x0, 32, 10)
    exp = [320.7715465563316, 320.52306717985095, 320.73908732434757, 320.8887184341115]
    assert np.abs(out - exp).max() / 320 <= 1e-12


# ---------------------------------------------------------------- residency
def test_residency_fig7_trace(golden_dir):
    exp = [(op, int(r), int(p)) for op, r, p in
           _read_rows(os.path.join(golden_dir, "residency_fig7.txt"))]
    ro = oracle.ResidencyOracle(2)
    for _ in range(2):
        for r in range(4):
            ro.gpu_request(r)
    assert ro.trace == exp


def _residency_cases(path):
    cases, cur = [], None
    for row in _read_rows(path):
        if row[0] == "case":
            cur = {"nslots": int(row[2]), "steps": []}
            cases.append(cur)
        elif row[0] == ">":
            cur["steps"].append((row[1:], []))
        else:
            cur["steps"][-1][1].append((row[0], int(row[1]), int(row[2])))
    return cases


@pytest.mark.parametrize("track_dirty", [True, False])
def test_residency_dirty_tracking_golden(golden_dir, track_dirty):
    """Hand-derived traces (readings R4/R10). Without dirty
    tracking (the paper's literal rule) every drop becomes a D2H and every
    GPU-disabled request of a device region copies."""
    for case in _residency_cases(os.path.join(golden_dir, "residency_dirty.txt")):
        ro = oracle.ResidencyOracle(case["nslots"], track_dirty=track_dirty)
        for req, exp in case["steps"]:
            n0 = len(ro.trace)
            if req[0] == "gpu":
                ro.gpu_request(int(req[1]), writes=req[2] == "w")
            elif req[0] == "cpu":
                ro.cpu_request(int(req[1]))
            else:
                ro.jacobi_request(int(req[1]), int(req[2]), int(req[3]))
            if not track_dirty:
                exp = [("d2h",) + e[1:] if e[0] == "drop" else e for e in exp]
                if req[0] == "cpu" and not exp and int(req[1]) in ro.cache:
                    exp = [("d2h", int(req[1]), ro.cache.index(int(req[1])))]
            assert ro.trace[n0:] == exp, (req, ro.trace[n0:], exp)


def test_residency_one_pointer_per_region():
    ro = oracle.ResidencyOracle(3, track_dirty=True)
    ro.jacobi_request(0, 0, 1)
    with pytest.raises(ValueError):
        ro.gpu_request(0, slot=2)      # region 0 lives in pointer 1
    with pytest.raises(ValueError):
        ro.jacobi_request(0, 0, 2)
    with pytest.raises(ValueError):
        ro.jacobi_request(1, 2, 2)


def test_residency_all_fit_only_first_sweep_transfers():
    ro = oracle.ResidencyOracle(4)
    for _ in range(3):
        for r in range(4):
            ro.gpu_request(r)
    ops = [t[0] for t in ro.trace]
    assert ops.count("h2d") == 4 and ops.count("d2h") == 0 and ops.count("hit") == 8
    ro.cpu_request(2)
    assert ro.trace[-1] == ("d2h", 2, 2)


def test_all_core_twin_is_bit_identical():
    """The OpenMP twin (all-core CPU baseline) equals the
    single-threaded oracle bit for bit, and both equal the NumPy twin."""
    u = synth.uniform_grid(24, 20, 18, 42)
    one = oracle.heat_c(u, ALPHA, 4)
    for th in (2, 3, 8):
        assert np.array_equal(oracle.heat_c(u, ALPHA, 4, threads=th), one)
    assert np.array_equal(one, oracle.heat_np(u, ALPHA, 4))
