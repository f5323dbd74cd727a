"""GPU parity at BASELINE.json's full sizes, in the launch configurations
bench.py times (C2 value + e2e paths, C3 out-of-core, C4, C5 per-GPU slab).

Grids of 8-69 GB cannot be run whole by the oracle, so sampled outputs are
checked against values the oracle computes one block at a time:
- heat: the cone oracle (oracle.cone_block, SURVEY §8(c) supporting oracle 4):
  a cell after T steps depends only on initial cells within L1 distance T, so
  a (b+2T)^3 neighbourhood regenerated from the position-addressable input
  generator gives the exact b^3 centre. Bit-exact, like every heat test.
- sincos (pointwise): the oracle on the gathered sampled cells,
  within 1e-12 relative, plus the closed form x_T ~ x_0 + K*T.
Blocks cover tile seams, unit/slab seams, the periodic corners and random
interior positions (seed 1234).

The multi-GB tests read results straight from the pinned tile store
(tile_host_tile after tile_sync), as bench.py does, so the host never holds a
second dense copy; they skip when the box lacks the host RAM.
"""
import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu

from tests.conftest import cuda_available, import_tiles

T = import_tiles()  # on a GPU box a missing libtiles.so fails, never skips
_HAVE_CUDA = cuda_available()

ALPHA = 0.125


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not _HAVE_CUDA:
        pytest.skip("no CUDA device")
    import torch
    torch.cuda.init()


def _need_host(nbytes):
    import psutil
    avail = psutil.virtual_memory().available
    if avail < 1.25 * nbytes:
        pytest.skip(f"needs {nbytes / 1e9:.0f} GB of host RAM, {avail / 1e9:.0f} GB available")


def _fill(dom, gdims, td, seed):
    """The generator's values straight into the pinned tile store (bench.py
    fill_tiles)."""
    ntx, nty, _ = dom.info["tiles"]
    for k in range(dom.info["ntiles"]):
        ix, iy, iz = k % ntx, (k // ntx) % nty, k // (ntx * nty)
        v = dom.host_tile(k)
        synth.fill_uniform_native(v.ctypes.data, gdims[0], gdims[1], gdims[2], iz * td[2], td[2],
                                  iy * td[1], td[1], ix * td[0], td[0], seed)
    dom.mark_host_dirty()


def _gather(dom, gdims, td, z0, y0, x0, b):
    """b^3 block at (z0,y0,x0) (periodic wrap) from the tile-blocked host store."""
    nx, ny, nz = gdims
    ntx, nty, _ = dom.info["tiles"]
    out = np.empty((b, b, b))
    for i in range(b):
        z = (z0 + i) % nz
        for j in range(b):
            y = (y0 + j) % ny
            for l in range(b):
                x = (x0 + l) % nx
                k = (z // td[2]) * nty * ntx + (y // td[1]) * ntx + x // td[0]
                out[i, j, l] = dom.host_tile(k)[z % td[2], y % td[1], x % td[0]]
    return out


def _seam_blocks(gdims, td, nrand, b=2):
    nx, ny, nz = gdims
    blocks = [(0, 0, 0), (nz - b // 2, ny - b // 2, nx - b // 2), (nz - 1, 0, nx - 1),
              (td[2] - 1, td[1] - 1, td[0] - 1), (nz // 2 - 1, ny // 2, nx // 2 - 1),
              (td[2] - 1, 3 * td[1] // 2, 2 * td[0] - 1)]
    rng = np.random.default_rng(1234)
    blocks += [(int(rng.integers(0, nz)), int(rng.integers(0, ny)), int(rng.integers(0, nx)))
               for _ in range(nrand)]
    return blocks


def _check_cone(dom, gdims, td, steps, blocks, b=2):
    nx, ny, nz = gdims
    for z0, y0, x0 in blocks:
        ref = oracle.cone_block(nx, ny, nz, 42, ALPHA, steps, z0, y0, x0, b, synth.uniform_block)
        got = _gather(dom, gdims, td, z0, y0, x0, b)
        assert np.array_equal(got, ref), (z0, y0, x0, np.abs(got - ref).max())


def test_c2_wavefront_fig5_path():
    """C2 512^3, 64^3 tiles, 4 streams, a fresh upload with T = 64 (the
    Fig. 5 sweep's mid range, bench.py --config fig5): the cost model takes
    the wavefront; sampled blocks at the tile, chunk and periodic seams vs
    the cone oracle, bit-exact."""
    n, td = 512, (64, 64, 64)
    gdims = (n, n, n)
    with T.Domain(gdims, td) as d:
        _fill(d, gdims, td, 42)
        d.run(T.heat7(ALPHA), 64, 4)
        d.sync()
        assert d.get_info()["last_schedule"] == 6
        blocks = _seam_blocks(gdims, td, 2)[:5] + [(n - 64, 7, 300), (n - 1, n - 1, n - 1), (n - 130, 0, 0)]
        _check_cone(d, gdims, td, 64, blocks)


@pytest.mark.parametrize("T_", [130, 131])
def test_split_large_T_schedule_full_plane_bit_exact(T_):
    """A fresh upload at T beyond the wavefront's reach on a 512 x 64 x 512
    grid (64^3 tiles): wavefront of 64 levels during the
    upload, the middle steps two per kernel, a wavefront of the last 64 (65)
    levels during the download (last_schedule 8); every cell against the
    OpenMP twin of the oracle, bit-exact."""
    import os
    dims, td = (512, 64, 512), (64, 64, 64)
    u0 = synth.uniform_grid(*dims, 41)
    with T.Domain(dims, td) as d:
        d.load(u0)
        d.run(T.heat7(ALPHA), T_, 4)
        out = d.store()
        assert d.get_info()["last_schedule"] == 8
    ref = oracle.heat_c(u0, ALPHA, T_, threads=max(1, min(16, os.cpu_count() or 1)))
    assert np.array_equal(out, ref)


@pytest.mark.parametrize("two_step", [0, -1])
def test_c2_value_path_persistent_resident(two_step):
    """C2 512^3, 64^3 tiles, 4 streams: the first run after the upload is the
    e2e (stream-through) path, the next two are bench.py's `resident` path
    (two steps per kernel, heat2_band; with two_step = -1 the persistent
    single-step launch); 30 steps in all."""
    n, td = 512, (64, 64, 64)
    gdims = (n, n, n)
    with T.Domain(gdims, td, two_step=two_step) as d:
        _fill(d, gdims, td, 42)
        for _ in range(3):
            d.run(T.heat7(ALPHA), 10, 4)
        d.sync()
        st = d.stats()
        assert d.get_info()["last_schedule"] == (7 if two_step == 0 else 1)
        _check_cone(d, gdims, td, 30, _seam_blocks(gdims, td, 6))
    assert st["n_kernels"] > 0


def test_c3_out_of_core_full_size():
    """C3 2048^3 (68.7 GB) out-of-core: device budget capped at 12 GiB
    (P:L232), 256^3 tiles, T = 10, 4 streams: bench.py --config c3 (the
    out-of-core stream-through schedule)."""
    n, td = 2048, (256, 256, 256)
    gdims = (n, n, n)
    _need_host(n ** 3 * 8)
    with T.Domain(gdims, td, sched="stream", device_budget_bytes=12 << 30) as d:
        assert d.info["nslots"] < d.info["ntiles"]  # really out of core
        _fill(d, gdims, td, 42)
        d.run(T.heat7(ALPHA), 10, 4)
        d.sync()
        st = d.stats()
        _check_cone(d, gdims, td, 10, _seam_blocks(gdims, td, 6))
    assert st["bytes_h2d"] >= n ** 3 * 8 and st["bytes_d2h"] >= n ** 3 * 8


def test_c4_sincos_full_size_sampled():
    """C4 sincos 1024^3 (8.6 GB), 128^3 tiles, K = 32, T = 10, 4 streams
    (bench.py --config c4): 8192 sampled cells vs the libm oracle."""
    n, K, steps = 1024, 32, 10
    td = (128, 128, 128)
    gdims = (n, n, n)
    _need_host(n ** 3 * 8)
    rng = np.random.default_rng(1234)
    idx = rng.integers(0, n, size=(8192, 3))
    idx[:4] = [[0, 0, 0], [n - 1, n - 1, n - 1], [127, 128, 255], [n - 1, 0, 511]]
    with T.Domain(gdims, td, ghost=1) as d:
        _fill(d, gdims, td, 7)
        d.run(T.sincos(K), steps, 4)
        d.sync()
        ntx, nty, _ = d.info["tiles"]
        got = np.array([d.host_tile((z // 128) * nty * ntx + (y // 128) * ntx + x // 128)[z % 128, y % 128, x % 128]
                        for z, y, x in idx])
    x0 = np.array([synth.uniform_block(n, n, n, 7, z, y, x, 1, 1, 1)[0, 0, 0] for z, y, x in idx])
    ref = oracle.sincos_c(x0, K, steps)
    assert np.abs(got - ref).max() / np.abs(ref).max() <= 1e-12
    s = x0.copy()
    for _ in range(K * steps):
        s = s + 1.0
    assert np.all(np.abs(got - s) <= 4 * np.spacing(got))


def test_c5_per_gpu_slab_full_size():
    """C5 per-GPU slab of the G = 8 decomposition of 4096^3 (4096 x 4096 x 512,
    68.7 GB, z-periodic alone), 64^3 tiles (32768 of them), 4 streams:
    bench.py --config c5's sequence (one step after the upload, then T = 10
    resident in one persistent launch)."""
    n, nzl = 4096, 512
    gdims, td = (n, n, nzl), (64, 64, 64)
    _need_host(n * n * nzl * 8)
    with T.Domain(gdims, td, ghost=1) as d:
        _fill(d, gdims, td, 42)
        d.run(T.heat7(ALPHA), 1, 4)
        d.run(T.heat7(ALPHA), 10, 4)
        d.sync()
        _check_cone(d, gdims, td, 11, _seam_blocks(gdims, td, 6))
