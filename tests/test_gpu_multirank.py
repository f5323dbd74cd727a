"""Multi-rank (z-slab) CUDA path on ONE GPU through the in-process transport
(tile_local_group_create): one domain per rank, each driven by its own host
thread; halo exchanges are real device copies ordered by cross-rank events.
Checks the whole multi-rank scheduling path (halo ops, boundary batches,
halo-sourced ghost planes in the kernels) bit-exactly against the oracle on
the global grid. The NCCL transport replaces only the copy step."""
import threading

import numpy as np
import pytest

import oracle
import synth

pytestmark = pytest.mark.gpu
T = pytest.importorskip("paper_conf_icpp_bastemuzas17_b200.tiles")
ALPHA = 0.125


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")


def _budget(dims, td, nslots, **kw):
    lo, hi = 1, 1 << 40
    while lo < hi:
        mid = (lo + hi) // 2
        try:
            n = T.Domain(dims, td, dry_run=True, sched="stream", device_budget_bytes=mid, **kw).info["nslots"]
        except T.TileError:
            n = -1
        lo, hi = (lo, mid) if n >= nslots else (mid + 1, hi)
    return lo


@pytest.mark.parametrize("G,bc,sched,runs", [(2, "periodic", "resident", [5]), (2, "dirichlet", "resident", [3, 2]),
                                             (4, "periodic", "resident", [4, 3]), (2, "periodic", "stream", [4]),
                                             (3, "dirichlet", "stream", [2, 3]), (8, "periodic", "resident", [6])])
def test_local_group_slabs_bit_exact(G, bc, sched, runs):
    dims, td = (64, 32, 16 * G), (32, 16, 8)
    nx, ny, nz = dims
    nzl = nz // G
    if bc == "periodic":
        u = synth.uniform_grid(nx, ny, nz, 42)
        ref = oracle.heat_c(u, ALPHA, sum(runs))
    else:
        ext = synth.uniform_grid(nx + 2, ny + 2, nz + 2, 5)
        ref = oracle.heat_c(ext, ALPHA, sum(runs), oracle.BC_DIRICHLET)[1:-1, 1:-1, 1:-1]
    group = T.LocalGroup(G)
    out = [None] * G
    err = []

    def rank(r):
        try:
            kw = {"sched": sched}
            if sched == "stream":
                kw["device_budget_bytes"] = _budget(dims, td, 3, bc=bc, nranks=G, rank=r)
            with T.Domain(dims, td, bc=bc, nranks=G, rank=r, local_group=group, device=0, **kw) as d:
                d.load(u[r * nzl:(r + 1) * nzl] if bc == "periodic" else ext[r * nzl:r * nzl + nzl + 2])
                for s in runs:
                    d.run(T.heat7(ALPHA), s, 2)
                o = d.store()
                out[r] = o if bc == "periodic" else o[1:-1, 1:-1, 1:-1]
        except Exception as e:  # noqa
            err.append(e)

    th = [threading.Thread(target=rank, args=(r,)) for r in range(G)]
    for t in th:
        t.start()
    for t in th:
        t.join(120)
    group.free()
    assert not err, err
    got = np.concatenate(out, axis=0)
    assert np.array_equal(got, ref), np.abs(got - ref).max()
