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
from tests.conftest import import_tiles

T = import_tiles()
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


@pytest.mark.parametrize("G,bc,sched,runs,transport", [
    (2, "periodic", "resident", [5], 1), (3, "periodic", "resident", [4, 3], 1),
    (2, "dirichlet", "resident", [3], 1), (4, "periodic", "stream", [3], 1),
    (3, "dirichlet", "stream", [2, 2], 1),
    (2, "periodic", "resident", [7, 5], 2), (3, "periodic", "resident", [6, 9], 2),
    (4, "dirichlet", "resident", [8], 2), (2, "dirichlet", "resident", [4, 4], 2)])
def test_peer_transport_processes_bit_exact(G, bc, sched, runs, transport):
    """Peer transport (tile_options.peer_transport): one PROCESS per rank, all
    on the one GPU of the pool (CUDA IPC works between processes on a device
    as between devices); the halo exchange is the IPC window push with
    stream-memory-op counters, no NCCL. transport 2 = fused: the stencil
    kernel of every resident step stores its slab-end layers straight into
    the neighbours' windows and the exchange only signals. Bit-exact against
    the oracle."""
    dims, td = (64, 32, 16 * G), (32, 16, 8)
    nx, ny, nz = dims
    budget = _budget(dims, td, 3, bc=bc, nranks=G, rank=0) if sched == "stream" else 0
    outs = _peer_procs(G, dims, td, bc, sched, budget, runs, transport)
    got = np.concatenate([m[1] for m in outs], axis=0)
    if bc == "periodic":
        ref = oracle.heat_c(synth.uniform_grid(nx, ny, nz, 42), ALPHA, sum(runs))
    else:
        ext = synth.uniform_grid(nx + 2, ny + 2, nz + 2, 42)
        ref = oracle.heat_c(ext, ALPHA, sum(runs), oracle.BC_DIRICHLET)[1:-1, 1:-1, 1:-1]
        got = np.concatenate([m[1][1:-1, 1:-1, 1:-1] for m in outs], axis=0)
    assert np.array_equal(got, ref), np.abs(got - ref).max()
    assert all(m[2] > 0 and m[3] > 0 for m in outs)  # halo exchanges happened through the window


def _peer_procs(G, dims, td, bc, sched, budget, runs, transport, stream_through=0, user_runs=(),
                multi_device=False):
    """One spawned process per rank (tests/peer_worker.py), IPC handles
    relayed through pipes; returns every rank's ("out", ...) message.
    multi_device: rank r on CUDA device r (transport 0 = NCCL needs it)."""
    import multiprocessing as mp
    from tests import peer_worker
    ctx = mp.get_context("spawn")
    pipes, procs = [], []
    nid = T.nccl_unique_id() if transport == 0 else None
    for r in range(G):
        a, b = ctx.Pipe()
        p = ctx.Process(target=peer_worker.run,
                        args=(r, G, dims, td, bc, sched, budget, runs, 42, b, transport, stream_through,
                              tuple(user_runs), r if multi_device else 0, nid))
        p.start()
        pipes.append(a)
        procs.append(p)
    try:
        handles = []
        for a in pipes:
            assert a.poll(180), "worker did not report its handle"
            msg = a.recv()
            assert msg[0] == "handle", msg
            handles.append(msg[1])
        for a in pipes:
            a.send(("handles", handles))
        outs = []
        for a in pipes:
            assert a.poll(300), "worker did not finish"
            msg = a.recv()
            assert msg[0] == "out", msg
            outs.append(msg)
    finally:
        for p in procs:
            p.join(30)
            if p.is_alive():
                p.kill()
    return outs


@pytest.mark.parametrize("G,T,tz,runs_after", [(2, 4, 8, [3]), (3, 8, 16, []), (4, 1, 8, [2]),
                                               (2, 8, 16, [5, 4]), (2, 3, 8, [])])
def test_peer_stream_through_slabs_bit_exact(G, T, tz, runs_after):
    """Multi-rank stream-through (fresh upload, T <= tz, peer transport): each
    rank sweeps its slab in units of planes; the T planes of initial data
    beyond each slab end come once per run from the neighbours' halo layers
    (comm_peer.cu peer_st_halo) instead of the periodic wrap. One process per
    rank on the pool's GPU; the first run's result (host) and the resident
    runs that continue from the device copy are bit-exact against the oracle,
    and the first run moved each cell across the link exactly once per
    direction."""
    dims, td = (64, 32, 8 * tz * G), (32, 16, tz)  # 8 tile layers per rank
    nx, ny, nz = dims
    runs = [T] + runs_after
    outs = _peer_procs(G, dims, td, "periodic", "auto", 0, runs, transport=2, stream_through=1)
    u0 = synth.uniform_grid(nx, ny, nz, 42)
    first = np.concatenate([m[4][1] for m in outs], axis=0)
    assert np.array_equal(first, oracle.heat_c(u0, ALPHA, T)), np.abs(first - oracle.heat_c(u0, ALPHA, T)).max()
    got = np.concatenate([m[1] for m in outs], axis=0)
    assert np.array_equal(got, oracle.heat_c(u0, ALPHA, sum(runs)))
    nzl = nz // G
    for m in outs:
        st = m[4][0]
        assert st["bytes_h2d"] == nx * ny * nzl * 8 and st["bytes_d2h"] == nx * ny * nzl * 8
        assert st["bytes_halo"] == 2 * nx * ny * T * 8  # one layer of T planes to each neighbour


@pytest.mark.parametrize("G,bc,sched", [(2, "periodic", "resident"), (3, "dirichlet", "resident"),
                                        (4, "periodic", "stream")])
def test_local_group_user_stencil_bit_exact(G, bc, sched):
    """User 7-point stencil (the heat update as NVRTC source) on z-slab ranks
    (in-process transport), interleaved with built-in HEAT7 runs: bit-exact."""
    dims, td = (64, 32, 16 * G), (32, 16, 8)
    nx, ny, nz = dims
    nzl = nz // G
    runs = [("user", 3), ("heat", 2), ("user", 2)]
    if bc == "periodic":
        u = synth.uniform_grid(nx, ny, nz, 42)
        ref = oracle.heat_c(u, ALPHA, 7)
    else:
        ext = synth.uniform_grid(nx + 2, ny + 2, nz + 2, 5)
        ref = oracle.heat_c(ext, ALPHA, 7, oracle.BC_DIRICHLET)[1:-1, 1:-1, 1:-1]
    fs = T.UserFn("__device__ double hu(double c, double xm, double xp, double ym, double yp, double zm,"
                  " double zp) { return c + 0.125 * ((((xm + xp) + (ym + yp)) + (zm + zp)) - 6.0 * c); }",
                  "hu", stencil=True)
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
                for kind, s in runs:
                    d.run(T.user_stencil(fs) if kind == "user" else T.heat7(ALPHA), s, 2)
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


@pytest.mark.parametrize("G,transport", [(2, 2), (3, 1)])
def test_peer_user_stencil_interleaved_bit_exact(G, transport):
    """One process per rank over the peer transport (2 = fused: HEAT7 runs push
    in-kernel, user-stencil runs exchange by copies, the counters shared):
    HEAT7 / user stencil / HEAT7 / user stencil runs, bit-exact."""
    dims, td = (64, 32, 16 * G), (32, 16, 8)
    nx, ny, nz = dims
    runs = [4, 3, 5, 2]
    outs = _peer_procs(G, dims, td, "periodic", "resident", 0, runs, transport, user_runs=(1, 3))
    got = np.concatenate([m[1] for m in outs], axis=0)
    assert np.array_equal(got, oracle.heat_c(synth.uniform_grid(nx, ny, nz, 42), ALPHA, sum(runs)))



# ------------------------------------------------ several physical devices
def _need_devices(G):
    import torch
    if torch.cuda.device_count() < G:
        pytest.skip(f"needs {G} CUDA devices (this box has {torch.cuda.device_count()})")


def _oracle_ref(dims, bc, steps):
    nx, ny, nz = dims
    if bc == "periodic":
        return oracle.heat_c(synth.uniform_grid(nx, ny, nz, 42), ALPHA, steps)
    ext = synth.uniform_grid(nx + 2, ny + 2, nz + 2, 42)
    return oracle.heat_c(ext, ALPHA, steps, oracle.BC_DIRICHLET)[1:-1, 1:-1, 1:-1]


@pytest.mark.parametrize("G,transport,bc,sched,runs", [
    (2, 0, "periodic", "resident", [5, 3]), (2, 0, "dirichlet", "resident", [4]),
    (2, 0, "periodic", "stream", [3]), (4, 0, "periodic", "resident", [6]),
    (2, 1, "periodic", "resident", [5]), (2, 2, "periodic", "resident", [7, 4]),
    (4, 2, "dirichlet", "resident", [6]), (8, 2, "periodic", "resident", [5]),
    (8, 0, "periodic", "resident", [5])])
def test_multi_device_halo_transports_bit_exact(G, transport, bc, sched, runs):
    """One process per rank, rank r on CUDA device r: the NCCL send/recv
    exchange (transport 0), the peer-window copies over NVLink (1) and the
    fused in-kernel push into the neighbour GPU's window (2), bit-exact
    against the oracle on the global grid. Skips with fewer devices."""
    _need_devices(G)
    dims, td = (64, 32, 16 * G), (32, 16, 8)
    budget = _budget(dims, td, 3, bc=bc, nranks=G, rank=0) if sched == "stream" else 0
    outs = _peer_procs(G, dims, td, bc, sched, budget, runs, transport, multi_device=True)
    got = np.concatenate([m[1] if bc == "periodic" else m[1][1:-1, 1:-1, 1:-1] for m in outs], axis=0)
    ref = _oracle_ref(dims, bc, sum(runs))
    assert np.array_equal(got, ref), np.abs(got - ref).max()
    assert all(m[2] > 0 for m in outs)


@pytest.mark.parametrize("G,T,runs_after", [(2, 8, [3]), (4, 4, [2])])
def test_multi_device_stream_through_bit_exact(G, T, runs_after):
    """Multi-rank stream-through across physical devices (halo layers of
    initial data pushed once per run into the neighbour GPU's window)."""
    _need_devices(G)
    tz = 16
    dims, td = (64, 32, 8 * tz * G), (32, 16, tz)
    runs = [T] + runs_after
    outs = _peer_procs(G, dims, td, "periodic", "auto", 0, runs, transport=2, stream_through=1,
                       multi_device=True)
    u0 = synth.uniform_grid(*dims, 42)
    first = np.concatenate([m[4][1] for m in outs], axis=0)
    assert np.array_equal(first, oracle.heat_c(u0, ALPHA, T))
    got = np.concatenate([m[1] for m in outs], axis=0)
    assert np.array_equal(got, oracle.heat_c(u0, ALPHA, sum(runs)))


def _bench_line(args, env_extra):
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = {k: v for k, v in os.environ.items()
           if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT")}
    env.update(env_extra)
    r = subprocess.run([sys.executable, os.path.join(root, "bench.py"), *args], capture_output=True,
                       text=True, env=env, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [json.loads(x) for x in r.stdout.splitlines() if x.startswith("{")]
    assert len(lines) == 1, r.stdout[-3000:]
    return lines[0]


def test_bench_two_ranks_spawned_on_one_gpu():
    """`bench.py --gpus 2` spawns its own two ranks (TILES_BENCH_ONE_GPU=1:
    both on the pool's one GPU, gloo; a functional check, not a number)."""
    ln = _bench_line(["--gpus", "2", "--steps", "2", "--warmup", "1", "--no-extras", "--no-cpu-baseline"],
                     {"TILES_BENCH_ONE_GPU": "1"})
    assert ln["n_gpus"] == 2 and ln["config"]["comm_ranks"] == 2
    assert ln["config"]["transport"] == "peer" and ln["value"] > 0
    assert ln["e2e"]["h2d_bytes_per_step"] == 512 ** 3 * 8


def test_bench_multi_device_spawn():
    """`bench.py --gpus 2` over two physical devices (peer transport, then
    NCCL): one line, n_gpus 2, the transport named."""
    _need_devices(2)
    for tr in ("peer", "nccl"):
        ln = _bench_line(["--gpus", "2", "--steps", "2", "--warmup", "1", "--no-extras", "--no-cpu-baseline",
                          "--transport", tr], {})
        assert ln["n_gpus"] == 2 and ln["config"]["transport"].startswith(tr)
