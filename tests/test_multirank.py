"""Multi-GPU (z-slab) host logic on CPU, no GPU and no NCCL.

1. In-process: G dry-run ranks' op traces are replayed jointly in random
   valid orders (tests/replay.py); the k-th halo op of every rank executes as
   one collective. The assembled slabs must equal the untiled oracle on the
   global grid, bit-exactly.
2. world_size 2 over gloo (torch.distributed, 127.0.0.1): each process
   replays its own rank's trace and performs the halo exchange with gloo
   send/recv, exactly as libtiles pairs its NCCL sends/receives.
"""
import os
import socket

import numpy as np
import pytest

import oracle
import synth
from tests.replay import Geometry, Replayer, halo_payload, halo_peers, replay_ranks, split_tiles

T = pytest.importorskip("paper_conf_icpp_bastemuzas17_b200.tiles")
ALPHA = 0.125


def _global(dims, bc):
    nx, ny, nz = dims
    if bc == "periodic":
        u = synth.uniform_grid(nx, ny, nz, 42)
        return u, None, oracle.heat_c
    ext = synth.uniform_grid(nx + 2, ny + 2, nz + 2, 5)
    return ext[1:-1, 1:-1, 1:-1].copy(), ext, oracle.heat_c


def _rank_domain(dims, td, G, r, bc, ext, u, **kw):
    d = T.Domain(dims, td, bc=bc, nranks=G, rank=r, dry_run=True, **kw)
    nzl = dims[2] // G
    if bc == "dirichlet":
        d.load(ext[r * nzl:(r + 1) * nzl + 2])
    else:
        d.load(u[r * nzl:(r + 1) * nzl])
    return d


@pytest.mark.parametrize("G", [2, 3, 4])
@pytest.mark.parametrize("bc", ["periodic", "dirichlet"])
@pytest.mark.parametrize("sched", ["resident", "stream"])
@pytest.mark.parametrize("td,fused", [((8, 4, 4), 0), ((32, 8, 4), 0), ((32, 8, 4), 2)])
def test_slab_replay_matches_global_oracle(G, bc, sched, td, fused):
    # 4 tile layers per rank; 32-wide tiles take the specialised kernel, so
    # resident single steps read y/z ghosts directly (KERNELD) and export only
    # x faces and the slab-end z faces the halo exchange sends. fused = 2: the
    # peer transport's fused mode, where those kernels also store the slab-end
    # layers straight into the neighbour ranks' receive buffers and the halo
    # op after a step only synchronises (the replay applies each push when its
    # kernel executes, so a push racing a reader breaks bit-exactness)
    if fused and sched != "resident":
        pytest.skip("fused pushes are a resident direct-pass feature")
    dims = (2 * td[0], 2 * td[1], 16 * G)
    u, ext, _ = _global(dims, bc)
    steps = [6, 5]   # first run: layered / whole-slab / layered phases; second: one phase
    kw = {"sched": sched}
    if fused:
        kw["peer_transport"] = fused
    if sched == "stream":
        kw["device_budget_bytes"] = 1  # replaced below by the minimum budget
    doms, reps = [], []
    nzl = dims[2] // G
    for r in range(G):
        if sched == "stream":
            # smallest budget giving 3 slots
            lo, hi = 1, 1 << 32
            while lo < hi:
                mid = (lo + hi) // 2
                try:
                    n = T.Domain(dims, td, bc=bc, nranks=G, rank=r, dry_run=True, sched="stream",
                                 device_budget_bytes=mid).info["nslots"]
                except T.TileError:
                    n = -1
                lo, hi = (lo, mid) if n >= 3 else (mid + 1, hi)
            kw["device_budget_bytes"] = lo
        d = _rank_domain(dims, td, G, r, bc, ext, u, **kw)
        doms.append(d)
        geo = Geometry(dims, td, nranks=G, rank=r, bc=T.BCS[bc])
        rext = ext[r * nzl:(r + 1) * nzl + 2] if ext is not None else None
        reps.append(Replayer(geo, split_tiles(geo, u[r * nzl:(r + 1) * nzl]), ALPHA, ext=rext))
    for s in steps:
        traces = []
        for d in doms:
            d.clear_trace()
            d.run(T.heat7(ALPHA), s, 2)
            d.sync()
            traces.append(d.trace())
        assert all(sum(op[0] == "halo" for op in tr) == sum(op[0] == "halo" for op in traces[0])
                   for tr in traces)
        if sched == "resident" and td[0] == 32:
            assert all(any(op[0] == "kerneld" for op in tr) for tr in traces)
            assert not any(op[0] == "kernel" for tr in traces for op in tr)
            pushes = [op for tr in traces for op in tr if op[0] == "kerneld" and op[5] & 0x100]
            signals = [op for tr in traces for op in tr if op[0] == "halo_signal"]
            assert bool(pushes) == bool(fused) and bool(signals) == bool(fused)
        replay_ranks(reps, traces, seed=s * 7 + G)
    out = np.concatenate([rep.grid() for rep in reps], axis=0)
    if bc == "periodic":
        ref = oracle.heat_c(u, ALPHA, sum(steps))
    else:
        ref = oracle.heat_c(ext, ALPHA, sum(steps), oracle.BC_DIRICHLET)[1:-1, 1:-1, 1:-1]
    assert np.array_equal(out, ref), np.abs(out - ref).max()


@pytest.mark.parametrize("G,T_,tz,ns", [(2, 4, 8, 2), (3, 3, 8, 4), (4, 1, 8, 2), (2, 8, 16, 3)])
def test_slab_stream_through_replay_matches_global_oracle(G, T_, tz, ns):
    """Multi-rank stream-through (peer transport, fresh upload, T <= tz): each
    rank's dry-run trace holds its unit pipeline plus the st_halo ops — push
    the slab-end T planes of initial data once its H2D landed and the receiver
    released the previous run's layer; wait for the neighbours' layers before
    the slab-end units' first sweeps; release after them. The joint random
    replay moves the planes between ranks only when a push executes, poisons
    a layer on release, and makes waits / pushes block on the counters, so a
    missing dependency reads NaN or stale planes. Two stream-through runs
    (fresh uploads, the second pushing into layers the first released) and a
    resident run from the device copy must equal the global oracle."""
    dims, td = (64, 32, 8 * tz * G), (32, 16, tz)
    u, _, _ = _global(dims, "periodic")
    nzl = dims[2] // G
    doms, reps = [], []
    for r in range(G):
        doms.append(_rank_domain(dims, td, G, r, "periodic", None, u, peer_transport=2, stream_through=1))
        geo = Geometry(dims, td, nranks=G, rank=r, bc=0)
        reps.append(Replayer(geo, split_tiles(geo, u[r * nzl:(r + 1) * nzl]), ALPHA))
    total = 0
    for run, (steps, fresh) in enumerate([(T_, True), (T_, True), (3, False)]):
        traces = []
        for d in doms:
            if fresh and run:
                d.invalidate()  # re-upload from the host store: a fresh stream-through run
            d.clear_trace()
            d.run(T.heat7(ALPHA), steps, ns)
            d.sync()
            traces.append(d.trace())
        sth = [op for op in traces[0] if op[0] == "st_halo"]
        assert (len(sth) == 6) == fresh, sth   # 2 pushes, 2 waits, 2 releases per rank
        assert all(op[5] == run + 1 for op in sth)
        # odd runs: halo ops as late as possible (a push that the final
        # write-back does not wait for would then read results, not u^0)
        replay_ranks(reps, traces, seed=17 * run + G, lazy=("st_halo",) if run % 2 else ())
        total += steps
        out = np.concatenate([rep.grid() for rep in reps], axis=0)
        assert np.array_equal(out, oracle.heat_c(u, ALPHA, total)), (run, np.abs(out - oracle.heat_c(u, ALPHA, total)).max())


@pytest.mark.parametrize("bc,kw,expect", [("periodic", {"peer_transport": 2}, True),
                                           ("periodic", {"peer_transport": 2, "stream_through": -1}, False),
                                           ("periodic", {"peer_transport": 1}, True),
                                           ("dirichlet", {"peer_transport": 2}, False),
                                           ("periodic", {}, False)])
def test_multi_rank_stream_through_eligibility(bc, kw, expect):
    """Multi-rank stream-through needs the peer transport (its windows carry
    the halo layers), a periodic slab and stream_through >= 0; everything
    else keeps the batched schedule (no st_halo ops in the trace)."""
    G, tz = 2, 8
    dims, td = (64, 32, 8 * tz * G), (32, 16, tz)
    u, ext, _ = _global(dims, bc)
    d = _rank_domain(dims, td, G, 0, bc, ext, u, stream_through=kw.pop("stream_through", 1), **kw)
    d.clear_trace()
    d.run(T.heat7(ALPHA), 4, 2)
    d.sync()
    tr = d.trace()
    assert any(op[0] == "st_halo" for op in tr) == expect
    assert any(op[0] == "sweep" for op in tr) == expect


def test_slab_geometry_and_face_kinds():
    d = T.Domain((16, 16, 32), (8, 8, 4), nranks=4, rank=1, dry_run=True)
    info = d.info
    assert info["local_dims"] == (16, 16, 8) and info["z_offset"] == 8 and info["tiles"] == (2, 2, 2)
    fs = d.face_sources(0)           # bottom layer: z- from the rank below
    assert tuple(fs[4]) == (2, 0)
    fs = d.face_sources(7)           # top layer, position 3: z+ from the rank above
    assert tuple(fs[5]) == (3, 3)
    dd = T.Domain((16, 16, 32), (8, 8, 4), nranks=4, rank=0, bc="dirichlet", dry_run=True)
    assert tuple(dd.face_sources(0)[4]) == (1, 0)   # global bottom: Dirichlet fixed face
    m = d.ghost_map(0)
    assert m[0, 1, 1] == (7 * 16 + 0) * 16 + 0      # z = 8 - 1 = 7 (rank 0's top plane)


# ----------------------------------------------------------------- gloo
def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _gloo_worker(rank, world, port, bc, sched, out_q):
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        dims, td = (16, 8, 16), (8, 4, 4)
        u, ext, _ = _global(dims, bc)
        nzl = dims[2] // world
        kw = {"sched": sched}
        if sched == "stream":
            kw["device_budget_bytes"] = 600_000
        d = _rank_domain(dims, td, world, rank, bc, ext, u, **kw)
        geo = Geometry(dims, td, nranks=world, rank=rank, bc=T.BCS[bc])
        rext = ext[rank * nzl:(rank + 1) * nzl + 2] if ext is not None else None

        def comm(rep, par):
            top, bot = halo_payload(rep, par)
            up, dn = halo_peers(rep.G)
            shape = top[0].shape
            send_top = torch.from_numpy(np.stack(top))
            send_bot = torch.from_numpy(np.stack(bot))
            recv_lo = torch.empty((len(top),) + shape, dtype=torch.float64)
            recv_hi = torch.empty_like(recv_lo)
            ops = []
            # same pairing as comm_nccl.cpp: sends first, then receives
            if up is not None:
                ops.append(dist.P2POp(dist.isend, send_top, up))
            if dn is not None:
                ops.append(dist.P2POp(dist.isend, send_bot, dn))
            if dn is not None:
                ops.append(dist.P2POp(dist.irecv, recv_lo, dn))
            if up is not None:
                ops.append(dist.P2POp(dist.irecv, recv_hi, up))
            for w in dist.batch_isend_irecv(ops):
                w.wait()
            if dn is not None:
                rep.halo[(0, par)] = list(recv_lo.numpy())
            if up is not None:
                rep.halo[(1, par)] = list(recv_hi.numpy())

        rep = Replayer(geo, split_tiles(geo, u[rank * nzl:(rank + 1) * nzl]), ALPHA, ext=rext, comm=comm)
        d.run(T.heat7(ALPHA), 4, 2)
        d.sync()
        rep.replay(d.trace(), seed=rank + 11)
        if bc == "periodic":
            ref = oracle.heat_c(u, ALPHA, 4)
        else:
            ref = oracle.heat_c(ext, ALPHA, 4, oracle.BC_DIRICHLET)[1:-1, 1:-1, 1:-1]
        ok = np.array_equal(rep.grid(), ref[rank * nzl:(rank + 1) * nzl])
        out_q.put((rank, bool(ok)))
    finally:
        dist.destroy_process_group()


def _gloo_st_worker(rank, world, port, out_q):
    """Multi-rank stream-through over gloo: this process replays its rank's
    dry-run trace; an st_halo push is a gloo isend of the slab-end T planes
    (tag = the receiver's side), a wait is runnable once the matching irecv
    (posted up front) has completed, a release poisons the layer."""
    import torch
    import torch.distributed as dist
    dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
    try:
        Tst, tz = 4, 8
        dims, td = (64, 32, 8 * tz * world), (32, 16, tz)
        u, _, _ = _global(dims, "periodic")
        nzl = dims[2] // world
        d = _rank_domain(dims, td, world, rank, "periodic", None, u, peer_transport=2, stream_through=1)
        geo = Geometry(dims, td, nranks=world, rank=rank, bc=0)
        rep = Replayer(geo, split_tiles(geo, u[rank * nzl:(rank + 1) * nzl]), ALPHA)
        d.run(T.heat7(ALPHA), Tst, 2)
        d.sync()
        tr = d.trace()
        assert sum(op[0] == "st_halo" for op in tr) == 6
        up, dn = halo_peers(geo)
        bufs = {side: torch.empty((Tst, dims[1], dims[0]), dtype=torch.float64) for side in (0, 1)}
        recv = {0: dist.irecv(bufs[0], src=dn, tag=0), 1: dist.irecv(bufs[1], src=up, tag=1)}
        # gloo marks an irecv complete only in wait(): wait in helper threads
        import threading
        arrived = {side: threading.Event() for side in (0, 1)}
        for side in (0, 1):
            threading.Thread(target=lambda sd=side: (recv[sd].wait(), arrived[sd].set()), daemon=True).start()
        sends = []

        def st_ready(r, op):
            return op[2] != 1 or arrived[op[3]].is_set()

        def st_exec(r, op):
            _, _, a, side, T_, _ = op
            if a == 0:  # top -> upper's lo (tag 0), bottom -> lower's hi (tag 1)
                planes = r.gather(T_, nzl - T_ if side == 1 else 0)
                sends.append(dist.isend(torch.from_numpy(np.ascontiguousarray(planes)),
                                        dst=up if side == 1 else dn, tag=1 - side))
            elif a == 1:
                r.st[side] = bufs[side].numpy().copy()
            else:
                r.st[side] = np.full_like(r.st[side], np.nan)

        rep.replay(tr, seed=rank + 5, st_ready=st_ready, st_exec=st_exec)
        for w in sends:
            w.wait()
        ok = np.array_equal(rep.grid(), oracle.heat_c(u, ALPHA, Tst)[rank * nzl:(rank + 1) * nzl])
        out_q.put((rank, bool(ok)))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_stream_through():
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_gloo_st_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(180)
    res = dict(q.get(timeout=5) for _ in range(2))
    assert res == {0: True, 1: True}


@pytest.mark.parametrize("bc,sched", [("periodic", "resident"), ("dirichlet", "stream"),
                                      ("periodic", "stream")])
def test_gloo_world2_halo_exchange(bc, sched):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_gloo_worker, args=(r, 2, port, bc, sched, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(180)
    res = dict(q.get(timeout=5) for _ in range(2))
    assert res == {0: True, 1: True}
