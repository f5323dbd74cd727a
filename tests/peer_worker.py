"""Worker process for the peer-transport tests (test_gpu_multirank.py): one
rank of a z-slab domain with tile_options.peer_transport, exchanging its CUDA
IPC window handle with the parent over a pipe. Test infrastructure only."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


HEAT_AS_USER = ("__device__ double hu(double c, double xm, double xp, double ym, double yp, double zm,"
                " double zp) { return c + 0.125 * ((((xm + xp) + (ym + yp)) + (zm + zp)) - 6.0 * c); }")


def run(r, G, dims, td, bc, sched, budget, runs, seed, conn, transport=1, stream_through=0, user_runs=(),
        device=0, nccl_id=None):
    """transport 1/2: peer windows (copies / fused); 0: NCCL (nccl_id given,
    each rank on its own device). device: this rank's CUDA ordinal."""
    sys.path.insert(0, ROOT)
    try:
        import synth
        from paper_conf_icpp_bastemuzas17_b200 import tiles as T
        nx, ny, nz = dims
        nzl = nz // G
        kw = {"sched": sched, "stream_through": stream_through}
        if budget:
            kw["device_budget_bytes"] = budget
        if transport == 0:
            kw["nccl_id"] = nccl_id
        else:
            kw["peer_transport"] = transport
        with T.Domain(dims, td, bc=bc, nranks=G, rank=r, device=device, **kw) as d:
            conn.send(("handle", d.peer_handle() if transport else b""))
            kind, handles = conn.recv()
            if transport:
                d.peer_connect(handles)
            if bc == "periodic":
                u = synth.uniform_grid(nx, ny, nz, seed)
                d.load(u[r * nzl:(r + 1) * nzl])
            else:
                ext = synth.uniform_grid(nx + 2, ny + 2, nz + 2, seed)
                d.load(ext[r * nzl:r * nzl + nzl + 2])
            firsts = []
            fs = T.UserFn(HEAT_AS_USER, "hu", stencil=True) if user_runs else None
            for i, s in enumerate(runs):
                d.run(T.user_stencil(fs) if i in user_runs else T.heat7(0.125), s, 2)
                if i == 0:
                    d.sync()
                    firsts = [d.stats(), d.store()]
            out = d.store()
            st = d.stats()
        conn.send(("out", out, st["n_halo"], st["bytes_halo"], firsts))
    except Exception as e:  # noqa: BLE001
        conn.send(("error", repr(e)))
