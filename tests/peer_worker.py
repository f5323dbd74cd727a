"""Worker process for the peer-transport tests (test_gpu_multirank.py): one
rank of a z-slab domain with tile_options.peer_transport, exchanging its CUDA
IPC window handle with the parent over a pipe. Test infrastructure only."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


HEAT_AS_USER = ("__device__ double hu(double c, double xm, double xp, double ym, double yp, double zm,"
                " double zp) { return c + 0.125 * ((((xm + xp) + (ym + yp)) + (zm + zp)) - 6.0 * c); }")


def run(r, G, dims, td, bc, sched, budget, runs, seed, conn, transport=1, stream_through=0, user_runs=()):
    sys.path.insert(0, ROOT)
    try:
        import synth
        from paper_conf_icpp_bastemuzas17_b200 import tiles as T
        nx, ny, nz = dims
        nzl = nz // G
        kw = {"sched": sched, "stream_through": stream_through}
        if budget:
            kw["device_budget_bytes"] = budget
        with T.Domain(dims, td, bc=bc, nranks=G, rank=r, peer_transport=transport, device=0, **kw) as d:
            conn.send(("handle", d.peer_handle()))
            kind, handles = conn.recv()
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
