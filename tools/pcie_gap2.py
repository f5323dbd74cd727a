import json, sys, torch
from torch.profiler import ProfilerActivity, profile
MB = 1 << 20
def run(chunk_mb, n, nin, nout, duplex=True):
    dev = torch.device("cuda")
    nb = chunk_mb * MB
    h_in = torch.empty(n * nb, dtype=torch.uint8, pin_memory=True)
    h_out = torch.empty(n * nb, dtype=torch.uint8, pin_memory=True)
    d_buf = torch.empty(n * nb, dtype=torch.uint8, device=dev)
    d_src = torch.empty(n * nb, dtype=torch.uint8, device=dev)
    sin = [torch.cuda.Stream() for _ in range(nin)]
    sout = [torch.cuda.Stream() for _ in range(nout)]
    torch.cuda.synchronize()
    def issue():
        for i in range(n):
            with torch.cuda.stream(sin[i % nin]):
                d_buf[i * nb:(i + 1) * nb].copy_(h_in[i * nb:(i + 1) * nb], non_blocking=True)
            if duplex:
                with torch.cuda.stream(sout[i % nout]):
                    h_out[i * nb:(i + 1) * nb].copy_(d_src[i * nb:(i + 1) * nb], non_blocking=True)
    issue(); torch.cuda.synchronize()
    a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    a.record(); issue()
    for s in sin + sout: torch.cuda.current_stream().wait_stream(s)
    b.record(); torch.cuda.synchronize()
    ms = a.elapsed_time(b)
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        issue(); torch.cuda.synchronize()
    ev = [e for e in prof.events() if e.device_type.name == "CUDA"]
    h = sorted((e.time_range.start, e.time_range.end) for e in ev if "HtoD" in e.name)
    d = sorted((e.time_range.start, e.time_range.end) for e in ev if "DtoH" in e.name)
    hs = h[-1][1] - h[0][0]; ds = (d[-1][1] - d[0][0]) if d else 1
    return {"chunk_mb": chunk_mb, "nin": nin, "nout": nout, "duplex": duplex, "ms": ms,
            "total_gbs": (2 if duplex else 1) * n * nb / ms / 1e6,
            "h2d_gbs": n * nb / hs / 1e3, "d2h_gbs": n * nb / ds / 1e3 if d else None}
out = []
cfgs = [(8, 1, 1), (32, 1, 1), (64, 1, 1), (32, 2, 2), (32, 4, 4), (64, 2, 2), (8, 4, 4)]
res = {c: [] for c in cfgs}
for rep in range(5):
    for c in cfgs:
        res[c].append(run(c[0], 1024 // c[0], c[1], c[2]))
for c in cfgs:
    rs = sorted(res[c], key=lambda r: r["ms"])
    m = rs[len(rs) // 2]
    r = {"chunk_mb": c[0], "nin": c[1], "nout": c[2], "ms_median": m["ms"], "ms_min": rs[0]["ms"],
         "total_gbs_median": m["total_gbs"], "h2d_gbs": m["h2d_gbs"], "d2h_gbs": m["d2h_gbs"]}
    print(json.dumps(r), flush=True)
    out.append(r)
json.dump(out, open(sys.argv[1], "w"), indent=1)
