"""CUPTI timeline (torch.profiler) of one e2e run — the Fig. 7 analogue
(nsys is not in the image). Writes a chrome trace and an overlap summary:
busy time of kernels, H2D and D2H and their pairwise overlaps.

  python tools/timeline.py {c4|c3|c2|wave} out_prefix
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from torch.profiler import ProfilerActivity, profile

import synth
from paper_conf_icpp_bastemuzas17_b200 import tiles as T


def union(iv):
    iv = sorted(iv)
    out = []
    for a, b in iv:
        if out and a <= out[-1][1]:
            out[-1][1] = max(out[-1][1], b)
        else:
            out.append([a, b])
    return out


def inter(a, b):
    i = j = 0
    tot = 0.0
    while i < len(a) and j < len(b):
        lo, hi = max(a[i][0], b[j][0]), min(a[i][1], b[j][1])
        if hi > lo:
            tot += hi - lo
        if a[i][1] < b[j][1]:
            i += 1
        else:
            j += 1
    return tot


def main():
    cfg, prefix = sys.argv[1], sys.argv[2]
    if cfg == "c4":
        n, td, kern, steps, kw = 512, (64, 64, 64), T.sincos(32), 10, {}
    elif cfg == "c2":
        n, td, kern, steps, kw = 512, (64, 64, 64), T.heat7(), 10, {}
    elif cfg == "wave":   # C2 shape, fresh upload at T = 64 (env T): the wavefront schedule
        n, td, kern, steps, kw = 512, (64, 64, 64), T.heat7(), int(os.environ.get("T", "64")), {}
    else:  # small out-of-core heat, budget for 8 tiles
        n, td, kern, steps, kw = 512, (128, 128, 128), T.heat7(), 2, {"sched": "stream",
                                                                        "device_budget_bytes": 1200 << 20}
    d = T.Domain((n, n, n), td, **kw)
    u = np.empty((n, n, n))
    synth.fill_uniform_native(u.ctypes.data, n, n, n, 0, n, 0, n, 0, n, 7)
    d.load(u)
    d.run(kern, steps, 4)  # warm-up at the same T (schedule, scratch)
    d.sync()
    d.invalidate()
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA, ProfilerActivity.CPU]) as prof:
        d.run(kern, steps, 4)
        d.sync()
        torch.cuda.synchronize()
    prof.export_chrome_trace(prefix + ".trace.json")
    ev = json.load(open(prefix + ".trace.json"))["traceEvents"]
    ker, h2d, d2h = [], [], []
    for e in ev:
        if e.get("ph") != "X" or "dur" not in e:
            continue
        iv = (e["ts"], e["ts"] + e["dur"])
        cat, name = e.get("cat", ""), e.get("name", "")
        if cat == "kernel":
            ker.append(iv)
        elif cat in ("gpu_memcpy", "memcpy") or "Memcpy" in name:
            (h2d if "HtoD" in name else d2h if "DtoH" in name else []).append(iv)
    K, H, D = union(ker), union(h2d), union(d2h)
    span = max(x[1] for x in ker + h2d + d2h) - min(x[0] for x in ker + h2d + d2h)
    busy = lambda s: sum(b - a for a, b in s)
    summ = {"config": cfg, "span_us": span, "kernel_busy_us": busy(K), "h2d_busy_us": busy(H),
            "d2h_busy_us": busy(D), "kernel_and_h2d_us": inter(K, H), "kernel_and_d2h_us": inter(K, D),
            "h2d_and_d2h_us": inter(H, D), "n_kernels": len(ker), "n_h2d": len(h2d), "n_d2h": len(d2h)}
    xfer = union(h2d + d2h)
    summ["transfer_busy_us"] = busy(xfer)
    summ["transfer_hidden_under_kernels"] = inter(xfer, K) / max(1e-9, busy(xfer))
    t0 = min(x[0] for x in ker + h2d + d2h)
    rel = lambda L: [[round(a - t0, 1), round(b - t0, 1)] for a, b in sorted(L)]
    json.dump({"h2d": rel(h2d), "d2h": rel(d2h), "kernels": rel(ker)}, open(prefix + ".intervals.json", "w"))
    json.dump(summ, open(prefix + ".summary.json", "w"), indent=1)
    print(json.dumps(summ))


if __name__ == "__main__":
    main()
