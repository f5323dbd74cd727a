"""Copy-engine gap probe: back-to-back H2D copies on one stream while D2H
copies run on another (the stream-through pattern), timed with CUPTI
(torch.profiler). Reports the idle gap between consecutive H2D copies for
1-D and strided 2-D copies, with and without concurrent D2H.

  python tools/pcie_gap.py out.json
"""
import json
import sys

import torch
from torch.profiler import ProfilerActivity, profile

MB = 1 << 20


def run(kind, duplex, chunk_mb=32, n=24, rows=64):
    dev = torch.device("cuda")
    nb = chunk_mb * MB
    h_in = torch.empty(n * nb, dtype=torch.uint8, pin_memory=True)
    h_out = torch.empty(n * nb, dtype=torch.uint8, pin_memory=True)
    d_buf = torch.empty(n * nb, dtype=torch.uint8, device=dev)
    d_src = torch.empty(n * nb, dtype=torch.uint8, device=dev)
    s_in, s_out = torch.cuda.Stream(), torch.cuda.Stream()
    torch.cuda.synchronize()

    def issue():
        for i in range(n):
            with torch.cuda.stream(s_in):
                if kind == "1d":
                    d_buf[i * nb:(i + 1) * nb].copy_(h_in[i * nb:(i + 1) * nb], non_blocking=True)
                else:  # strided: rows pieces of nb/rows bytes, host pitch 4x
                    w = nb // rows
                    src = h_in[i * nb:(i + 1) * nb].view(rows, w)
                    d_buf[i * nb:(i + 1) * nb].view(rows, w).copy_(src, non_blocking=True)
            if duplex:
                with torch.cuda.stream(s_out):
                    h_out[i * nb:(i + 1) * nb].copy_(d_src[i * nb:(i + 1) * nb], non_blocking=True)
    issue()
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        issue()
        torch.cuda.synchronize()
    ev = [e for e in prof.events() if e.device_type.name == "CUDA"]
    h = sorted((e.time_range.start, e.time_range.end) for e in ev if "HtoD" in e.name)
    d = sorted((e.time_range.start, e.time_range.end) for e in ev if "DtoH" in e.name)
    gaps = [h[i + 1][0] - h[i][1] for i in range(len(h) - 1)]
    durs = [b - a for a, b in h]
    span = h[-1][1] - h[0][0]
    return {"kind": kind, "duplex": duplex, "chunk_mb": chunk_mb, "n_h2d": len(h), "n_d2h": len(d),
            "h2d_us_median": sorted(durs)[len(durs) // 2], "gap_us_median": sorted(gaps)[len(gaps) // 2],
            "gap_us_max": max(gaps), "h2d_span_us": span, "h2d_gbs": n * nb / span / 1e3}


def main():
    out = []
    for kind in ("1d", "2d"):
        for duplex in (False, True):
            for chunk in (8, 32, 128):
                r = run(kind, duplex, chunk, n=max(8, 768 // chunk))
                print(json.dumps(r), flush=True)
                out.append(r)
    json.dump(out, open(sys.argv[1], "w"), indent=1)


if __name__ == "__main__":
    main()
