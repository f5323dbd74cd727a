"""Duplex PCIe probe: H2D split over 1, 2 or 3 copy streams (alternating
chunks) while D2H runs on 0, 1 or 2 streams; reports per-direction GB/s from
CUDA events around the whole batch. Question: does a second H2D copy stream
(another copy engine, more outstanding reads) raise the H2D rate in duplex?

  python tools/pcie_dual.py out.json
"""
import json
import sys

import torch

MB = 1 << 20


def run(n_in, n_out, chunk_mb=32, total_mb=1024):
    nb = chunk_mb * MB
    n = total_mb // chunk_mb
    h_in = torch.empty(n * nb, dtype=torch.uint8, pin_memory=True)
    h_out = torch.empty(n * nb, dtype=torch.uint8, pin_memory=True)
    d_in = torch.empty(n * nb, dtype=torch.uint8, device="cuda")
    d_out = torch.empty(n * nb, dtype=torch.uint8, device="cuda")
    si = [torch.cuda.Stream() for _ in range(max(1, n_in))]
    so = [torch.cuda.Stream() for _ in range(max(1, n_out))]
    res = []
    for rep in range(4):
        torch.cuda.synchronize()
        ev = {k: (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for k in ("in", "out")}
        start = torch.cuda.Event(enable_timing=True)
        start.record()
        for s in si + so:
            s.wait_event(start)
        ends_in, ends_out = [], []
        for i in range(n):
            if n_in:
                with torch.cuda.stream(si[i % n_in]):
                    d_in[i * nb:(i + 1) * nb].copy_(h_in[i * nb:(i + 1) * nb], non_blocking=True)
            if n_out:
                with torch.cuda.stream(so[i % n_out]):
                    h_out[i * nb:(i + 1) * nb].copy_(d_out[i * nb:(i + 1) * nb], non_blocking=True)
        for s in si[:n_in]:
            e = torch.cuda.Event(enable_timing=True); e.record(s); ends_in.append(e)
        for s in so[:n_out]:
            e = torch.cuda.Event(enable_timing=True); e.record(s); ends_out.append(e)
        torch.cuda.synchronize()
        t_in = max(start.elapsed_time(e) for e in ends_in) if ends_in else 0
        t_out = max(start.elapsed_time(e) for e in ends_out) if ends_out else 0
        res.append((t_in, t_out))
    t_in, t_out = sorted(res)[1]
    gb = n * nb / 1e9
    return {"h2d_streams": n_in, "d2h_streams": n_out, "chunk_mb": chunk_mb,
            "h2d_gbs": gb / (t_in / 1e3) if t_in else None, "d2h_gbs": gb / (t_out / 1e3) if t_out else None}


def main():
    out = []
    for n_in, n_out in [(1, 0), (2, 0), (0, 1), (0, 2), (1, 1), (2, 1), (3, 1), (2, 2), (1, 2)]:
        for chunk in (8, 32):
            r = run(n_in, n_out, chunk)
            print(json.dumps(r), flush=True)
            out.append(r)
    json.dump(out, open(sys.argv[1], "w"), indent=1)


if __name__ == "__main__":
    main()
