"""Duplex PCIe probe of the stream-through's copy pattern: does the tile-
blocked host store's strided 2-D copy shape (H2D: 64 rows of `rows_h` bytes,
D2H: 64 rows of `rows_d` bytes, both with a 2 MiB pitch = one 64^3 fp64 tile)
move as fast as plain 1-D copies of the same bytes?

Per pattern: H2D of 1 GiB as a sequence of copies on one stream while D2H of
1 GiB runs as a sequence on another (no dependencies between them), span from
CUDA events; best and median of `reps`. Also each direction alone.

  python tools/pcie_pattern.py out.json
"""
import json
import statistics
import sys

import torch
from cuda.bindings import runtime as rt

MB = 1 << 20
TILE = 2 * MB  # 64^3 fp64
NT = 64        # tiles per layer


def main(out):
    total = 1 << 30
    h_in = torch.empty(total, dtype=torch.uint8).pin_memory()
    h_out = torch.empty(total, dtype=torch.uint8).pin_memory()
    d_in = torch.empty(total, dtype=torch.uint8, device="cuda")
    d_out = torch.empty(total, dtype=torch.uint8, device="cuda")
    s_in, s_out = torch.cuda.Stream(), torch.cuda.Stream()
    H2D, D2H = rt.cudaMemcpyKind.cudaMemcpyHostToDevice, rt.cudaMemcpyKind.cudaMemcpyDeviceToHost

    def issue(kind, stream, pattern, chunk):
        """1 GiB in copies of `chunk` bytes: 1-D, or 2-D = NT rows of chunk/NT
        bytes at a TILE pitch inside one 128 MiB layer (16 layers)."""
        if kind == "h2d":
            dst, src, k = d_in.data_ptr(), h_in.data_ptr(), H2D
        else:
            dst, src, k = h_out.data_ptr(), d_out.data_ptr(), D2H
        sh = stream.cuda_stream
        n = total // chunk
        if pattern == "1d":
            for i in range(n):
                rt.cudaMemcpyAsync(dst + i * chunk, src + i * chunk, chunk, k, sh)
        else:
            row = chunk // NT
            per_layer = TILE // row
            for i in range(n):
                L, j = divmod(i, per_layer)
                off = L * NT * TILE + j * row
                rt.cudaMemcpy2DAsync(dst + off, TILE, src + off, TILE, row, NT, k, sh)

    def timed(dirs, pattern, ch_in, ch_out, reps=7):
        spans = []
        for r in range(reps + 2):
            torch.cuda.synchronize()
            e0 = torch.cuda.Event(enable_timing=True)
            e0.record()
            ends = []
            for kind, s, ch in (("h2d", s_in, ch_in), ("d2h", s_out, ch_out)):
                if kind not in dirs:
                    continue
                s.wait_event(e0)
                issue(kind, s, pattern, ch)
                e = torch.cuda.Event(enable_timing=True)
                e.record(s)
                ends.append(e)
            torch.cuda.synchronize()
            if r >= 2:
                spans.append(max(e0.elapsed_time(e) for e in ends))
        gb = total * len(dirs) / 1e9
        return {"best_ms": min(spans), "median_ms": statistics.median(spans),
                "gbs_best": gb / (min(spans) / 1e3), "gbs_median": gb / (statistics.median(spans) / 1e3)}

    res = {}
    if len(sys.argv) > 2 and sys.argv[2] == "rows":
        # 2-D duplex by row size (chunk = 64 rows), rounds interleaved so that
        # drift of the link rate hits every variant alike
        cases = [(64 * MB, 32 * MB), (16 * MB, 16 * MB), (8 * MB, 8 * MB), (4 * MB, 4 * MB), (2 * MB, 2 * MB),
                 (8 * MB, 32 * MB), (64 * MB, 8 * MB)]
        for rnd in range(4):
            for ch_in, ch_out in cases:
                key = f"2d_rows_in{ch_in // NT // 1024}k_out{ch_out // NT // 1024}k"
                res.setdefault(key, []).append(timed(("h2d", "d2h"), "2d", ch_in, ch_out, reps=3)["gbs_median"])
        for k, v in res.items():
            print(k, [round(x, 1) for x in v], "median", round(statistics.median(v), 1), flush=True)
        json.dump(res, open(out, "w"), indent=1)
        return
    for pattern in ("1d", "2d"):
        for ch_in, ch_out in ((64 * MB, 32 * MB), (32 * MB, 32 * MB), (8 * MB, 8 * MB)):
            key = f"{pattern}_in{ch_in // MB}_out{ch_out // MB}"
            res[key] = {"duplex": timed(("h2d", "d2h"), pattern, ch_in, ch_out),
                        "h2d": timed(("h2d",), pattern, ch_in, ch_out),
                        "d2h": timed(("d2h",), pattern, ch_in, ch_out)}
            print(key, {k: round(v["gbs_median"], 1) for k, v in res[key].items()}, flush=True)
    json.dump(res, open(out, "w"), indent=1)


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "pcie_pattern.json")
