"""DRAM bytes per swept cell of the stream-through / wavefront sweep kernel,
for bench.py's roofline.traffic: ncu launch list (dram__bytes_read/write per
launch, warm L2: --cache-control none) of tools/prof_sweep.py, divided by the
cells the same run sweeps (from the dry-run trace of the identical
configuration, sweep_link_ratio fixed at 0.021 in both).

  python tools/sweep_traffic.py launches.csv SCHED T out.json [KERNEL]

KERNEL: slab_sweep (default: the single-level sweeps, trace ops sweep /
sweep_u / wsweep) or heat2_band_slab (the two-level passes, trace op wsweep2:
cells = the pass's level-s planes, each read and written once per pass).
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from tools.ncu_csv import load  # noqa: E402

from paper_conf_icpp_bastemuzas17_b200 import tiles as T  # noqa: E402
from tests.replay import wsweep_range  # noqa: E402


def main():
    csv_path, sched, steps, out = sys.argv[1], sys.argv[2], int(sys.argv[3]), sys.argv[4]
    kern = sys.argv[5] if len(sys.argv) > 5 else "slab_sweep"
    ops1 = ("wsweep2", "sweep2s") if kern == "heat2_band_slab" else ("sweep", "sweep_u", "wsweep")
    k = load(csv_path)
    rd = wr = 0.0
    n = 0
    for v in k.values():
        if kern not in v["name"]:
            continue
        rd += v.get("dram__bytes_read.sum", 0.0)
        wr += v.get("dram__bytes_write.sum", 0.0)
        n += 1
    kw = {"wavefront": 1} if sched == "wave" else {"stream_through": 1, "wavefront": -1}
    d = T.Domain((512, 512, 512), (64, 64, 64), dry_run=True, sweep_link_ratio=0.021, **kw)
    d.invalidate()
    d.run(T.heat7(), steps, 4)
    cells, launches = 0, 0
    for op in d.trace():
        if op[0] not in ops1:
            continue
        if op[0] in ("sweep", "sweep_u", "sweep2s"):
            lo, hi = op[4] & 0xffffffff, op[4] >> 32
        else:
            lo, hi = wsweep_range(op[4])
        cells += (hi - lo) * 512 * 512
        launches += 1
    # ncu reports MB for bytes in the csv loader's units? the loader keeps raw values (bytes)
    res = {"kernel": "heat2_band_slab" if kern == "heat2_band_slab" else "slab_sweep_tile", "schedule": sched, "T": steps, "launches_ncu": n, "launches_trace": launches,
           "dram_read_bytes": rd, "dram_write_bytes": wr, "cells_swept": cells,
           "dram_bytes_per_cell": (rd + wr) / cells if cells and n == launches else None,
           "algorithmic_bytes_per_cell": 16.0,
           "source": f"ncu --cache-control none launch list of tools/prof_sweep.py (SCHED={sched}, T={steps}) "
                     f"on the pool's B200; cells from the dry-run trace of the same configuration"}
    json.dump(res, open(out, "w"), indent=1)
    print(json.dumps(res))


if __name__ == "__main__":
    main()
