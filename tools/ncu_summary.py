"""Summarise ncu outputs into profiles/<round>/ (tracked).

  python tools/ncu_summary.py r01 [launches.csv] [full.ncu-rep]

Writes launches_summary.json (per-kernel launch counts, summed device time
and share of the step; ncu per-launch times are cold-cache and serialised,
so only SHARES are meaningful) and <kernel>_full.json (key metrics of one
--set full capture), and updates profiles/heat7_ncu_traffic.json (dram bytes
per launch for bench.py's roofline.traffic).
"""
import csv
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    out = defaultdict(lambda: {"count": 0, "us": 0.0})
    for r in rows:
        if "Kernel Name" in r:
            hdr = r
            continue
        if not hdr or len(r) != len(hdr):
            continue
        d = dict(zip(hdr, r))
        if d.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = d["Kernel Name"].split("(")[0]
        v = float(d["Metric Value"].replace(",", ""))
        unit = d.get("Metric Unit", "ns")
        us = v / 1000 if unit == "ns" else v * 1000 if unit == "ms" else v
        out[name]["count"] += 1
        out[name]["us"] += us
    tot = sum(v["us"] for v in out.values()) or 1
    return {k: {**v, "share": v["us"] / tot} for k, v in sorted(out.items(), key=lambda kv: -kv[1]["us"])}


WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
        "launch__shared_mem_per_block_dynamic", "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active"]


def full(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    hdr, units = rows[0], rows[1]
    res = []
    for vals in rows[2:]:
        d = {"kernel": vals[hdr.index("Kernel Name")]}
        for i, h in enumerate(hdr):
            if h in WANT or (h.startswith("smsp__average_warps_issue_stalled") and h.endswith("per_issue_active.ratio")):
                try:
                    d[h] = {"value": float(vals[i].replace(",", "")), "unit": units[i]}
                except ValueError:
                    pass
        res.append(d)
    return res


if __name__ == "__main__":
    rnd = sys.argv[1]
    lpath = sys.argv[2] if len(sys.argv) > 2 else os.path.join(ROOT, "gpurun_out", "launches.csv")
    fpath = sys.argv[3] if len(sys.argv) > 3 else os.path.join(ROOT, "gpurun_out", "heat7_full.ncu-rep")
    outdir = os.path.join(ROOT, "profiles", rnd)
    os.makedirs(outdir, exist_ok=True)
    if os.path.exists(lpath):
        L = launches(lpath)
        json.dump(L, open(os.path.join(outdir, "launches_summary.json"), "w"), indent=1)
        for k, v in L.items():
            print(f"{k:60s} n={v['count']:4d} {v['us']:10.1f} us  share {v['share']*100:5.1f}%")
    if os.path.exists(fpath):
        F = full(fpath)
        tag = os.path.splitext(os.path.basename(fpath))[0]
        json.dump(F, open(os.path.join(outdir, tag + ".json"), "w"), indent=1)
        for d in F:
            g = lambda k: d.get(k, {}).get("value")
            unit = d.get("dram__bytes_read.sum", {}).get("unit", "")
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)
            traffic = (g("dram__bytes_read.sum") + g("dram__bytes_write.sum")) * scale
            print(d["kernel"][:80], "dur", g("gpu__time_duration.sum"), d["gpu__time_duration.sum"]["unit"],
                  "dram R+W bytes", traffic, "dram%", g("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"))
            if "heat7_fixed" in d["kernel"]:
                # per STEP: a persistent capture covers NCU_STEPS steps (tools/prof_heat.py STEPS)
                steps = int(os.environ.get("NCU_STEPS", "4")) if "persistent" in tag else 1
                tp = os.path.join(ROOT, "profiles", "heat7_ncu_traffic.json")
                j = json.load(open(tp)) if os.path.exists(tp) else {}
                j["c2"] = traffic / steps
                j["c2_source"] = (f"profiles/{rnd}/{tag}.json (ncu --set full, whole-domain launch of C2, "
                                  f"{steps} step(s) per launch; DRAM read + write per step)")
                json.dump(j, open(tp, "w"), indent=1)
