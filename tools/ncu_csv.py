"""Summarise an `ncu --metrics ... --csv --log-file` launch list: one line
per launch (time, DRAM read/write, achieved GB/s) and per-kernel totals.

  python tools/ncu_csv.py file.csv [max_lines]
"""
import csv
import sys
from collections import OrderedDict, defaultdict


def load(path):
    lines = open(path).read().splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    k = OrderedDict()
    for r in csv.DictReader(lines[start:]):
        d = k.setdefault(r["ID"], {"name": r["Kernel Name"], "grid": r["Grid Size"], "block": r["Block Size"]})
        try:
            d[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
        except ValueError:
            d[r["Metric Name"]] = r["Metric Value"]
    return k


def main():
    k = load(sys.argv[1])
    nmax = int(sys.argv[2]) if len(sys.argv) > 2 else 30
    tot = defaultdict(lambda: [0, 0.0, 0.0])
    for i, (kid, v) in enumerate(k.items()):
        t = v.get("gpu__time_duration.sum", 0.0)
        rd, wr = v.get("dram__bytes_read.sum", 0.0), v.get("dram__bytes_write.sum", 0.0)
        name = v["name"].split("(")[0]
        tot[name][0] += 1
        tot[name][1] += t
        tot[name][2] += rd + wr
        if i < nmax:
            extra = " ".join(f"{m.split('.')[0].split('__')[-1]}={v[m]:.3g}" for m in v
                             if m not in ("name", "grid", "block", "gpu__time_duration.sum",
                                          "dram__bytes_read.sum", "dram__bytes_write.sum")
                             and isinstance(v[m], float))
            print(f"{kid:>4} {name[:32]:32} grid{v['grid']:>14} {t / 1e3:8.1f} us  rd {rd / 1e6:7.1f} MB"
                  f"  wr {wr / 1e6:7.1f} MB  {(rd + wr) / max(t, 1):6.0f} GB/s  {extra}")
    print("-- totals")
    for name, (n, t, b) in tot.items():
        print(f"{name[:40]:40} n={n:4d} {t / 1e6:8.3f} ms  {b / 1e9:7.3f} GB  {b / max(t, 1):6.0f} GB/s")


if __name__ == "__main__":
    main()
