"""Box census: host/GPU facts and pinned PCIe bandwidth.

Writes gpurun_out/census.json. Measures the host link denominators used by the
roofline: pinned H2D, D2H and concurrent bidirectional copy.
"""
import json, os, subprocess, time
import torch

def sh(cmd):
    try:
        return subprocess.run(cmd, shell=True, capture_output=True, text=True, timeout=60).stdout
    except Exception as e:  # noqa
        return str(e)

def bw(nbytes, reps=10):
    h = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    h2 = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    d = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    d2 = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    res = {"h2d": [], "d2h": [], "bidir": []}
    for _ in range(reps):
        for k in ("h2d", "d2h"):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            if k == "h2d":
                d.copy_(h, non_blocking=True)
            else:
                h.copy_(d, non_blocking=True)
            torch.cuda.synchronize()
            res[k].append(nbytes / (time.perf_counter() - t0) / 1e9)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        with torch.cuda.stream(s1):
            d.copy_(h, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)
        torch.cuda.synchronize()
        res["bidir"].append(2 * nbytes / (time.perf_counter() - t0) / 1e9)
    return {k: {"best": max(v), "median": sorted(v)[len(v) // 2]} for k, v in res.items()}

def hbm(nbytes=4 << 30, reps=10):
    a = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    b = torch.empty_like(a)
    best = 0
    for _ in range(reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(); b.copy_(a); e1.record(); torch.cuda.synchronize()
        best = max(best, 2 * nbytes / (e0.elapsed_time(e1) / 1e3) / 1e9)
    return best

if __name__ == "__main__":
    os.makedirs("gpurun_out", exist_ok=True)
    p = torch.cuda.get_device_properties(0)
    out = {
        "gpu": p.name, "sms": p.multi_processor_count, "mem_gb": p.total_memory / 1e9,
        "l2_bytes": getattr(p, "L2_cache_size", None),
        "nproc": os.cpu_count(),
        "lscpu": sh("lscpu"), "free_g": sh("free -g"), "numactl": sh("numactl -H"),
        "ulimit_l": sh("ulimit -l"), "topo": sh("nvidia-smi topo -m"),
        "smi": sh("nvidia-smi --query-gpu=name,pcie.link.gen.max,pcie.link.gen.current,pcie.link.width.current,clocks.max.sm,driver_version --format=csv"),
        "pcie_256MiB": bw(256 << 20), "pcie_1GiB": bw(1 << 30, reps=5), "hbm_copy_gbs": hbm(),
    }
    json.dump(out, open("gpurun_out/census.json", "w"), indent=1)
    print(json.dumps({k: v for k, v in out.items() if k.startswith(("pcie", "hbm", "gpu", "nproc", "sms"))}, indent=1))
    print(out["free_g"]); print(out["smi"]); print(out["lscpu"][:1500])
