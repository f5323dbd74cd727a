"""Benchmark of the tiled heat path.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl tiles|reference]
                    [--config c2|c1|c3|c4|c5|fig5|fig5tiles|fig8] [--T STEPS] [--nstreams S]

One bench "step" = one pass of the whole hot path over one batch of input:
T heat steps over every tile of the workload (C2 by default: 512^3 fp64,
8^3 tiles of 64^3, ghost 1, 4 streams, T = 10, periodic, alpha = 0.125),
with every cell's H2D and D2H inside the step.

  value  the metric as BASELINE.json defines it: Gcell-updates/s INCLUDING
         H2D/D2H, through the public C API from the library's pinned host
         store: tile_invalidate -> tile_run(T) -> tile_sync (H2D of every
         tile, T steps, D2H of every tile inside the timed region). `e2e`
         repeats this measurement with its byte counts.
  resident  the same T steps with the grid already resident in HBM (the
         kernel-level rate; its roofline is the heat7 kernel's).
  roofline  the dominant kernel of the timed step (the stream-through sweep
         at T <= 16; heat7 when the batched schedule runs), achieved HBM
         bytes from per-launch CUDA events on the launching streams.

Timing: CUDA events recorded by libtiles on its own streams (tile_timer_*),
barrier + synchronize on both sides, max over ranks. Inputs (2 x 1.07 GB per
GPU) are larger than the 126 MB L2. N > 1: one process per GPU (bench.py
re-launches itself under torch.distributed.run when WORLD_SIZE is unset),
weak scaling, each rank owns a 512^3 z-slab of a 512 x 512 x 512N grid,
halos over CUDA IPC peer memory (default) or NCCL.
"""
import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CONFIGS = {
    # name: (per-GPU dims, tile dims, T, nstreams, description)
    "c1": ((64, 64, 64), (32, 32, 32), 10, 2, "C1 heat fp64 64^3, 2x2x2 tiles, g=1, T=10, 2 streams"),
    "c2": ((512, 512, 512), (64, 64, 64), 10, 4,
           "C2 heat fp64 512^3, 8^3 tiles (64^3 cells), g=1, T=10, 4 streams; every cell's H2D and D2H "
           "inside the step (fresh upload from the pinned host store)"),
}
ALPHA = 0.125
METRIC = "Gcell-updates/s incl. H2D/D2H at 1/2/4/8 B200; % transfer time hidden"


# Test hook: TILES_BENCH_ONE_GPU=1 runs every rank of a torchrun launch on
# cuda:0 with a gloo process group (exercises the multi-rank bench path and
# the peer transport on a one-GPU box; never used for reported numbers).
ONE_GPU = os.environ.get("TILES_BENCH_ONE_GPU") == "1"


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rk = int(os.environ.get("RANK", "0"))
    lr = int(os.environ.get("LOCAL_RANK", str(rk)))
    return ws, rk, (0 if ONE_GPU else lr)


def init_dist(torch, dist, lr):
    if ONE_GPU:
        dist.init_process_group("gloo")
    else:
        dist.init_process_group("nccl", device_id=torch.device("cuda", lr))


def bind_numa(torch, dev):
    """Pin this process to the CPUs local to its GPU's PCIe root (sysfs
    local_cpulist) before any pinned host memory is allocated, so the host
    tile store and its DMA stay on the GPU's NUMA node (one process per GPU
    on a multi-socket box). Returns the CPU list used, or None (no-op)."""
    try:
        p = torch.cuda.get_device_properties(dev)
        path = f"/sys/bus/pci/devices/{p.pci_domain_id:04x}:{p.pci_bus_id:02x}:{p.pci_device_id:02x}.0/local_cpulist"
        spec = open(path).read().strip()
        cpus = set()
        for part in spec.split(","):
            a, _, b = part.partition("-")
            cpus.update(range(int(a), int(b or a) + 1))
        cur = os.sched_getaffinity(0)
        cpus &= cur
        if cpus and cpus != cur:
            os.sched_setaffinity(0, cpus)
        return spec
    except Exception:  # no sysfs entry (VM, container): leave the affinity alone
        return None


def red_dev():
    return "cpu" if ONE_GPU else "cuda"


class Clocks:
    """Clock / throttle-reason sampler for the timed region (B200_PROFILING.md
    clocks line): NVML polled every ~2 ms from a thread (a C2 value leg lasts
    ~80 ms, too short for nvidia-smi's 100 ms loop); nvidia-smi if NVML is
    unavailable."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")
    NAMES = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]

    def __init__(self, gpu):
        self.gpu, self.rows, self.p, self.nv, self.stop = gpu, [], None, None, False

    def __enter__(self):
        try:
            import pynvml as nv
            nv.nvmlInit()
            h = nv.nvmlDeviceGetHandleByIndex(self.gpu)
            self.nv = nv
            self.maxc = nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM)
            bits = [nv.nvmlClocksEventReasonHwSlowdown, nv.nvmlClocksEventReasonHwThermalSlowdown,
                    nv.nvmlClocksEventReasonSwThermalSlowdown, nv.nvmlClocksEventReasonSwPowerCap]

            def poll():
                while not self.stop:
                    try:
                        sm = nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)
                        rs = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                        self.rows.append([str(sm), str(self.maxc), "", *["Active" if rs & b else "Not Active"
                                                                       for b in bits]])
                    except Exception:
                        pass
                    time.sleep(0.002)
            self.t = threading.Thread(target=poll, daemon=True)
            self.t.start()
            return self
        except Exception:
            self.nv = None
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.Q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.p = None
        return self

    def _read(self):
        for line in self.p.stdout:
            parts = [x.strip() for x in line.split(",")]
            if len(parts) == 7:
                self.rows.append(parts)

    def __exit__(self, *a):
        self.stop = True
        if self.nv is not None:
            self.t.join(1)
        if self.p:
            self.p.terminate()
            try:
                self.p.wait(2)
            except Exception:
                self.p.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = sorted(float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit())
        reasons = set()
        for r in self.rows:
            for n, v in zip(self.NAMES, r[3:]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": sm[len(sm) // 2] if sm else None,
                "sm_max_mhz": float(self.rows[0][1]) if self.rows[0][1].replace(".", "").isdigit() else None,
                "reasons": sorted(reasons), "samples": len(self.rows),
                "source": "nvml" if self.nv is not None else "nvidia-smi"}


def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        j = json.load(open(p))
        return float(j["hbm_gbs"]), "MEASURED_PEAKS.json hbm_gbs (measured)"
    return 6650.0, "B200_PROFILING.md fallback 6.65 TB/s"


def pcie_bandwidth(torch, nbytes=1 << 30, reps=8, warm=2):
    """Pinned single-direction link rates (GB/s): best of `reps` 1 GiB copies
    after `warm` untimed ones (a fresh pinned buffer's first DMAs run slower
    on these VMs), CUDA events on the copy stream."""
    h = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    d = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    out = {}
    for k in ("h2d", "d2h"):
        best = 0
        for i in range(warm + reps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            d.copy_(h, non_blocking=True) if k == "h2d" else h.copy_(d, non_blocking=True)
            e1.record()
            torch.cuda.synchronize()
            if i >= warm:
                best = max(best, nbytes / (e0.elapsed_time(e1) / 1e3) / 1e9)
        out[k] = best
    return out


def traffic_from_profile(cfg):
    p = os.path.join(ROOT, "profiles", "heat7_ncu_traffic.json")
    if os.path.exists(p):
        j = json.load(open(p))
        return j.get(cfg)
    return None


def traffic_per_cell(kernel):
    """ncu DRAM bytes per swept cell of `kernel` from a committed capture
    (profiles/<kernel>_ncu_traffic.json), with its source; None if absent."""
    p = os.path.join(ROOT, "profiles", f"{kernel}_ncu_traffic.json")
    if os.path.exists(p):
        j = json.load(open(p))
        return j["dram_bytes_per_cell"], j.get("source", p)
    return None


def host_cores():
    try:
        return len(os.sched_getaffinity(0))
    except Exception:
        return os.cpu_count() or 1


def cpu_oracle_time(n, T, threads=1):
    """Seconds for T untiled oracle steps on an n^3 sample (the C oracle;
    threads > 1: its bit-identical OpenMP twin)."""
    import oracle
    import synth
    u = np.empty((n, n, n))
    synth.fill_uniform_native(u.ctypes.data, n, n, n, 0, n, 0, n, 0, n, 42)
    t0 = time.perf_counter()
    oracle.heat_c(u, ALPHA, T, threads=threads)
    return time.perf_counter() - t0


def cpu_baseline(T, n1=384, nall=512):
    """The oracle on the host cores: 1 thread on an n1^3 sample and all cores
    (OpenMP twin) on an nall^3 sample, T steps each (~10-20 s together)."""
    cores = host_cores()
    t1 = cpu_oracle_time(n1, T, 1)
    ta = cpu_oracle_time(nall, T, cores)
    v1, va = n1 ** 3 * T / t1 / 1e9, nall ** 3 * T / ta / 1e9
    return {"value": va, "unit": "Gcell-updates/s", "cores": cores, "kind": "oracle",
            "sample": f"{nall}^3 grid x T={T} on {cores} threads (oracle/heat_oracle.c OpenMP twin, "
                      f"bit-identical); 1 thread: {n1}^3 x T={T}",
            "by_cores": {"1": v1, str(cores): va}}


def run_reference(args):
    """--impl reference: the CPU oracle as it stands on the host's cores (the
    OpenMP twin of the untiled C oracle, bit-identical to it), one bounded
    sample of the workload per step. Under torchrun only rank 0 runs."""
    ws, rk, _ = dist_env()
    if rk != 0:
        return 0
    dims, td, T, ns, desc = CONFIGS.get(args.config, CONFIGS["c2"])
    cores = host_cores()
    n = 320 if args.config != "c1" else dims[0]   # bounded sample per step
    for _ in range(args.warmup):
        cpu_oracle_time(n, T, cores)
    t = sum(cpu_oracle_time(n, T, cores) for _ in range(args.steps))
    val = n ** 3 * T * args.steps / t / 1e9
    sample = f"{n}^3 grid x T={T} per step (untiled fp64 Jacobi, oracle/heat_oracle.c OpenMP twin, {cores} threads)"
    line = {"impl": "reference", "metric": METRIC, "value": val, "unit": "Gcell-updates/s", "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": t / args.steps * 1e3,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": {"workload": desc, "sample": sample},
            "cpu_baseline": {"value": val, "unit": "Gcell-updates/s", "cores": cores, "kind": "oracle",
                             "sample": sample},
            "e2e": {"value": val, "unit": "Gcell-updates/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ---------------------------------------------------------------- CUPTI
def _union(iv):
    out = []
    for a, b in sorted(iv):
        if out and a <= out[-1][1]:
            out[-1][1] = max(out[-1][1], b)
        else:
            out.append([a, b])
    return out


def _inter(a, b):
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


def cupti_overlap(torch, fn):
    """Run fn() once under torch.profiler (CUPTI activity records of every
    kernel and memcpy in the process, libtiles' included) and return the
    interval statistics: busy times, Σ(copy ∩ kernel) / min(Σcopy, Σkernel)
    (SURVEY §8(d) cross-check of the overlap metric) and H2D ∥ D2H."""
    import tempfile
    from torch.profiler import ProfilerActivity, profile
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        fn()
        torch.cuda.synchronize()
    with tempfile.NamedTemporaryFile(suffix=".json", delete=False) as f:
        path = f.name
    try:
        prof.export_chrome_trace(path)
        ev = json.load(open(path))["traceEvents"]
    finally:
        os.unlink(path)
    ker, h2d, d2h = [], [], []
    for e in ev:
        if e.get("ph") != "X" or "dur" not in e:
            continue
        iv = (e["ts"], e["ts"] + e["dur"])
        cat, name = e.get("cat", ""), e.get("name", "")
        if cat == "kernel":
            ker.append(iv)
        elif cat in ("gpu_memcpy", "memcpy") or "Memcpy" in name:
            if "HtoD" in name:
                h2d.append(iv)
            elif "DtoH" in name:
                d2h.append(iv)
    if not ker or not (h2d or d2h):
        return None
    K, H, D = _union(ker), _union(h2d), _union(d2h)
    X = _union(h2d + d2h)
    busy = lambda s_: sum(b - a for a, b in s_)
    allv = ker + h2d + d2h
    span = max(x[1] for x in allv) - min(x[0] for x in allv)
    return {"span_ms": span / 1e3, "kernel_busy_ms": busy(K) / 1e3, "h2d_busy_ms": busy(H) / 1e3,
            "d2h_busy_ms": busy(D) / 1e3, "copy_busy_ms": busy(X) / 1e3,
            "copy_and_kernel_ms": _inter(X, K) / 1e3, "h2d_and_d2h_ms": _inter(H, D) / 1e3,
            "hidden_frac": _inter(X, K) / max(1e-9, min(busy(X), busy(K))),
            "n_kernels": len(ker), "n_h2d": len(h2d), "n_d2h": len(d2h),
            "definition": "CUPTI activity intervals: sum(copy ∩ kernel) / min(sum copy, sum kernel)"}


def fill_tiles(dom, Tl, synth, gdims, td, z_base, seed):
    """Write the generator's values straight into the pinned tile store."""
    info = dom.info
    ntx, nty, ntz = info["tiles"]
    for k in range(info["ntiles"]):
        ix, iy, iz = k % ntx, (k // ntx) % nty, k // (ntx * nty)
        v = dom.host_tile(k)
        synth.fill_uniform_native(v.ctypes.data, gdims[0], gdims[1], gdims[2], z_base + iz * td[2], td[2],
                                  iy * td[1], td[1], ix * td[0], td[0], seed)
    dom.mark_host_dirty()


def c3_line(args):
    """C3: heat 2048^3 fp64 out-of-core: the device budget is CAPPED (the
    paper's "limiting GPU memory" method) so only a fraction of the
    tiles fits; every step streams the tiles through the slot pool.
    value = e2e: tile_invalidate + tile_run(T) + tile_sync from pinned host."""
    import torch
    from paper_conf_icpp_bastemuzas17_b200 import tiles as Tl
    import synth
    n = args.n or 2048
    td = (256, 256, 256) if n % 256 == 0 else (n // 8, n // 8, n // 8)
    T = args.T if args.T is not None else 10
    ns = args.nstreams or 4
    budget = int((args.budget_gb or 12.0) * (1 << 30))
    gdims = (n, n, n)
    cells = n ** 3
    torch.cuda.set_device(0)
    t0 = time.perf_counter()
    dom = Tl.Domain(gdims, td, ghost=args.ghost, device=0, sched="stream", device_budget_bytes=budget,
                    stream_through=args.stream_through)
    t_alloc = time.perf_counter() - t0
    t0 = time.perf_counter()
    fill_tiles(dom, Tl, synth, gdims, td, 0, 42)
    t_fill = time.perf_counter() - t0
    k = Tl.heat7(ALPHA)
    for _ in range(args.warmup):
        dom.invalidate()
        dom.run(k, T, ns)
        dom.sync()
    dom.reset_stats()
    torch.cuda.synchronize()
    tot = 0.0
    with Clocks(0) as clk:
        for _ in range(args.steps):
            dom.invalidate()
            dom.timer_start()
            dom.run(k, T, ns)
            dom.sync()
            tot += dom.timer_stop()
    st = dom.stats()
    val = cells * T * args.steps / (tot / 1e3) / 1e9
    info = dom.info
    Bh_ = st["bytes_h2d"] / args.steps
    # overlap: same schedule, transfers only / kernels only
    def leg(mode, steps=1):
        dom.set_measure(mode)
        t = 0.0
        for _ in range(steps):
            dom.invalidate()
            dom.timer_start()
            dom.run(k, T, ns)
            dom.sync()
            t += dom.timer_stop()
        dom.set_measure(Tl.TILE_MEASURE_NORMAL)
        return t / steps
    xo, co = leg(Tl.TILE_MEASURE_XFER_ONLY, args.steps), leg(Tl.TILE_MEASURE_COMP_ONLY, args.steps)
    wall = tot / args.steps
    hidden = (xo + co - wall) / min(xo, co)   # unclamped; same repetitions as the wall time
    dom.free()
    bw = pcie_bandwidth(torch)
    bidir = pcie_bidir(torch)
    Bh, Bd = st["bytes_h2d"] / args.steps, st["bytes_d2h"] / args.steps
    t_link = max(Bh / (bw["h2d"] * 1e9), Bd / (bw["d2h"] * 1e9), (Bh + Bd) / (bidir * 1e9))
    line = {"metric": METRIC, "value": val, "unit": "Gcell-updates/s", "n_gpus": 1, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": wall, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"C3 heat fp64 {n}^3 out-of-core (device budget capped at "
                                   f"{budget / 2**30:.1f} GiB, paper method P:L232), T={T}, ghost={args.ghost}",
                       "ghost": args.ghost, "steps_per_pass": info["steps_per_pass"],
                       "link_passes_per_run": Bh_ / (cells * 8),
                       "stream_through": args.stream_through,
                       "dims": gdims, "tile_dims": td, "T": T, "nstreams": ns, "nslots": info["nslots"],
                       "ntiles": info["ntiles"], "host_gb": info["host_bytes"] / 1e9,
                       "device_gb": info["device_bytes"] / 1e9,
                       "value_def": "e2e streaming: invalidate + tile_run(T) + tile_sync from pinned host",
                       "setup_s": {"pinned_alloc": t_alloc, "generate": t_fill}},
            "e2e": {"value": val, "unit": "Gcell-updates/s", "h2d_bytes_per_step": int(Bh),
                    "d2h_bytes_per_step": int(Bd), "ms_per_step": wall},
            "gpu_launches": st["n_kernels"] // max(1, args.steps),
            "residency": {k2: st[k2] // args.steps for k2 in ("hits", "misses", "evictions", "writebacks")},
            "overlap": {"hidden_frac": hidden, "t_wall_ms": wall, "t_xfer_only_ms": xo, "t_comp_only_ms": co,
                        "reps": args.steps},
            "roofline": {"bound": "pcie", "form": "streaming: max(Bh/BWh, Bd/BWd, (Bh+Bd)/BWbidir)",
                         "t_link_ms": t_link * 1e3, "frac": t_link * 1e3 / wall,
                         "achieved": (Bh + Bd) / (wall / 1e3) / 1e9, "peak": bidir, "unit": "GB/s",
                         "pcie_gbs": {**bw, "bidir": bidir}},
            "clocks": clk.summary()}
    return line


def pcie_bidir(torch, nbytes=1 << 30, reps=6, warm=2):
    """Both directions at once (H2D and D2H of 1 GiB each on two streams):
    (bytes H2D + bytes D2H) / span, span from CUDA events (start on the
    current stream, both copy streams wait on it, end = the later stream)."""
    h1 = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    h2 = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    d1 = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    d2 = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    best = 0
    for i in range(warm + reps):
        torch.cuda.synchronize()
        e0 = torch.cuda.Event(enable_timing=True)
        e0.record()
        ends = []
        for s_, dst, src in ((s1, d1, h1), (s2, h2, d2)):
            s_.wait_event(e0)
            with torch.cuda.stream(s_):
                dst.copy_(src, non_blocking=True)
                e = torch.cuda.Event(enable_timing=True)
                e.record(s_)
                ends.append(e)
        torch.cuda.synchronize()
        if i >= warm:
            span = max(e0.elapsed_time(e) for e in ends)
            best = max(best, 2 * nbytes / (span / 1e3) / 1e9)
    return best


def c4_line(args):
    """C4: the compute-intensive kernel at 1024^3 fp64, 8^3
    tiles of 128^3, K = 32 inner iterations (reading R12), T = 10 outer steps
    fused per residency pass; nstreams sweep 1..8 (e2e from pinned host)."""
    import torch
    from paper_conf_icpp_bastemuzas17_b200 import tiles as Tl
    import synth
    n = args.n or 1024
    td = (n // 8, n // 8, n // 8)
    T = args.T if args.T is not None else 10
    K = args.K
    gdims = (n, n, n)
    cells = n ** 3
    torch.cuda.set_device(0)
    dom = Tl.Domain(gdims, td, ghost=1, device=0)
    fill_tiles(dom, Tl, synth, gdims, td, 0, 7)
    k = Tl.sincos(K)
    sweep = {}
    for ns in ([int(v) for v in args.sweep.split(",")] if args.sweep else [1, 2, 4, 8]):
        for _ in range(max(1, args.warmup)):
            dom.invalidate()
            dom.run(k, T, ns)
            dom.sync()
        tot = 0.0
        for _ in range(args.steps):
            dom.invalidate()
            dom.timer_start()
            dom.run(k, T, ns)
            dom.sync()
            tot += dom.timer_stop()
        sweep[ns] = cells * T * args.steps / (tot / 1e3) / 1e9
    ns_best = max(sweep, key=sweep.get)
    ns = args.nstreams or 4
    # resident (compute only) with kernel timing, and the overlap legs
    dom.invalidate()
    dom.run(k, T, ns)
    dom.sync()
    dom.set_kernel_timing(True)
    dom.reset_stats()
    with Clocks(0) as clk:
        dom.timer_start()
        for _ in range(args.steps):
            dom.run(k, T, ns)
        ms_res = dom.timer_stop()
    st = dom.stats()
    dom.set_kernel_timing(False)
    dom.sync()
    def leg(mode, reps):
        dom.set_measure(mode)
        t = 0.0
        for _ in range(reps):
            dom.invalidate()
            dom.timer_start()
            dom.run(k, T, ns)
            dom.sync()
            t += dom.timer_stop()
        dom.set_measure(Tl.TILE_MEASURE_NORMAL)
        return t / reps
    wall = leg(Tl.TILE_MEASURE_NORMAL, args.steps)
    xo, co = leg(Tl.TILE_MEASURE_XFER_ONLY, args.steps), leg(Tl.TILE_MEASURE_COMP_ONLY, args.steps)
    hidden = (xo + co - wall) / min(xo, co)   # unclamped, equal repetitions
    dom.free()
    value = cells * T * args.steps / (ms_res / 1e3) / 1e9
    # achieved over the resident wall time (per-launch event durations of
    # concurrent streams overlap, so their sum is not a time)
    iters_per_s = cells * K * T * args.steps / (ms_res / 1e3)
    prof = os.path.join(ROOT, "profiles", "sincos_fp64.json")
    roof = {"bound": "alu", "achieved": iters_per_s / 1e9, "unit": "Gcell-iter/s", "peak": None, "frac": None,
            "traffic": None, "kernel": "sincos_iter"}
    if os.path.exists(prof):
        pj = json.load(open(prof))
        peak = pj["dp_inst_per_s"] / pj["dp_inst_per_cell_iter"] / 1e9
        roof.update({"peak": peak, "frac": roof["achieved"] / peak, "peak_source": pj.get("source")})
    line = {"metric": METRIC, "value": value, "unit": "Gcell-steps/s", "n_gpus": 1, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_res / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"C4 compute-intensive kernel (P:L219-L224) {n}^3 fp64, tiles {td}, "
                                   f"K={K} inner iterations, T={T} outer steps fused per residency pass",
                       "nstreams": ns, "value_def": "grid resident; unit = one outer step (K iterations) of one cell"},
            "e2e": {"value": sweep.get(ns), "unit": "Gcell-steps/s", "h2d_bytes_per_step": cells * 8,
                    "d2h_bytes_per_step": cells * 8},
            "stream_sweep_e2e": sweep, "best_nstreams": ns_best,
            "overlap": {"hidden_frac": hidden, "t_wall_ms": wall, "t_xfer_only_ms": xo, "t_comp_only_ms": co,
                        "reps": args.steps},
            "gpu_launches": st["n_kernels"], "roofline": roof, "clocks": clk.summary()}
    return line


def budget_for_slots(Tl, dims, td, nslots, **kw):
    """Smallest device budget giving `nslots` tile slots (dry-run plan)."""
    lo, hi = 1, 1 << 42
    while lo < hi:
        mid = (lo + hi) // 2
        try:
            n = Tl.Domain(dims, td, dry_run=True, device_budget_bytes=mid, **kw).info["nslots"]
        except Tl.TileError:
            n = -1
        lo, hi = (lo, mid) if n >= nslots else (mid + 1, hi)
    return lo


def run_fig8_leg(args):
    """NEXT #1 (Fig. 8): the compute-intensive kernel at 512^3,
    GPU memory limited to two regions vs unlimited vs one region, step-major
    (every step visits every region, as the paper's time loop does). Also the
    limited case with tile-major fusion (each region streamed once for all
    steps) — a schedule the pointwise kernel allows. Swept over K (--sweep,
    default 32 and 256): the paper tuned K so the kernel outweighs the
    transfers; on B200 that needs K ~ 256 for a step-major pass."""
    import torch
    from paper_conf_icpp_bastemuzas17_b200 import tiles as Tl
    import synth
    n = args.n or 512
    T = args.T if args.T is not None else 100
    Ks = [int(v) for v in (args.sweep or f"{args.K},{8 * args.K}").split(",")]
    ns = args.nstreams or 2
    gdims = (n, n, n)
    cells = n ** 3
    regions = (n, n, n // 16)  # 16 regions (z-slabs), the paper's region count at 512^3
    torch.cuda.set_device(0)
    variants = {
        "unlimited_16_regions": dict(td=regions, kw=dict(fuse_pointwise_steps=False)),
        "limited_2_regions": dict(td=regions, kw=dict(sched="stream", fuse_pointwise_steps=False,
                                                       device_budget_bytes=budget_for_slots(
                                                           Tl, gdims, regions, 2, sched="stream"))),
        "one_region": dict(td=gdims, kw=dict(fuse_pointwise_steps=False)),
        "limited_2_regions_tile_major": dict(td=regions, kw=dict(sched="stream", fuse_pointwise_steps=True,
                                                                  device_budget_bytes=budget_for_slots(
                                                                      Tl, gdims, regions, 2, sched="stream"))),
    }
    out = {}
    for K in Ks:
        res = {}
        for name, v in variants.items():
            dom = Tl.Domain(gdims, v["td"], ghost=1, device=0, **v["kw"])
            fill_tiles(dom, Tl, synth, gdims, v["td"], 0, 7)
            k = Tl.sincos(K)
            dom.run(k, 1, ns)
            dom.sync()
            dom.invalidate()
            dom.reset_stats()
            dom.timer_start()
            dom.run(k, T, ns)
            dom.sync()
            ms = dom.timer_stop()
            st = dom.stats()
            res[name] = {"ms": ms, "gcell_steps_per_s": cells * T / (ms / 1e3) / 1e9,
                         "nslots": dom.info["nslots"], "h2d_gb": st["bytes_h2d"] / 1e9,
                         "d2h_gb": st["bytes_d2h"] / 1e9, "launches": st["n_kernels"]}
            dom.free()
        base = res["unlimited_16_regions"]["ms"]
        for r in res.values():
            r["time_vs_unlimited"] = r["ms"] / base
        out[str(K)] = res
    line = {"metric": "time, compute-intensive kernel, limited vs unlimited GPU memory (Fig. 8 analogue)",
            "value": out[str(Ks[-1])]["limited_2_regions"]["time_vs_unlimited"], "unit": "x unlimited time",
            "higher_is_better": False, "n_gpus": 1, "steps": 1, "warmup": 1, "dtype": "f64",
            "data": "synthetic", "vs_baseline": None, "scaling": "weak",
            "config": {"workload": f"Fig. 8: sincos kernel {n}^3, K in {Ks} (value at K={Ks[-1]}), "
                                   f"T={T} outer steps, 16 regions, {ns} streams", "regions": regions},
            "variants_by_K": out}
    print(json.dumps(line), flush=True)
    return 0


def run_fig5_leg(args):
    """Fig. 5 analogue: C2 heat 512^3, e2e incl. H2D/D2H for
    T in {1, 10, 100, 1000}: the tiled 4-stream schedule vs the synchronous
    one-stream schedule (H2D all, T steps, D2H all), same kernels."""
    import torch
    from paper_conf_icpp_bastemuzas17_b200 import tiles as Tl
    import synth
    n = args.n or 512
    td = (64, 64, 64)
    gdims = (n, n, n)
    cells = n ** 3
    Ts = [int(v) for v in (args.sweep or "1,10,32,48,64,100,1000").split(",")]
    torch.cuda.set_device(0)
    out = {}
    for sched, ns, pageable in (("auto", args.nstreams or 4, False), ("sync", 1, False),
                                ("sync_pageable", 1, True)):
        dom = Tl.Domain(gdims, td, ghost=1, device=0, sched=sched.split("_")[0], pageable_host=pageable,
                        stream_through=args.stream_through if sched == "auto" else 0,
                        wavefront=args.wavefront if sched == "auto" else -1)
        fill_tiles(dom, Tl, synth, gdims, td, 0, 42)
        k = Tl.heat7(ALPHA)
        for T in Ts:
            reps = 3 if T <= 10 else 1
            dom.invalidate()
            dom.run(k, T, ns)   # warm-up at the same T (schedule, scratch)
            dom.sync()
            best = 1e30
            for _ in range(reps):
                dom.invalidate()
                dom.timer_start()
                dom.run(k, T, ns)
                dom.sync()
                best = min(best, dom.timer_stop())
            out.setdefault(str(T), {})[sched if sched.startswith("sync") else "tiled"] = {
                "ms": best, "gcell_per_s": cells * T / (best / 1e3) / 1e9,
                "schedule": SCHED_NAMES.get(dom.get_info()["last_schedule"])}
        dom.free()
    bw = pcie_bandwidth(torch)
    bidir = pcie_bidir(torch)
    hbm, _ = measured_peaks()
    for T, r in out.items():
        r["speedup_tiled_vs_sync"] = r["sync"]["ms"] / r["tiled"]["ms"]
        r["speedup_tiled_vs_sync_pageable"] = r["sync_pageable"]["ms"] / r["tiled"]["ms"]
        r["speedup_sync_vs_sync_pageable"] = r["sync_pageable"]["ms"] / r["sync"]["ms"]
        t_dep = cells * 8 / (bw["h2d"] * 1e9) + cells * 8 / (bw["d2h"] * 1e9)
        t_duplex = max(cells * 8 / (bw["h2d"] * 1e9), cells * 8 / (bw["d2h"] * 1e9), 2 * cells * 8 / (bidir * 1e9))
        # HBM at the schedule's algorithmic bytes: 8 B per cell-step where two
        # steps run per pass (heat2_band / heat2_band_slab, grids 512 wide),
        # else 16 B (the one-step figure is reported beside it)
        two_level = n == 512 and td[0] == 64 and int(T) >= 2
        t_hbm1 = int(T) * 16 * cells / (hbm * 1e9)
        t_hbm = t_hbm1 / 2 if two_level else t_hbm1
        # a cell after T steps depends on the initial planes within T of it, so
        # no schedule returns a final plane before 2T+1 planes have crossed
        # H2D (solo rate), and the whole grid must then still cross D2H
        plane_b = cells * 8 / n
        t_cone = min(2 * int(T) + 1, n) * plane_b / (bw["h2d"] * 1e9)
        t_causal = t_cone + cells * 8 / (bw["d2h"] * 1e9)
        r["roofline_ms"] = {"t_link_dependency": t_dep * 1e3, "t_link_duplex": t_duplex * 1e3,
                            "t_hbm": t_hbm * 1e3, "t_hbm_one_step_per_pass": t_hbm1 * 1e3,
                            "hbm_bytes_per_cell_step": 8 if two_level else 16,
                            "bound_ms": max(t_duplex, t_hbm) * 1e3,
                            "t_cone_then_d2h": t_causal * 1e3,
                            "bound_causal_ms": max(t_duplex, t_hbm, t_causal) * 1e3,
                            "serial_ms": (t_dep + t_hbm) * 1e3}
        r["tiled_frac_of_bound"] = max(t_duplex, t_hbm) * 1e3 / r["tiled"]["ms"]
        r["tiled_frac_of_causal_bound"] = max(t_duplex, t_hbm, t_causal) * 1e3 / r["tiled"]["ms"]
    line = {"metric": "Gcell-updates/s incl. H2D/D2H, tiled vs synchronous (Fig. 5 analogue)",
            "value": out[str(Ts[0])]["speedup_tiled_vs_sync"], "unit": "x speedup at first T",
            "higher_is_better": True, "n_gpus": 1, "dtype": "f64", "data": "synthetic",
            "config": {"workload": f"C2 heat {n}^3, tiles {td}, T sweep {Ts}"}, "sweep": out,
            "pcie_gbs": {**bw, "bidir": bidir}}
    print(json.dumps(line), flush=True)
    return 0


def run_fig5_tiles_leg(args):
    """Region-count sweep of the Fig. 5 analogue (the paper's best was
    16 regions at 512^3): C2 heat e2e (H2D + T steps + D2H) with the default
    schedule for several tile shapes."""
    import torch
    from paper_conf_icpp_bastemuzas17_b200 import tiles as Tl
    import synth
    n = args.n or 512
    gdims = (n, n, n)
    cells = n ** 3
    Ts = [int(v) for v in (args.sweep or "1,10,100").split(",")]
    shapes = [(n, n, n // 16), (n, n // 2, n // 8), (n // 2, n // 2, n // 4), (n // 4, n // 4, n // 4),
              (n // 8, n // 8, n // 8), (n // 16, n // 16, n // 16)]
    torch.cuda.set_device(0)
    out = {}
    k = Tl.heat7(ALPHA)
    ns = args.nstreams or 4
    for td in shapes:
        dom = Tl.Domain(gdims, td, ghost=1, device=0)
        fill_tiles(dom, Tl, synth, gdims, td, 0, 42)
        key = f"{n // td[0] * (n // td[1]) * (n // td[2])} tiles of {td}"
        for T in Ts:
            dom.invalidate(); dom.run(k, min(T, 10), ns); dom.sync()
            best = 1e30
            for _ in range(3 if T <= 10 else 1):
                dom.invalidate()
                dom.timer_start()
                dom.run(k, T, ns)
                dom.sync()
                best = min(best, dom.timer_stop())
            out.setdefault(key, {})[str(T)] = {"ms": best, "gcell_per_s": cells * T / (best / 1e3) / 1e9}
        dom.free()
    line = {"metric": "Gcell-updates/s incl. H2D/D2H vs region count (Fig. 5 analogue)", "value": None,
            "unit": "Gcell-updates/s", "higher_is_better": True, "n_gpus": 1, "dtype": "f64",
            "data": "synthetic", "config": {"workload": f"C2 heat {n}^3, T sweep {Ts}, tile sweep"},
            "sweep": out}
    print(json.dumps(line), flush=True)
    return 0


def multi_domain(Tl, dist, ws, rk, transport, *args, **kw):
    """Domain for rank rk of ws. transport "peer": halo windows over CUDA IPC
    (handles all-gathered through torch.distributed), the stencil kernel of
    resident steps storing its slab-end layers straight into the neighbours'
    windows (fused, tile_options.peer_transport = 2); "peer-copy": the same
    windows filled by copy-engine pushes after each step (1); "nccl": NCCL p2p."""
    if ws == 1:
        return Tl.Domain(*args, nranks=1, rank=0, **kw)
    if transport in ("peer", "peer-copy"):
        # the IPC windows need peer access between every z-neighbour pair; if
        # any rank cannot set them up (e.g. no P2P between two GPUs of this
        # box), every rank takes the NCCL transport instead, and says so
        dom, err = None, ""
        try:
            dom = Tl.Domain(*args, nranks=ws, rank=rk, peer_transport=2 if transport == "peer" else 1, **kw)
            hs = [None] * ws
            dist.all_gather_object(hs, dom.peer_handle())
            dom.peer_connect(hs)
        except Tl.TileError as e:
            err = str(e)
        import torch
        ok = torch.tensor([0 if err else 1], dtype=torch.int32, device=red_dev())
        dist.all_reduce(ok, op=dist.ReduceOp.MIN)
        if int(ok.item()) == 1:
            return dom
        print(f"rank {rk}: peer transport unavailable ({err or 'on another rank'}); using NCCL",
              file=sys.stderr, flush=True)
        if dom is not None:
            dom.free()
        multi_domain.fallback = "nccl (peer transport setup failed)"
    obj = [Tl.nccl_unique_id() if rk == 0 else None]
    dist.broadcast_object_list(obj, src=0)
    return Tl.Domain(*args, nranks=ws, rank=rk, nccl_id=obj[0], **kw)


def run_c5_leg(args):
    """C5 line on rank 0 (c5_line)."""
    line = c5_line(args)
    if line is not None:
        print(json.dumps(line), flush=True)
    return 0


def c5_line(args):
    """C5: heat 4096^3 fp64 slab-decomposed over N GPUs (z-slabs, NCCL halo
    exchange), each rank streaming its own tiles from pinned host memory.
    With N = 1 this runs the per-GPU slab of the 8-GPU decomposition
    (4096 x 4096 x 512) alone (z-periodic), i.e. one rank's work. Returns
    the JSON line on rank 0, None on the others."""
    import torch
    import torch.distributed as dist
    from paper_conf_icpp_bastemuzas17_b200 import tiles as Tl
    import synth
    ws, rk, lr = dist_env()
    torch.cuda.set_device(lr)
    bind_numa(torch, lr)
    if ws > 1:
        init_dist(torch, dist, lr)
    n = args.n
    if not n:
        # SURVEY §8(d) fallback ladder: the largest n whose pinned host stores
        # (all ranks of this node, single array + faces) fit 0.8 x MemAvailable
        import psutil
        avail = psutil.virtual_memory().available
        nloc = int(os.environ.get("LOCAL_WORLD_SIZE", str(ws)))
        n = 2048
        for cand in (4096, 3584, 3072, 2560, 2048):
            per_rank = cand * cand * (cand // (8 if ws == 1 else ws)) * 8 * 1.05
            if per_rank * (1 if ws == 1 else nloc) <= 0.8 * avail:
                n = cand
                break
        if ws > 1:  # every rank must use the same grid
            t = torch.tensor([n], dtype=torch.int64, device=red_dev())
            dist.all_reduce(t, op=dist.ReduceOp.MIN)
            n = int(t.item())
    nzl = n // 8 if ws == 1 else n // ws
    gdims = (n, n, nzl * ws)
    # 64^3 tiles (the C2 kernel plan, one band per tile): 372.9 vs 338.3 Gcell/s
    # with 256^2 x 64 (16-row bands re-read halo rows), profiles/r01/bench_c5_tiles.json
    td = tuple(int(v) for v in args.tile.split(",")) if args.tile else (64, 64, 64)
    T = args.T if args.T is not None else 10
    ns = args.nstreams or 4
    cells = n * n * nzl

    def barrier():
        if ws > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def mx(x):
        if ws == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=red_dev())
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    t0 = time.perf_counter()
    dom = multi_domain(Tl, dist, ws, rk, args.transport, gdims, td, ghost=1, device=lr)
    fill_tiles(dom, Tl, synth, gdims, td, rk * nzl, 42)
    t_setup = time.perf_counter() - t0
    k = Tl.heat7(ALPHA)
    dom.run(k, 1, ns)
    dom.sync()
    barrier()
    dom.set_kernel_timing(True)
    dom.reset_stats()
    with Clocks(lr) as clk:
        dom.timer_start()
        for _ in range(args.steps):
            dom.run(k, T, ns)
        ms = mx(dom.timer_stop())
    st = dom.stats()
    dom.set_kernel_timing(False)
    dom.sync()
    value = ws * cells * T * args.steps / (ms / 1e3) / 1e9
    barrier()
    tot = 0.0
    dom.reset_stats()
    for _ in range(max(1, args.steps // 2)):
        dom.invalidate()
        dom.timer_start()
        dom.run(k, T, ns)
        dom.sync()
        tot += dom.timer_stop()
    tot = mx(tot)
    reps = max(1, args.steps // 2)
    st2 = dom.stats()
    info = dom.info
    dom.free()
    e2e = ws * cells * T * reps / (tot / 1e3) / 1e9
    peak, src = measured_peaks()
    avg = st["kernel_ms"] / max(1, st["kernel_timed"])
    per_launch = cells * T * args.steps / max(1, st["kernel_timed"])
    if rk == 0:
        line = {"metric": METRIC, "value": value, "unit": "Gcell-updates/s", "n_gpus": ws,
                "steps": args.steps, "warmup": 1, "ms_per_step": ms / args.steps, "higher_is_better": True,
                "scaling": "weak" if ws == 1 else "strong", "vs_baseline": None, "dtype": "f64",
                "data": "synthetic",
                "config": {"workload": f"C5 heat {n}^3 z-slabs" + (" (per-GPU slab of G=8 on 1 GPU)" if ws == 1 else f" over {ws} GPUs"),
                           "global_dims": gdims, "slab": (n, n, nzl), "tile_dims": td, "T": T, "nstreams": ns,
                           "sched": info["sched"], "nslots": info["nslots"], "setup_s": t_setup},
                "e2e": {"value": e2e, "unit": "Gcell-updates/s", "h2d_bytes_per_step": st2["bytes_h2d"] // reps,
                        "d2h_bytes_per_step": st2["bytes_d2h"] // reps, "ms_per_step": tot / reps},
                "gpu_launches": st["n_kernels"],
                "roofline": {"bound": "hbm", "achieved": 16 * per_launch / (avg / 1e3) / 1e9, "peak": peak,
                             "unit": "GB/s", "frac": 16 * per_launch / (avg / 1e3) / 1e9 / peak, "traffic": None,
                             "kernel": f"heat7_fixed (tiles {td[0]}x{td[1]}x{td[2]})", "peak_source": src},
                "halo_bytes_per_step": st["bytes_halo"] // max(1, args.steps), "clocks": clk.summary()}
    if ws > 1:
        dist.destroy_process_group()
    return line if rk == 0 else None



# ------------------------------------------------------------ multi-process
def free_port():
    import socket
    with socket.socket() as so:
        so.bind(("127.0.0.1", 0))
        return so.getsockname()[1]


def spawn_cmd(argv, n, port):
    """One process per GPU on this node, the driver's own launch line."""
    return [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
            "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *argv]


def maybe_spawn(args, argv):
    """--gpus N > 1 with no torchrun environment: re-launch this script under
    torch.distributed.run (N ranks, 127.0.0.1) and return its exit code;
    None when this process is already a rank (or N = 1)."""
    if args.gpus <= 1 or "WORLD_SIZE" in os.environ:
        return None
    if not args.spawn_probe and not ONE_GPU:
        import torch
        have = torch.cuda.device_count()
        if have < args.gpus:
            print(f"bench.py: --gpus {args.gpus} but only {have} CUDA device(s) visible", file=sys.stderr)
            return 2
    return subprocess.call(spawn_cmd(argv, args.gpus, free_port()))


def check_world(args):
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    if ws != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={ws}")
    return ws


def run_spawn_probe(args):
    """--spawn-probe: the multi-process launch alone (CPU, gloo): every rank
    reports itself, rank 0 prints the world it sees."""
    import torch.distributed as dist
    ws, rk, lr = dist_env()
    got = [{"rank": rk, "local_rank": lr, "pid": os.getpid()}]
    if ws > 1:
        dist.init_process_group("gloo")
        got = [None] * ws
        dist.all_gather_object(got, {"rank": rk, "local_rank": lr, "pid": os.getpid()})
        dist.destroy_process_group()
    if rk == 0:
        print(json.dumps({"spawn_probe": True, "world_size": ws, "ranks": got}), flush=True)
    return 0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="tiles", choices=["tiles", "reference"])
    ap.add_argument("--config", default="c2", choices=sorted(CONFIGS) + ["c3", "c4", "c5", "fig5", "fig5tiles", "fig8"])
    ap.add_argument("--T", type=int, default=None)
    ap.add_argument("--nstreams", type=int, default=None)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-extras", action="store_true",
                    help="skip the overlap / sync-baseline / CUPTI / C3 / C4 extras")
    ap.add_argument("--n", type=int, default=None, help="c3/c4: grid edge")
    ap.add_argument("--budget-gb", type=float, default=None, help="c3: device budget cap")
    ap.add_argument("--K", type=int, default=32, help="c4: kernel_iteration (reading R12)")
    ap.add_argument("--tile", default=None, help="c5: tile dims tx,ty,tz (default 64,64,64)")
    ap.add_argument("--sweep", default=None, help="c4: comma list of nstreams")
    ap.add_argument("--ghost", type=int, default=1,
                    help="c2/c3: ghost width; 2 = two Jacobi steps per pass (temporal blocking)")
    ap.add_argument("--two-step", type=int, default=0, help="tile_options.two_step (-1, 0, 1)")
    ap.add_argument("--transport", default="peer", choices=["peer", "peer-copy", "nccl"],
                    help="N > 1 halo exchange: CUDA IPC windows written by the stencil kernel "
                         "(default), the same windows written by copies, or NCCL p2p")
    ap.add_argument("--stream-through", type=int, default=0,
                    help="tile_options.stream_through (-1 never, 0 cost model, 1 when feasible)")
    ap.add_argument("--wavefront", type=int, default=0,
                    help="tile_options.wavefront (-1 never, 0 cost model, 1 when feasible)")
    ap.add_argument("--spawn-probe", action="store_true", help="test hook: the N-process launch only")
    argv = sys.argv[1:]
    args = ap.parse_args(argv)
    rc = maybe_spawn(args, argv)
    if rc is not None:
        return rc
    check_world(args)
    if args.spawn_probe:
        return run_spawn_probe(args)
    if args.impl == "reference":
        return run_reference(args)
    if args.config == "c3":
        print(json.dumps(c3_line(args)), flush=True)
        return 0
    if args.config == "c4":
        print(json.dumps(c4_line(args)), flush=True)
        return 0
    if args.config == "fig8":
        return run_fig8_leg(args)
    if args.config == "fig5":
        return run_fig5_leg(args)
    if args.config == "fig5tiles":
        return run_fig5_tiles_leg(args)
    if args.config == "c5":
        return run_c5_leg(args)
    return run_main_leg(args)


SCHED_NAMES = {0: "none", 1: "resident batched (layer batches + whole-domain steps)",
               2: "stream-through (fresh upload, T <= tz)", 3: "out-of-core per-tile stream",
               4: "out-of-core stream-through", 5: "synchronous (one stream)", 6: "wavefront (fresh upload)",
               7: "resident, two steps per kernel (heat2_band)",
               8: "wavefront (upload) + resident two-step passes + wavefront (download)"}
SWEEP_KERNEL = {1: "heat7_fixed", 2: "slab_sweep_tile", 4: "slab_sweep_tile", 5: "heat7_fixed",
                6: "slab_sweep_tile", 7: "heat2_band", 8: "heat2_band"}


def n_two_level(gdims, td, T, args):
    """The stream-through / wavefront sweeps run two levels per kernel
    (heat2_band_slab) on single-rank grids 512 wide with 64-wide tiles."""
    return gdims[0] == 512 and td[0] == 64 and T >= 2 and args.two_step >= 0


def run_main_leg(args):
    import argparse as _ap

    import torch
    import torch.distributed as dist

    from paper_conf_icpp_bastemuzas17_b200 import tiles as Tl
    import synth

    ws, rk, lr = dist_env()
    torch.cuda.set_device(lr)
    numa = bind_numa(torch, lr)
    if ws > 1:
        init_dist(torch, dist, lr)
    dims, td, T, ns, desc = CONFIGS[args.config]
    T = args.T if args.T is not None else T
    ns = args.nstreams or ns
    nx, ny, nzl = dims
    gdims = (nx, ny, nzl * ws)
    cells = nx * ny * nzl  # per rank
    NORMAL = Tl.TILE_MEASURE_NORMAL

    def barrier():
        if ws > 1:
            dist.barrier()
        torch.cuda.synchronize()

    def max_over_ranks(x):
        if ws == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=red_dev())
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    u0 = np.empty((nzl, ny, nx))
    synth.fill_uniform_native(u0.ctypes.data, gdims[0], gdims[1], gdims[2], rk * nzl, nzl, 0, ny, 0, nx, 42)
    dom = multi_domain(Tl, dist, ws, rk, args.transport, gdims, td, ghost=args.ghost, device=lr,
                       two_step=args.two_step, stream_through=args.stream_through, wavefront=args.wavefront)
    t0 = time.perf_counter()
    dom.load(u0)   # tile_load: dense slab -> tile-blocked pinned store (outside the timed region)
    t_load_ms = (time.perf_counter() - t0) * 1e3
    del u0
    k = Tl.heat7(ALPHA)
    spp = dom.info["steps_per_pass"]

    def e2e_steps(mode, reps, timing=False):
        """reps bench steps: tile_invalidate (host store is the source) ->
        tile_run(T) -> tile_sync (every tile back in the pinned store)."""
        dom.set_measure(mode)
        dom.set_kernel_timing(timing)
        dom.reset_stats()
        barrier()
        tot = 0.0
        for _ in range(reps):
            dom.invalidate()
            dom.timer_start()
            dom.run(k, T, ns)
            dom.sync()
            tot += dom.timer_stop()
        st_ = dom.stats()
        dom.set_kernel_timing(False)
        dom.set_measure(NORMAL)
        return max_over_ranks(tot), st_

    # ---- value: the metric, H2D and D2H of every cell inside the step --------
    for _ in range(args.warmup):
        dom.invalidate()
        dom.run(k, T, ns)
        dom.sync()
    with Clocks(lr) as clk:
        ms, st = e2e_steps(NORMAL, args.steps)
    value = ws * cells * T * args.steps / (ms / 1e3) / 1e9
    sched = dom.get_info().get("last_schedule", 0)
    h2d_b = st["bytes_h2d"] // args.steps
    d2h_b = st["bytes_d2h"] // args.steps
    peak, peak_src = measured_peaks()
    # the step's kernels with CUDA events: the same schedule with
    # the copies skipped (TILE_MEASURE_COMP_ONLY), so the launches run back to
    # back and each event pair brackets its kernel (timed inside the e2e leg,
    # the events would also bracket the host's enqueue gaps while the stream
    # waits on uploads, and they perturb the copy pipeline)
    co_t_ms, stk = e2e_steps(Tl.TILE_MEASURE_COMP_ONLY, args.steps, timing=True)
    sw_ms, sw_cells, sw_n = stk["sweep_ms"], stk["sweep_cells"], max(1, stk["sweep_timed"])
    achieved = 16.0 * sw_cells / (sw_ms / 1e3) / 1e9 if sw_ms > 0 else None
    kname = SWEEP_KERNEL.get(sched, "stencil sweeps")
    if (sched == 6 or (sched == 2 and args.two_step > 0)) and ws == 1 and n_two_level(gdims, td, T, args):
        kname = "heat2_band_slab"   # two sweeps / levels per kernel on grids 512 wide
    prof = traffic_per_cell(kname)
    roof = {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
            "frac": achieved / peak if achieved else None,
            "traffic": prof[0] * sw_cells / sw_n if prof else None,
            "traffic_source": prof[1] if prof else None,
            "kernel": kname, "schedule": SCHED_NAMES.get(sched, str(sched)),
            "algorithmic_bytes_per_cell_sweep": 16.0,
            "algorithmic_bytes_per_launch": 16.0 * sw_cells / sw_n,
            "launches_per_step": sw_n / args.steps, "avg_launch_ms": sw_ms / sw_n,
            "kernel_ms_per_step": sw_ms / args.steps,
            "kernel_share_of_step": sw_ms / ms if ms > 0 else None,
            "note": "achieved = 16 B x cells swept by the step's sweep launches / their summed CUDA-event "
                    "durations on the launching stream (one event pair per run of consecutive sweeps on a "
                    "stream, so programmatic dependent launch keeps overlapping them), measured on the same "
                    "schedule with the copies skipped (comp-only) so that launches run back to back; the "
                    "e2e step itself is host-link-bound: see roofline_link",
            "peak_source": peak_src}

    # ---- the kernel-level rate: grid resident in HBM ------------------------
    dom.run(k, 1, ns)
    dom.sync()
    for _ in range(args.warmup):
        dom.run(k, T, ns)
    dom.sync()
    dom.set_kernel_timing(True)
    dom.reset_stats()
    barrier()
    with Clocks(lr) as clk_res:
        dom.timer_start()
        for _ in range(args.steps):
            dom.run(k, T, ns)
        ms_res = dom.timer_stop()
    st_res = dom.stats()
    dom.set_kernel_timing(False)
    ms_res = max_over_ranks(ms_res)
    dom.sync()
    res_value = ws * cells * T * args.steps / (ms_res / 1e3) / 1e9
    rs_ms, rs_cells, rs_n = st_res["sweep_ms"], st_res["sweep_cells"], max(1, st_res["sweep_timed"])
    r_ach = 16.0 * rs_cells / (rs_ms / 1e3) / 1e9 if rs_ms > 0 else None
    res_sched = dom.get_info().get("last_schedule", 1)
    band2 = res_sched == 7   # heat2_band: one launch = one pass = two steps
    tps = traffic_from_profile("band2" if band2 else args.config) if (spp == 1 or band2) else None
    steps_per_launch = rs_cells / rs_n / cells * (2 if band2 else 1)
    resident = {"value": res_value, "unit": "Gcell-updates/s", "ms_per_step": ms_res / args.steps,
                "def": "grid resident in HBM; tile_run(T) per step, no host transfers",
                "gpu_launches": st_res["n_kernels"],
                "roofline": {"bound": "hbm", "achieved": r_ach, "peak": peak, "unit": "GB/s",
                             "frac": r_ach / peak if r_ach else None,
                             "traffic": tps * steps_per_launch if tps else None, "traffic_per_step": tps,
                             "kernel": "heat2_band (2 steps per pass)" if band2 else
                                       "heat7_fixed" if spp == 1 else "heat7x2 (2 steps per pass)",
                             "schedule": SCHED_NAMES.get(res_sched, str(res_sched)),
                             "algorithmic_bytes_per_cell_update": 8.0 if band2 else 16.0 / spp,
                             "algorithmic_bytes_per_launch": 16.0 * rs_cells / rs_n,
                             "steps_per_launch": steps_per_launch * (1 if band2 else spp),
                             "avg_launch_ms": rs_ms / rs_n,
                             "peak_source": peak_src},
                "clocks": clk_res.summary()}

    extras = {}
    if not args.no_extras:
        # overlap: the same schedule with kernels skipped / copies skipped,
        # as many repetitions as the timed value leg, unclamped
        xo_ms, _ = e2e_steps(Tl.TILE_MEASURE_XFER_ONLY, args.steps)
        co_ms, _ = e2e_steps(Tl.TILE_MEASURE_COMP_ONLY, args.steps)
        wall, xo, co = ms / args.steps, xo_ms / args.steps, co_ms / args.steps
        hidden = (xo + co - wall) / min(xo, co)
        ov = {"hidden_frac": hidden, "t_wall_ms": wall, "t_xfer_only_ms": xo, "t_comp_only_ms": co,
              "reps": args.steps, "definition": "(T_xfer_only + T_comp_only - T_wall) / min(...), unclamped",
              "note": "compute << transfer here, so this is the fraction of the kernel time hidden "
                      "under transfers; > 1 means T_wall < T_xfer_only (the xfer-only schedule "
                      "issues the same copies without the kernels' events, so it is not a strict bound)"}
        try:
            def one():
                dom.invalidate()
                dom.run(k, T, ns)
                dom.sync()
            ov["cupti"] = cupti_overlap(torch, one)
            kb = ov["cupti"]["kernel_busy_ms"] if ov["cupti"] else 0
            if kb and sw_cells:
                # the same step's kernels as the GPU ran them inside the
                # pipeline (CUPTI activity records: with programmatic dependent
                # launch the sweeps overlap their neighbours' ramp and drain,
                # which per-launch CUDA events cannot show)
                ach = 16.0 * (sw_cells / args.steps) / (kb / 1e3) / 1e9
                roof.update({"achieved_in_pipeline": ach, "frac_in_pipeline": ach / peak,
                             "in_pipeline_def": "16 B x cells swept per step / the step's CUPTI kernel-busy "
                                                "time (union of kernel intervals; only sweeps run in it)"})
        except Exception as e:  # profiler unavailable: say so
            ov["cupti"] = {"error": str(e)[:200]}
        bw = pcie_bandwidth(torch)
        bidir = pcie_bidir(torch)
        B = cells * 8
        # streaming (duplex) form: every byte crosses the link
        # once each way; no schedule beats max(B/h2d, B/d2h, 2B/bidir)
        t_link = max(B / (bw["h2d"] * 1e9), B / (bw["d2h"] * 1e9), 2 * B / (bidir * 1e9))
        t_dep = B / (bw["h2d"] * 1e9) + B / (bw["d2h"] * 1e9)     # tile-granular dependency form
        t_hbm = T * 16 * cells / (peak * 1e9)
        R = max(t_link, t_hbm)
        extras["overlap"] = ov
        extras["roofline_link"] = {"bound": "pcie (streaming/duplex form: max(B/h2d, B/d2h, 2B/bidir))",
                                   "t_bound_ms": R * 1e3, "t_link_ms": t_link * 1e3,
                                   "t_link_dependency_form_ms": t_dep * 1e3, "t_hbm_ms": t_hbm * 1e3,
                                   "frac": R / (wall / 1e3), "achieved_gbs": (h2d_b + d2h_b) / (wall / 1e3) / 1e9,
                                   "peak_gbs": bidir, "pcie_gbs": {**bw, "bidir": bidir}}
        # the stencil's own constraint on top of the duplex form: no output
        # plane before its 2T+1-plane cone has arrived (H2D alone), and the
        # last upload's cone returns alone (D2H alone); between, both ways
        cone = min(2 * T + 1, nzl) * nx * ny * 8
        t_causal = cone / (bw["h2d"] * 1e9) + cone / (bw["d2h"] * 1e9) + 2 * max(0, B - cone) / (bidir * 1e9)
        extras["roofline_link"].update({
            "t_causal_duplex_ms": t_causal * 1e3, "frac_causal_duplex": t_causal / (wall / 1e3),
            "causal_duplex_def": "(2T+1) planes H2D alone + (2T+1) planes D2H alone + the rest both ways "
                                 "at the bidirectional rate"})
        if ws == 1:
            dom.free()
            sdom = Tl.Domain(gdims, td, ghost=args.ghost, device=lr, sched="sync")
            u0 = np.empty((nzl, ny, nx))
            synth.fill_uniform_native(u0.ctypes.data, gdims[0], gdims[1], gdims[2], 0, nzl, 0, ny, 0, nx, 42)
            sdom.load(u0)
            del u0
            sdom.run(k, T, 1)
            sdom.sync()
            tot = 0.0
            reps = max(2, args.steps // 4)
            for _ in range(reps):
                sdom.invalidate()
                sdom.timer_start()
                sdom.run(k, T, 1)
                sdom.sync()
                tot += sdom.timer_stop()
            sdom.free()
            extras["sync_baseline_e2e"] = {"value": cells * T * reps / (tot / 1e3) / 1e9,
                                           "unit": "Gcell-updates/s", "ms_per_step": tot / reps,
                                           "schedule": "H2D all, T steps, D2H all, one stream (pinned)"}
    try:
        dom.free()
    except Exception:
        pass

    cpu = None
    if rk == 0 and ws == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(T, 384 if args.config == "c2" else dims[0], 512 if args.config == "c2" else dims[0])

    if ws == 1 and not args.no_extras and args.config == "c2":
        # the other BASELINE.json configs, driver-observed: C3 out of core
        # (2048^3, capped budget) and C4 (the compute-intensive kernel)
        for key, fn, kw in (("c3", c3_line, dict(n=None, T=None, nstreams=None, budget_gb=None, ghost=1,
                                                  stream_through=0, steps=2, warmup=1)),
                            ("c4", c4_line, dict(n=None, T=None, nstreams=None, K=args.K, sweep="1,2,4,8",
                                                  steps=2, warmup=1)),
                            # C5's per-GPU slab of the 8-GPU decomposition (4096 x 4096 x 512)
                            ("c5", c5_line, dict(n=None, T=None, nstreams=None, tile=None, transport=args.transport,
                                                  steps=2, warmup=1))):
            try:
                ln = fn(_ap.Namespace(**kw))
                extras[key] = {kk: ln[kk] for kk in ("value", "unit", "ms_per_step", "config", "e2e", "overlap",
                                                      "roofline", "clocks", "stream_sweep_e2e")
                               if kk in ln}
                if key == "c5":
                    extras[key]["value_def"] = "per-GPU slab resident in HBM (heat7_fixed); e2e: with H2D/D2H"
            except Exception as e:  # e.g. not enough host RAM for C3's pinned store
                extras[key] = {"error": str(e)[:300]}

    if rk == 0:
        line = {"metric": METRIC, "value": value, "unit": "Gcell-updates/s", "n_gpus": ws,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms / args.steps,
                "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
                "data": "synthetic",
                "config": {"workload": desc, "dims_per_gpu": dims, "global_dims": gdims, "tile_dims": td,
                           "ghost": args.ghost, "steps_per_pass": spp, "T": T, "nstreams": ns,
                           "bc": "periodic", "alpha": ALPHA,
                           "parallelism": f"z-slab x{ws}, one process per GPU" if ws > 1 else "1 GPU",
                           "transport": getattr(multi_domain, "fallback", args.transport) if ws > 1 else None,
                           "comm_ranks": ws,
                           "schedule": SCHED_NAMES.get(sched, str(sched)),
                           "host_cpus": numa, "tile_load_ms": t_load_ms,
                           "l2": "inputs larger than L2 (2 x 1.07 GB per GPU per step)",
                           "value_def": "the metric: tile_invalidate + tile_run(T) + tile_sync from the "
                                        "pinned host store, H2D and D2H of every cell inside the timed step",
                           "e2e_def": "same measurement as value (the metric includes H2D/D2H)"},
                "e2e": {"value": value, "unit": "Gcell-updates/s", "h2d_bytes_per_step": h2d_b,
                        "d2h_bytes_per_step": d2h_b, "ms_per_step": ms / args.steps},
                "gpu_launches": st["n_kernels"], "roofline": roof, "resident": resident,
                "cpu_baseline": cpu, "clocks": clk.summary()}
        line.update(extras)
        print(json.dumps(line), flush=True)
    if ws > 1:
        dist.destroy_process_group()
    return 0


if __name__ == "__main__":
    sys.exit(main())
