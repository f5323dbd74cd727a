"""Host-side logic of bench.py's multi-GPU launch on CPU (no GPU): NUMA
binding from sysfs, and the transport fallback every rank must agree on
(peer windows unavailable on any rank -> all ranks take NCCL)."""
import io
import os
import sys
import types

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402


class _Props:
    pci_domain_id, pci_bus_id, pci_device_id = 0, 0x66, 0


def _fake_torch():
    t = types.SimpleNamespace()
    t.cuda = types.SimpleNamespace(get_device_properties=lambda dev: _Props())
    return t


def test_bind_numa_parses_local_cpulist(monkeypatch):
    seen = {}
    real_open = open

    def fake_open(path, *a, **k):
        if path.endswith("local_cpulist"):
            seen["path"] = path
            return io.StringIO("0-3,8-11\n")
        return real_open(path, *a, **k)

    monkeypatch.setattr("builtins.open", fake_open)
    monkeypatch.setattr(os, "sched_getaffinity", lambda pid: set(range(16)))
    monkeypatch.setattr(os, "sched_setaffinity", lambda pid, cpus: seen.setdefault("cpus", set(cpus)))
    assert bench.bind_numa(_fake_torch(), 0) == "0-3,8-11"
    assert seen["path"] == "/sys/bus/pci/devices/0000:66:00.0/local_cpulist"
    assert seen["cpus"] == {0, 1, 2, 3, 8, 9, 10, 11}


def test_bind_numa_is_a_noop_without_sysfs(monkeypatch):
    def boom(*a, **k):
        raise FileNotFoundError

    monkeypatch.setattr("builtins.open", boom)
    called = []
    monkeypatch.setattr(os, "sched_setaffinity", lambda pid, cpus: called.append(cpus))
    assert bench.bind_numa(_fake_torch(), 0) is None and not called


class _TileError(RuntimeError):
    pass


def _fake_tiles(fail_peer_on_rank, rank):
    made = []

    class Dom:
        def __init__(self, *a, **kw):
            self.kw = kw
            made.append(self)
            if kw.get("peer_transport") and rank == fail_peer_on_rank:
                raise _TileError("tile_domain_create: ECUDA: no peer access")
            self.freed = False

        def peer_handle(self):
            return b"h" * 64

        def peer_connect(self, hs):
            pass

        def free(self):
            self.freed = True

    return types.SimpleNamespace(Domain=Dom, TileError=_TileError, nccl_unique_id=lambda: b"i" * 128), made


class _FakeDist:
    """Two ranks simulated by sharing one 'all_reduce MIN' verdict."""

    def __init__(self, other_ok):
        self.other_ok = other_ok

    class ReduceOp:
        MIN = "min"

    def all_gather_object(self, out, obj):
        for i in range(len(out)):
            out[i] = obj

    def all_reduce(self, t, op=None):
        t.copy_(t.clamp(max=1 if self.other_ok else 0))

    def broadcast_object_list(self, obj, src=0):
        pass


@pytest.mark.parametrize("fail_rank,other_ok,expect_nccl", [(None, True, False), (0, True, True),
                                                             (None, False, True)])
def test_multi_domain_transport_fallback(monkeypatch, fail_rank, other_ok, expect_nccl):
    monkeypatch.setattr(bench, "red_dev", lambda: "cpu")
    if hasattr(bench.multi_domain, "fallback"):
        monkeypatch.delattr(bench.multi_domain, "fallback")
    Tl, made = _fake_tiles(fail_rank, 0)
    dom = bench.multi_domain(Tl, _FakeDist(other_ok), 2, 0, "peer", (8, 8, 16), (8, 8, 8), ghost=1)
    uses_nccl = "nccl_id" in dom.kw
    assert uses_nccl == expect_nccl
    assert (getattr(bench.multi_domain, "fallback", None) is not None) == expect_nccl
    if expect_nccl and fail_rank is None:   # this rank's peer domain was built, then released
        assert made[0].freed


def test_bench_spawns_one_process_per_gpu():
    """`python bench.py --gpus 2` with no torchrun environment re-launches
    itself under torch.distributed.run (127.0.0.1), one process per GPU:
    the probe mode stops right after the launch and has rank 0 report the
    world it sees (gloo on CPU)."""
    import json
    import subprocess
    import sys
    env = {k: v for k, v in os.environ.items()
           if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--spawn-probe"],
                       capture_output=True, text=True, env=env, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [json.loads(x) for x in r.stdout.splitlines() if x.startswith("{")]
    assert len(lines) == 1, r.stdout
    ln = lines[0]
    assert ln["world_size"] == 2 and sorted(x["rank"] for x in ln["ranks"]) == [0, 1]
    assert len({x["pid"] for x in ln["ranks"]}) == 2


def test_bench_rejects_world_size_mismatch():
    import subprocess
    import sys
    env = dict(os.environ, WORLD_SIZE="3", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--spawn-probe"],
                       capture_output=True, text=True, env=env, timeout=120)
    assert r.returncode != 0 and "WORLD_SIZE=3" in r.stderr


def test_spawn_command_is_the_drivers_launch_line():
    cmd = bench.spawn_cmd(["--gpus", "4", "--steps", "5"], 4, 29511)
    assert cmd[1:4] == ["-m", "torch.distributed.run", "--nnodes=1"]
    assert "--nproc-per-node=4" in cmd and "127.0.0.1" in cmd and "--master-port=29511" in cmd
    assert cmd[-4:] == ["--gpus", "4", "--steps", "5"]
