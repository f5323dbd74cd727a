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
