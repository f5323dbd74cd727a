"""Host-side logic of libtiles on a CPU (dry-run executor, no GPU).

* The C ABI loads and exports every function include/tiles.h declares.
* tile_ghost_map / tile_face_sources equal the oracle's brute-force map.
* The scheduler's op trace, replayed in random valid orders with oracle
  arithmetic (tests/replay.py), reproduces the untiled oracle bit-exactly for
  resident, synchronous and out-of-core (streaming) schedules, periodic and
  Dirichlet boundaries, several stream counts and device budgets.
* Residency accounting: hits, misses, evictions, bytes.
"""
import os
import re
import subprocess
import sys

import numpy as np
import pytest

import oracle
import synth
from tests.replay import Geometry, Replayer, split_tiles, wsweep_range

T = pytest.importorskip("paper_conf_icpp_bastemuzas17_b200.tiles")

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ALPHA = 0.125


def test_cabi_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "tiles.h")).read()
    declared = set(re.findall(r"^\s*(?:tile_status|const char\*)\s+(tile_\w+)\s*\(", hdr, re.M))
    assert len(declared) >= 20
    out = subprocess.run(["nm", "-D", "--defined-only", T.LIB_PATH], capture_output=True, text=True).stdout
    exported = set(re.findall(r"\bT (tile_\w+)", out))
    assert declared <= exported, declared - exported
    assert declared == set(T.EXPORTED)


def test_invalid_arguments_have_no_side_effects():
    bad = [((64, 64, 64), (24, 32, 32), 1),   # ragged
           ((64, 64, 64), (31, 32, 32), 1),   # odd x
           ((64, 64, 64), (32, 32, 32), 0),   # ghost < 1
           ((64, 64, 64), (32, 32, 2), 3),    # ghost > min(tile)
           ((0, 64, 64), (32, 32, 32), 1)]
    for dims, td, g in bad:
        with pytest.raises(T.TileError) as e:
            T.Domain(dims, td, ghost=g, dry_run=True)
        assert e.value.code == T.TILE_EINVAL
    with pytest.raises(T.TileError) as e:
        T.Domain((16, 16, 16), (8, 8, 8), dry_run=True, peer_transport=3)
    assert e.value.code == T.TILE_EINVAL
    d = T.Domain((16, 16, 16), (8, 8, 8), dry_run=True)
    for k, steps, ns in [(T.heat7(0.2), 1, 1), (T.heat7(0.0), 1, 1), (T.heat7(), -1, 1),
                         (T.heat7(), 1, 0), (T.heat7(), 1, 65), (T.sincos(-1), 1, 1)]:
        with pytest.raises(T.TileError) as e:
            d.run(k, steps, ns)
        assert e.value.code == T.TILE_EINVAL
    assert d.trace() == []


@pytest.mark.parametrize("bc", ["periodic", "dirichlet"])
@pytest.mark.parametrize("dims,td,g", [((8, 4, 4), (2, 2, 2), 1), ((12, 8, 6), (4, 4, 3), 2),
                                       ((6, 6, 4), (6, 6, 4), 1)])
def test_ghost_map_matches_oracle(bc, dims, td, g):
    b = T.BCS[bc]
    d = T.Domain(dims, td, ghost=g, bc=bc, dry_run=True)
    for k in range(d.info["ntiles"]):
        assert np.array_equal(d.ghost_map(k), oracle.ghost_map(dims, td, g, k, b))


def test_face_sources_agree_with_ghost_map():
    # the face descriptor of face f names the tile whose cells fill the
    # ghost layer just outside f, per the brute-force map
    dims, td = (8, 12, 8), (4, 4, 4)
    d = T.Domain(dims, td, dry_run=True)
    for k in range(d.info["ntiles"]):
        m = oracle.ghost_map(dims, td, 1, k)
        fs = d.face_sources(k)
        probes = {0: m[2, 2, 0], 1: m[2, 2, -1], 2: m[2, 0, 2], 3: m[2, -1, 2], 4: m[0, 2, 2], 5: m[-1, 2, 2]}
        for f, gidx in probes.items():
            kind, nb = fs[f]
            assert kind == 0
            x, y, z = gidx % 8, (gidx // 8) % 12, gidx // 96
            assert nb == (z // 4 * 3 + y // 4) * 2 + x // 4


def _budget_for(dims, td, nslots, **kw):
    lo, hi = 1, 1 << 36
    tile_bytes = td[0] * td[1] * td[2] * 8
    while lo < hi:
        mid = (lo + hi) // 2
        try:
            n = T.Domain(dims, td, dry_run=True, device_budget_bytes=mid, **kw).info["nslots"]
        except T.TileError:
            n = -1
        if n >= nslots:
            hi = mid
        else:
            lo = mid + 1
    d = T.Domain(dims, td, dry_run=True, device_budget_bytes=lo, **kw)
    assert d.info["nslots"] == nslots, (d.info["nslots"], nslots, tile_bytes)
    return lo


def _run_and_replay(dims, td, steps_list, nstreams, seeds=(0, 1, 2), bc="periodic", ghost=1, lazy=(), **kw):
    nx, ny, nz = dims
    if bc == "periodic":
        u0 = synth.uniform_grid(nx, ny, nz, 42)
        ext = None
        ref = oracle.heat_c(u0, ALPHA, sum(steps_list))
    else:
        ext = synth.uniform_grid(nx + 2, ny + 2, nz + 2, 5)
        u0 = ext[1:-1, 1:-1, 1:-1].copy()
        ref = oracle.heat_c(ext, ALPHA, sum(steps_list), oracle.BC_DIRICHLET)[1:-1, 1:-1, 1:-1]
    for seed in seeds:
        d = T.Domain(dims, td, bc=bc, dry_run=True, ghost=ghost, **kw)
        d.load(ext if bc == "dirichlet" else u0)
        G = Geometry(dims, td, bc=T.BCS[bc], ghost=ghost)
        rep = Replayer(G, split_tiles(G, u0), ALPHA, ext=ext)
        for steps in steps_list:
            d.clear_trace()
            d.run(T.heat7(ALPHA), steps, nstreams)
            d.sync()
            rep.replay(d.trace(), seed, lazy=lazy)
        out = rep.grid()
        assert np.array_equal(out, ref), np.abs(out - ref).max()
    return d


@pytest.mark.parametrize("dims,td,ns", [((16, 16, 16), (8, 8, 8), 2), ((16, 8, 24), (8, 4, 4), 3),
                                        ((8, 8, 8), (8, 8, 8), 1), ((16, 16, 8), (4, 8, 2), 4)])
def test_resident_schedule_replays_to_oracle(dims, td, ns):
    d = _run_and_replay(dims, td, [5], ns)
    assert d.info["sched"] == T.TILE_SCHED_RESIDENT


def test_resident_multiple_runs_and_dirichlet():
    _run_and_replay((16, 8, 16), (8, 4, 4), [3, 2, 1], 2)
    _run_and_replay((16, 8, 16), (8, 4, 4), [4], 2, bc="dirichlet")


@pytest.mark.parametrize("dims,td,runs,ns", [((512, 8, 16), (64, 4, 8), [1, 4, 3, 2], 2),
                                             ((512, 12, 12), (64, 4, 4), [2, 5], 3),
                                             ((512, 4, 8), (64, 4, 8), [3, 6], 1),
                                             ((512, 4, 1), (64, 4, 1), [1, 4], 2)])   # nz = 1
def test_band2_resident_runs_replay_to_oracle(dims, td, runs, ns):
    """Resident periodic runs 512 cells wide take two steps per kernel over the
    whole grid (heat2_band, TILE_OP_BAND2; an odd step the face-ghost single
    step): replayed in random valid orders, bit-exact to the oracle, with the
    arrays alternating and every later run re-extracting the stale faces."""
    d = _run_and_replay(dims, td, runs, ns, seeds=(0, 1))
    assert d.get_info()["last_schedule"] == 7
    for T_ in (4, 5):
        d.clear_trace()
        d.run(T.heat7(ALPHA), T_, ns)
        d.sync()
        ops = [op[0] for op in d.trace()]
        assert ops.count("band2") == T_ // 2
        assert ("kernel" in ops or "kerneld" in ops) == bool(T_ % 2) and ("extract" in ops) == bool(T_ % 2)
        b2 = [op for op in d.trace() if op[0] == "band2"]
        assert all((op[2] >> 1) & 1 != (op[3] >> 1) & 1 for op in b2)
    # two_step = -1 keeps single steps
    d2 = _run_and_replay(dims, td, runs[:2], ns, seeds=(2,), two_step=-1)
    assert "band2" not in [op[0] for op in d2.trace()]


@pytest.mark.parametrize("T_", [9, 12, 7])
def test_band2_middle_of_batched_fresh_upload_replays(T_):
    """A fresh upload on the batched schedule (layer batches overlapping the
    load, whole-domain middle steps, a layered last step): the middle steps
    run in pairs on heat2_band once the load phase is joined, an odd one
    joins the last phase, which re-extracts the stale faces; replayed in
    random orders, bit-exact."""
    dims, td = (512, 8, 64), (64, 4, 8)   # 8 tile layers: load phase of 5 steps
    d = _run_and_replay(dims, td, [T_], 2, seeds=(0, 1, 2), wavefront=-1, stream_through=-1)
    ops = [op[0] for op in d.trace()]
    mid = T_ - 5 - 1
    assert ops.count("band2") == (mid // 2 if mid >= 2 else 0)
    assert d.get_info()["last_schedule"] == 1


@pytest.mark.parametrize("bc", ["periodic", "dirichlet"])
@pytest.mark.parametrize("dims,td,ns", [((64, 16, 16), (32, 8, 8), 2), ((64, 32, 24), (32, 16, 4), 3),
                                        ((32, 8, 8), (32, 8, 8), 1), ((64, 16, 32), (64, 8, 4), 4)])
def test_direct_ghost_passes_replay_to_oracle(bc, dims, td, ns):
    """Resident single steps with a specialised kernel read their y/z ghosts
    straight from the neighbours' interiors (KERNELD) and export
    only the x faces; the replay takes those ghosts from the neighbour slots
    of the same buffer array and poisons every stale export, so a schedule
    that reads a neighbour too early or too late, or a later pass that reads
    a y/z face a direct pass did not write, breaks bit-exactness."""
    d = _run_and_replay(dims, td, [3, 2, 1, 4], ns, seeds=(0, 1), bc=bc)
    ops = [op[0] for op in d.trace()]
    assert "kerneld" in ops and "kernel" not in ops


def test_direct_then_two_step_passes_reextract_faces():
    # a direct run leaves the y/z exports stale; a following run of two-step
    # passes (which read every face) must re-extract them first
    dims, td = (64, 32, 32), (32, 16, 8)
    d = _run_and_replay(dims, td, [3, 4, 1], 2, seeds=(0, 4), ghost=2, two_step=1)
    ops = [op[0] for op in d.trace()]
    assert "kerneld" in ops


def test_sync_baseline_schedule_is_one_stream():
    d = _run_and_replay((16, 16, 16), (8, 8, 8), [4], 4, sched="sync")
    assert {op[1] for op in d.trace() if op[0] in ("h2d", "kernel", "d2h")} == {0}


@pytest.mark.parametrize("nslots,ns", [(2, 1), (3, 2), (5, 1), (6, 3), (12, 2), (20, 4)])
def test_stream_schedule_replays_to_oracle(nslots, ns):
    dims, td = (16, 16, 16), (8, 8, 4)   # 16 tiles
    b = _budget_for(dims, td, nslots, sched="stream")
    d = _run_and_replay(dims, td, [3, 2], ns, seeds=(0, 7), sched="stream", device_budget_bytes=b)
    st = d.stats()
    assert d.info["sched"] == T.TILE_SCHED_STREAM and d.info["nslots"] == nslots
    assert st["misses"] + st["hits"] == 16 * 5  # 3 + 2 passes over 16 tiles


def test_stream_schedule_dirichlet():
    dims, td = (16, 8, 16), (8, 4, 4)
    b = _budget_for(dims, td, 5, sched="stream", bc="dirichlet")
    _run_and_replay(dims, td, [4], 2, seeds=(3,), bc="dirichlet", sched="stream", device_budget_bytes=b)


def test_stream_residency_accounting():
    # 16 tiles, few slots: every pass misses every tile (no window), each
    # tile is copied in and written back once per step
    dims, td = (16, 16, 16), (8, 8, 4)
    b = _budget_for(dims, td, 4, sched="stream")
    d = T.Domain(dims, td, dry_run=True, sched="stream", device_budget_bytes=b)
    d.load(np.zeros((16, 16, 16)))
    d.run(T.heat7(), 3, 1)
    d.sync()
    st = d.stats()
    tile_b = 8 * 8 * 4 * 8
    faces_b = sum(16 * n * 8 for n in (4 * 8, 4 * 8, 4 * 8, 4 * 8, 8 * 8, 8 * 8))
    # clean tiles left in a slot at the end of a pass are hits at the start
    # of the next (snake order): at most nslots per pass boundary
    assert st["misses"] + st["hits"] == 48 and st["hits"] <= 2 * 4
    assert st["bytes_h2d"] == st["misses"] * tile_b + faces_b
    assert st["bytes_d2h"] == 48 * tile_b  # write-through: no kept window
    # generous budget: the snake order turns the kept window into hits
    b2 = _budget_for(dims, td, 20, sched="stream")
    d2 = T.Domain(dims, td, dry_run=True, sched="stream", device_budget_bytes=b2)
    d2.load(np.zeros((16, 16, 16)))
    d2.run(T.heat7(), 3, 1)
    d2.sync()
    s2 = d2.stats()
    W = 20 - 4 - 2
    assert s2["hits"] >= 2 * W and s2["misses"] + s2["hits"] == 48
    assert s2["bytes_d2h"] == 48 * tile_b - 2 * W * tile_b  # kept tiles recomputed before write-back


def test_stream_never_evicts_tile_in_use():
    dims, td = (16, 16, 16), (8, 8, 4)
    b = _budget_for(dims, td, 2, sched="stream")
    d = T.Domain(dims, td, dry_run=True, sched="stream", device_budget_bytes=b)
    d.load(np.zeros((16, 16, 16)))
    d.run(T.heat7(), 2, 1)
    d.sync()
    owner = {}
    for op in d.trace():
        if op[0] == "h2d":
            owner[op[3]] = op[2]
        if op[0] == "kernel":
            assert owner[op[3]] == op[2] and op[3] != op[4]
            owner[op[4]] = op[2]


@pytest.mark.parametrize("sched,fuse,nslots", [("auto", True, None), ("stream", True, 3),
                                               ("stream", False, 3), ("resident", False, None)])
def test_pointwise_schedule_replays_to_oracle(sched, fuse, nslots):
    dims, td = (8, 8, 8), (4, 4, 4)
    K, steps = 3, 2
    kw = {"sched": sched, "fuse_pointwise_steps": fuse}
    if nslots:
        kw["device_budget_bytes"] = _budget_for(dims, td, nslots, sched=sched)
    x0 = synth.uniform_grid(8, 8, 8, 7)
    d = T.Domain(dims, td, dry_run=True, **kw)
    d.load(x0)
    d.run(T.sincos(K), steps, 2)
    d.sync()
    G = Geometry(dims, td)
    rep = Replayer(G, split_tiles(G, x0), ALPHA)
    rep.replay(d.trace(), 0)
    ref = oracle.sincos_c(x0, K, steps)
    assert np.array_equal(rep.grid(), ref)
    n_pw = sum(1 for op in d.trace() if op[0] == "pointwise")
    assert n_pw == (8 if fuse else 16)


def test_load_store_roundtrip_and_host_tile_view():
    dims, td = (16, 8, 8), (8, 4, 4)
    u = synth.uniform_grid(*dims, 3)
    d = T.Domain(dims, td, dry_run=True)
    d.load(u)
    assert np.array_equal(d.store(), u)
    v = d.host_tile(3)
    ix, iy, iz = 3 % 2, (3 // 2) % 2, 3 // 4
    assert np.array_equal(v, u[iz * 4:(iz + 1) * 4, iy * 4:(iy + 1) * 4, ix * 8:(ix + 1) * 8])
    v[:] = 1.5
    d.mark_host_dirty()
    assert (d.store()[0:4, 4:8, 8:16] == 1.5).all()
    ue = synth.uniform_grid(18, 10, 10, 4)
    dd = T.Domain(dims, td, bc="dirichlet", dry_run=True)
    dd.load(ue)
    out = np.zeros_like(ue)
    dd.store(out)
    assert np.array_equal(out[1:-1, 1:-1, 1:-1], ue[1:-1, 1:-1, 1:-1])


def test_trace_ops_are_issue_ordered_per_stream():
    d = T.Domain((16, 16, 16), (8, 8, 8), dry_run=True)
    d.load(np.zeros((16, 16, 16)))
    d.run(T.heat7(), 2, 2)
    tr = d.trace()
    # every layer kernel of step 0 follows its own layer's h2d on its stream
    seen_h2d = set()
    for op in tr:
        if op[0] == "h2d":
            seen_h2d.update(range(op[2], op[2] + op[4]))
        if op[0] == "kernel":
            assert op[2] in seen_h2d


@pytest.mark.parametrize("bc", ["periodic", "dirichlet"])
@pytest.mark.parametrize("sched", ["resident", "stream"])
def test_ghost2_schedules_replay_to_oracle(bc, sched):
    dims, td = (16, 8, 16), (8, 4, 4)
    kw = {"sched": sched}
    if sched == "stream":
        kw["device_budget_bytes"] = _budget_for(dims, td, 5, sched="stream", bc=bc, ghost=2)
    _run_and_replay(dims, td, [3, 2], 2, seeds=(0, 5), bc=bc, ghost=2, **kw)


@pytest.mark.parametrize("bc", ["periodic", "dirichlet"])
@pytest.mark.parametrize("sched,td", [("resident", (32, 16, 8)), ("stream", (32, 16, 8)),
                                      ("resident", (32, 32, 4)), ("resident", (32, 16, 16))])
def test_two_step_passes_replay_to_oracle(bc, sched, td):
    """ghost = 2: passes of two steps (temporal blocking). The replay builds
    each tile's u^s ghost region only from what the schedule made available
    (depth-2 faces of the neighbours at the read parity, edge cells out of the
    diagonal neighbours' faces, Dirichlet halo) and NaN elsewhere; two oracle
    steps must give the untiled oracle bit-exactly with no NaN reaching the
    tile."""
    dims = (64, 32, 32)
    kw = {"sched": sched, "two_step": 1}
    if sched == "stream":
        kw["device_budget_bytes"] = _budget_for(dims, td, 3, sched="stream", bc=bc, ghost=2)
    d = _run_and_replay(dims, td, [5, 2], 2, seeds=(0, 3), bc=bc, ghost=2, **kw)
    ops = [op[0] for op in d.trace()]
    assert "kernel2" in ops


@pytest.mark.parametrize("dims,td,T,ns", [((16, 16, 64), (8, 8, 8), 3, 2), ((16, 8, 64), (8, 4, 8), 4, 3),
                                          ((16, 16, 64), (8, 8, 8), 2, 1), ((32, 16, 48), (16, 8, 8), 1, 4),
                                          ((16, 16, 128), (8, 8, 32), 2, 2), ((16, 8, 192), (8, 4, 48), 7, 2),
                                          ((16, 16, 64), (8, 8, 8), 6, 2), ((16, 8, 384), (8, 4, 48), 20, 3)])
def test_stream_through_schedule_replays_to_oracle(dims, td, T, ns):
    """Fresh-upload heat runs with T <= tz use the stream-through schedule
    (per-unit T shrinking sweeps, resident array -> slabs -> sub-tiles, D2H); replayed in random
    valid orders it must give the oracle bit-exactly."""
    d = _run_and_replay(dims, td, [T], ns, seeds=(0, 1, 2), wavefront=-1)
    ops = [op[0] for op in d.trace()]
    assert "sweep" in ops and "h2d_part" in ops and "d2h_part" in ops
    sw = [op for op in d.trace() if op[0] == "sweep"]
    assert any(op[2] < 0 for op in sw) and any(op[3] < 0 for op in sw)   # fused gather / scatter
    assert d.get_info()["resident"]
    # then a resident continuation and a second stream-through
    _run_and_replay(dims, td, [T, T], ns, seeds=(3,), wavefront=-1)


@pytest.mark.parametrize("dims,td,T_,ns", [((512, 8, 128), (64, 4, 8), 4, 2), ((512, 8, 192), (64, 8, 16), 5, 3),
                                            ((512, 4, 256), (64, 4, 32), 10, 2), ((512, 8, 128), (64, 4, 8), 1, 2)])
def test_stream_through_two_sweeps_per_kernel_replays(dims, td, T_, ns):
    """Stream-through on grids 512 wide with two_step = 1: two sweeps per kernel
    (heat2_band_slab shrink mode, TILE_OP_SWEEP2S; an odd T's last sweep alone), first from the
    resident array, the last into the packed sub-tiles; the intermediate
    level never leaves the chip. Random valid orders give the oracle."""
    d = _run_and_replay(dims, td, [T_, 2], ns, seeds=(0, 1, 2), wavefront=-1, stream_through=1, two_step=1)
    d1 = T_run_dry(dims, td, T_, ns, wavefront=-1, stream_through=1, two_step=1)
    ops = [op[0] for op in d1.trace()]
    assert d1.get_info()["last_schedule"] == 2
    units = ops.count("d2h_part")
    assert ops.count("sweep2s") == units * (T_ // 2) and ops.count("sweep") == units * (T_ % 2)
    # the default (two_step = 0): single sweeps
    d3 = T_run_dry(dims, td, T_, ns, wavefront=-1, stream_through=1)
    assert "sweep2s" not in [op[0] for op in d3.trace()]


@pytest.mark.parametrize("env", ["TILES_ST_OFFSET=1", "TILES_ST_H2D_MERGE=3", "TILES_ST_THIN=0", "TILES_ST_HEAD=4"])
def test_stream_through_copy_plans_replay_to_oracle(env):
    """The stream-through's other H2D copy plans (copies cut T planes into the
    next unit; three units per copy; uniform units): the replays above in a
    fresh process with the knob set (the library reads it once)."""
    k, v = env.split("=")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-p", "no:cacheprovider", "-x",
                        "tests/test_schedule.py::test_stream_through_schedule_replays_to_oracle"],
                       cwd=root, env={**os.environ, k: v}, capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]


@pytest.mark.parametrize("dims,td,nslots,runs,ns", [
    ((16, 16, 128), (8, 8, 32), 30, [5], 2),          # one pass, units of 16 planes
    ((16, 16, 128), (8, 8, 32), 30, [12, 3], 3),      # two runs
    ((16, 8, 96), (8, 4, 16), 46, [40], 2),           # several passes (k <= tz = 16)
    ((8, 8, 64), (8, 8, 8), 14, [7, 2], 1),           # units = tile layers, U = 8
    ((8, 8, 48), (8, 8, 8), 12, [5], 2),              # U = 6, ring of 3
])
def test_ooc_stream_through_replays_to_oracle(dims, td, nslots, runs, ns):
    """Out-of-core heat runs with a budget below the resident footprint take
    the temporally blocked stream-through (passes of k >= 2 steps over units
    of planes with a ring of input units); replayed in random valid orders
    they give the oracle bit-exactly, and each pass moves every cell across
    the link once per direction."""
    b = _budget_for(dims, td, nslots, sched="stream")
    d = _run_and_replay(dims, td, runs, ns, seeds=(0, 1, 2), sched="stream", device_budget_bytes=b)
    ops = [op[0] for op in d.trace()]
    assert "sweep_u" in ops and "h2d_pack" in ops, sorted(set(ops))
    cells = dims[0] * dims[1] * dims[2]
    st = d.stats()
    assert st["bytes_h2d"] % (cells * 8) == 0 and st["bytes_h2d"] == st["bytes_d2h"]
    assert st["bytes_h2d"] // (cells * 8) < sum(runs)  # fewer link passes than steps


# ----------------------------------------------- residency protocol
def _trace_through_state_machine(trace, nslots):
    """Feed libtiles' own requests — (tile, pointer) of every kernel, in issue
    order — through the cache-list state machine of P:L88-L90
    (oracle.ResidencyOracle with dirty tracking, reading R10) and require the
    library's hit / h2d / d2h / drop ops to be exactly the ones the state
    machine emits for them, op for op. The pointer of a request is the
    library's choice (P:L79 leaves the region -> pointer map unspecified);
    a D2H of the tile just computed is a write-through, i.e. a GPU-disabled
    request; D2Hs issued by tile_sync are GPU-disabled requests too,
    after which no tile may be left newer on the device than on the host."""
    ro = oracle.ResidencyOracle(nslots, track_dirty=True)
    pending, last, nreq = [], None, 0
    for name, _st, a, b, c, _d in trace:
        if name in ("hit", "h2d", "d2h", "drop"):
            if name in ("h2d", "d2h"):
                assert c == 1, "the cache schedule moves one tile per copy"
            if name == "d2h" and a == last and not pending:
                n0 = len(ro.trace)
                ro.cpu_request(a)
                assert ro.trace[n0:] == [("d2h", a, b)], ("write-through", a, b, ro.trace[n0:])
                last = None
                continue
            pending.append((name, a, b))
            last = None
        elif name in ("kernel", "kernel2", "pointwise"):
            n0 = len(ro.trace)
            if name == "pointwise":
                ro.gpu_request(a, writes=True, slot=b)
            else:
                ro.jacobi_request(a, b, c)
            got = [e for e in ro.trace[n0:] if e[0] != "compute"]
            assert got == pending, (name, a, b, c, got, pending)
            pending, last, nreq = [], a, nreq + 1
        elif name == "sync":  # host sync: D2Hs queued since the last kernel were host requests
            for pn, pa, pb in pending:
                assert pn == "d2h", (pn, pa, pb)
                n0 = len(ro.trace)
                ro.cpu_request(pa)
                assert ro.trace[n0:] == [("d2h", pa, pb)]
            pending, last = [], None
        else:
            assert name in ("record", "wait", "faces_h2d", "halo"), name
    assert not pending, pending
    assert not any(ro.dirty), "tile_sync left device-only data"
    return ro, nreq


def test_fig7_residency_trace_matches_state_machine():
    """The Fig. 7 scenario: the compute-intensive kernel over
    4 regions with device memory limited to 2, 2 streams, step-major."""
    dims, td = (8, 8, 16), (8, 8, 4)
    kw = dict(sched="stream", fuse_pointwise_steps=False, stream_through=-1)
    b = _budget_for(dims, td, 2, **kw)
    d = T.Domain(dims, td, dry_run=True, device_budget_bytes=b, **kw)
    d.load(np.zeros((16, 8, 8)))
    d.run(T.sincos(2), 3, 2)
    d.sync()
    ro, nreq = _trace_through_state_machine(d.trace(), 2)
    assert nreq == 12
    ops = [e[0] for e in ro.trace]
    assert ops.count("h2d") + ops.count("hit") == 12


@pytest.mark.parametrize("kind", ["heat", "pointwise"])
@pytest.mark.parametrize("nslots,ns,steps", [(2, 1, [3]), (3, 2, [2, 1]), (5, 1, [2]), (6, 3, [1, 2]),
                                             (12, 2, [3]), (20, 4, [2, 2]), (17, 1, [4])])
def test_stream_residency_trace_matches_state_machine(kind, nslots, ns, steps):
    dims, td = (16, 16, 16), (8, 8, 4)   # 16 tiles
    kw = dict(sched="stream", stream_through=-1)
    b = _budget_for(dims, td, nslots, **kw)
    d = T.Domain(dims, td, dry_run=True, device_budget_bytes=b, fuse_pointwise_steps=False, **kw)
    d.load(np.zeros((16, 16, 16)))
    for s in steps:
        d.run(T.heat7() if kind == "heat" else T.sincos(1), s, ns)
    d.sync()
    _, nreq = _trace_through_state_machine(d.trace(), nslots)
    assert nreq == 16 * sum(steps)


def test_state_machine_check_catches_a_wrong_trace():
    """The comparison is not vacuous: dropping a write-back, or turning a
    drop of a dirty tile into a copy-free eviction, fails it."""
    dims, td = (16, 16, 16), (8, 8, 4)
    kw = dict(sched="stream", stream_through=-1)
    b = _budget_for(dims, td, 3, **kw)
    d = T.Domain(dims, td, dry_run=True, device_budget_bytes=b, **kw)
    d.load(np.zeros((16, 16, 16)))
    d.run(T.heat7(), 2, 1)
    d.sync()
    tr = d.trace()
    _trace_through_state_machine(tr, 3)
    i = next(i for i, op in enumerate(tr) if op[0] == "d2h")
    with pytest.raises(AssertionError):
        _trace_through_state_machine(tr[:i] + tr[i + 1:], 3)
    j = next(i for i, op in enumerate(tr) if op[0] == "drop")
    bad = list(tr)
    bad[j] = ("hit",) + tuple(bad[j][1:])
    with pytest.raises((AssertionError, ValueError)):
        _trace_through_state_machine(bad, 3)


@pytest.mark.parametrize("first", ["sincos", "heat"])
@pytest.mark.parametrize("nslots", [3, 24])
def test_stream_pointwise_then_heat_without_sync(first, nslots):
    """Out-of-core runs of different kernels back to back with no tile_sync
    between them: a heat run after a pointwise run needs its ghost faces from
    the pointwise run's results — including the tiles still dirty on the
    device and the write-backs still in flight — and a heat -> sincos ->
    heat sequence must not reuse faces extracted before the sincos run."""
    dims, td = (32, 16, 24), (8, 8, 4)
    kw = dict(sched="stream", stream_through=-1, fuse_pointwise_steps=False)
    b = _budget_for(dims, td, nslots, **kw)
    u0 = synth.uniform_grid(*dims, 42)
    runs = [("sincos", 1, 1), ("heat", 2, 0)] if first == "sincos" else \
        [("heat", 1, 0), ("sincos", 1, 1), ("heat", 2, 0)]
    ref = u0.copy()
    for kind, steps, K in runs:
        ref = oracle.sincos_c(ref, K, steps) if kind == "sincos" else oracle.heat_c(ref, ALPHA, steps)
    for seed in (0, 1, 2):
        d = T.Domain(dims, td, dry_run=True, device_budget_bytes=b, **kw)
        d.load(u0)
        for kind, steps, K in runs:
            d.run(T.sincos(K) if kind == "sincos" else T.heat7(ALPHA), steps, 2)
        d.sync()
        G = Geometry(dims, td)
        rep = Replayer(G, split_tiles(G, u0), ALPHA)
        rep.replay(d.trace(), seed)
        assert np.array_equal(rep.grid(), ref), np.abs(rep.grid() - ref).max()
        _trace_through_state_machine(d.trace(), nslots)


@pytest.mark.parametrize("dims,td,T,ns,runs_after", [
    ((16, 8, 64), (8, 4, 16), 3, 2, []),          # chunk 16 = tz / 1, bootstrap 16 planes
    ((16, 8, 128), (8, 4, 16), 20, 3, [2]),       # T > tz: nlo = 3 scratch layers
    ((16, 16, 96), (8, 8, 32), 17, 1, [5]),       # B = 48 (not a layer multiple)
    ((8, 8, 64), (8, 8, 8), 7, 2, [3, 1]),        # tz = 8 < chunk: c = 8
    ((16, 8, 80), (8, 8, 16), 1, 2, []),          # T = 1: no bootstrap sweep
    ((16, 8, 160), (8, 4, 32), 40, 4, [])])       # long run, 3 layers of scratch
def test_wavefront_schedule_replays_to_oracle(dims, td, T, ns, runs_after):
    """Fresh-upload heat runs on the time-skewed wavefront (run_wavefront):
    replayed in random valid orders the trace gives the untiled oracle
    bit-exactly — a missing dependency, a WAR on a level buffer or a wrong
    scratch mapping reads NaN or stale planes — moves every cell across the
    link exactly once per direction, leaves the domain resident for the
    following runs, and sweeps each cell once per step plus the ~T^2 bootstrap."""
    d = _run_and_replay(dims, td, [T] + runs_after, ns, seeds=(0, 1, 2), wavefront=1)
    assert d.get_info()["resident"]
    # adversarial orders: uploads as late as their waits allow (a sweep that
    # does not wait for its chunk reads NaN), then sweeps as late as possible
    # (a D2H or copy that does not wait for its iteration moves stale planes)
    for lazy in (("h2d_part",), ("wsweep",)):
        _run_and_replay(dims, td, [T], ns, seeds=(5,), wavefront=1, lazy=lazy)
    # the wavefront run on its own: ops, link bytes and swept cells
    d2 = T_run_dry(dims, td, T, ns, wavefront=1)
    ops = [op[0] for op in d2.trace()]
    assert "d2h_planes" in ops and "sweep" not in ops
    assert "wsweep2" not in ops   # one level per pass (two level buffers)
    st = d2.stats()
    cells = dims[0] * dims[1] * dims[2]
    assert st["bytes_h2d"] == cells * 8 and st["bytes_d2h"] == cells * 8
    assert d2.get_info()["last_schedule"] == 6
    planes = 0
    for op in d2.trace():
        if op[0] in ("wsweep", "wsweep2"):
            lo, hi = wsweep_range(op[4])
            planes += (hi - lo) * (2 if op[0] == "wsweep2" else 1)
    assert planes == dims[2] * T + sum(max(0, 2 * T - 2 * t) for t in range(1, T))
    # two levels per pass (three level buffers, wavefront = 2) replays exactly
    # too, in random and adversarial orders, with the same swept planes
    d3 = _run_and_replay(dims, td, [T], ns, seeds=(7, 8), wavefront=2)
    _run_and_replay(dims, td, [T], ns, seeds=(9,), wavefront=2, lazy=("wsweep",))
    ops3 = [op[0] for op in d3.trace()]
    assert ("wsweep2" in ops3) == (T >= 2)
    planes3 = 0
    for op in d3.trace():
        if op[0] in ("wsweep", "wsweep2"):
            lo, hi = wsweep_range(op[4])
            planes3 += (hi - lo) * (2 if op[0] == "wsweep2" else 1)
    assert planes3 == planes


@pytest.mark.parametrize("T_", [5, 20])
def test_wavefront_512_wide_default_two_levels(T_):
    """On grids 512 wide with 64-wide tiles the wavefront runs two levels per
    pass by default (heat2_band_slab on the GPU); wavefront = 3 keeps one
    level per pass. Both replay to the oracle bit-exactly."""
    dims, td = (512, 8, 128), (64, 4, 16)
    d = _run_and_replay(dims, td, [T_, 2], 2, seeds=(0, 1), wavefront=1)
    d1 = T_run_dry(dims, td, T_, 2, wavefront=1)
    assert "wsweep2" in [op[0] for op in d1.trace()]
    d3 = _run_and_replay(dims, td, [T_], 2, seeds=(2,), wavefront=3)
    assert "wsweep2" not in [op[0] for op in d3.trace()] and d3.get_info()["last_schedule"] == 6


@pytest.mark.parametrize("T_", [70, 71])
def test_large_T_split_wavefront_replays(T_):
    """A fresh upload at large T on a grid 512 wide: a wavefront of Tw levels
    during the upload (no D2H), the middle steps in pairs on heat2_band, a
    wavefront of the last Tw (+1) levels during the download (no H2D): every
    cell crosses the link once per direction, and random valid orders give
    the oracle bit-exactly."""
    dims, td = (512, 8, 128), (64, 4, 16)   # wavefront up to T = 56 here: Tw = 32
    d = _run_and_replay(dims, td, [T_, 2], 2, seeds=(0, 1))
    d1 = T_run_dry(dims, td, T_, 2)
    ops = [op[0] for op in d1.trace()]
    assert d1.get_info()["last_schedule"] == 8
    assert ops.count("band2") == (T_ - 64) // 2
    st = d1.stats()
    cells = dims[0] * dims[1] * dims[2]
    assert st["bytes_h2d"] == cells * 8 and st["bytes_d2h"] == cells * 8


@pytest.mark.parametrize("case", range(80))
def test_random_shapes_and_options_replay_to_oracle(case):
    """Seeded random small shapes, ghost widths, boundary conditions, device
    budgets and schedule options; the dry-run traces of a few runs replayed
    in random valid orders give the oracle bit-exactly."""
    import random
    rng = random.Random(700 + case)
    def dim():
        n = rng.choice([8, 16, 24, 32])
        return n, rng.choice([t for t in (4, 8, 16) if n % t == 0])
    (nx, tx), (ny, ty), (nz, tz) = dim(), dim(), dim()
    dims, td = (nx, ny, nz), (tx, ty, tz)
    bc = rng.choice(["periodic", "periodic", "dirichlet"])
    ghost = rng.choice([1, 1, 2])
    kw = {"wavefront": rng.choice([-1, 0, 1, 2, 3]), "stream_through": rng.choice([-1, 0, 1]),
          "two_step": rng.choice([-1, 0, 1])}
    if rng.random() < 0.4:
        kw["sched"] = "stream"
        try:
            kw["device_budget_bytes"] = _budget_for(dims, td, rng.choice([3, 4, 6]), sched="stream", bc=bc,
                                                    ghost=ghost)
        except Exception:
            pytest.skip("no stream budget for this shape")
    runs = [rng.choice([1, 2, 3, 5]) for _ in range(rng.choice([1, 2, 3]))]
    try:
        T.Domain(dims, td, dry_run=True, bc=bc, ghost=ghost, **kw).free()
    except T.TileError:
        pytest.skip("shape not accepted")
    _run_and_replay(dims, td, runs, rng.choice([1, 2, 3]), seeds=(case,), bc=bc, ghost=ghost, **kw)


@pytest.mark.parametrize("case", range(16))
def test_random_band_shapes_replay_to_oracle(case):
    """Seeded random 512-wide shapes (the band kernels' domain: heat2_band,
    the two-level wavefront, the split large-T schedule, two sweeps per
    stream-through kernel with two_step = 1) and run sequences, replayed."""
    import random
    rng = random.Random(900 + case)
    ny = rng.choice([4, 8, 12])
    ty = rng.choice([t for t in (4, 8, 12) if ny % t == 0])
    nz = rng.choice([8, 16, 32, 64, 96, 128])
    tz = rng.choice([t for t in (2, 4, 8, 16, 32) if nz % t == 0])
    dims, td = (512, ny, nz), (64, ty, tz)
    kw = {"two_step": rng.choice([0, 0, 1])}
    runs = [rng.choice([1, 2, 3, 5, 8, 20, 40, 70]) for _ in range(rng.choice([1, 2]))]
    try:
        T.Domain(dims, td, dry_run=True, **kw).free()
    except T.TileError:
        pytest.skip("shape not accepted")
    d = _run_and_replay(dims, td, runs, rng.choice([1, 2, 4]), seeds=(case,), **kw)
    assert d.get_info()["last_schedule"] in (1, 2, 6, 7, 8)


def T_run_dry(dims, td, steps, ns, **kw):
    d = T.Domain(dims, td, dry_run=True, **kw)
    d.load(np.zeros(dims[::-1]))
    d.run(T.heat7(ALPHA), steps, ns)
    d.sync()
    return d


def test_wavefront_cost_model_choice():
    """The fresh-upload schedule choice (cost model, link-plane units): at
    C2 shape, stream-through at T = 10, the wavefront at T = 32..100, the
    batched schedule where the seam's cone covers the ring."""
    dims, td = (512, 512, 512), (64, 64, 64)
    sched = {}
    for steps in (10, 32, 64, 100, 300):
        d = T.Domain(dims, td, dry_run=True)
        d.invalidate()
        d.run(T.heat7(ALPHA), steps, 4)
        sched[steps] = d.get_info()["last_schedule"]
        d.free()
    assert sched[10] == 2 and sched[32] == 6 and sched[64] == 6 and sched[100] == 6
    assert sched[300] == 8   # wavefront (upload) + two-step passes + wavefront (download)


def test_cost_model_ratio_option_and_report():
    """tile_options.sweep_link_ratio sets the fresh-upload cost model's
    sweep / link time ratio (dry runs: else the 0.021 fit); tile_info
    reports it, and it moves the schedule choice: a slow sweep (large ratio)
    sends a T = 32 run to the batched schedule, a fast one to the wavefront."""
    dims, td = (512, 512, 512), (64, 64, 64)
    d = T.Domain(dims, td, dry_run=True)
    assert abs(d.get_info()["sweep_link_ratio"] - 0.021) < 1e-12
    got = {}
    # (at C2's shape both the wavefront and the batched middle steps run two
    # levels per kernel, so only a much slower sweep tips T = 32 to batched:
    # the wavefront's T^2 seam bootstrap then dominates)
    for r in (0.005, 0.021, 5.0):
        d = T.Domain(dims, td, dry_run=True, sweep_link_ratio=r)
        assert d.get_info()["sweep_link_ratio"] == r
        d.invalidate()
        d.run(T.heat7(ALPHA), 32, 4)
        got[r] = d.get_info()["last_schedule"]
    assert got[0.005] in (2, 6) and got[0.021] == 6 and got[5.0] == 1
