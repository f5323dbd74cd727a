"""Replay of libtiles' dry-run op trace on the CPU (test infrastructure).

The scheduler's trace (tile_trace) lists every operation it would issue on
every stream, plus event records and waits. This replayer executes the ops
in a RANDOM order that respects exactly the CUDA semantics the real executor
relies on: each stream is a FIFO, and a wait blocks its stream until the
most recent record of that event issued BEFORE the wait has executed.
Data ops move NumPy arrays between a simulated host store, device slots and
face buffers; kernels apply the ORACLE's arithmetic (oracle.heat_np) to a
tile expanded with ghost cells taken from the neighbours' exported faces.
If the scheduler misses a dependency, some random order reads stale or
future data and the final grid differs from the untiled oracle.

Ghost-source neighbours are derived here from the tile grid (periodic wrap /
Dirichlet halo), independently of the library's own face tables.
"""
import random

import numpy as np

import oracle

XM, XP, YM, YP, ZM, ZP = range(6)


class Geometry:
    def __init__(self, dims, tile_dims, nranks=1, rank=0, bc=0, ghost=1):
        self.depth = 1 if ghost < 2 else 2   # face depth D
        self.g = tuple(dims)
        self.t = tuple(tile_dims)
        self.nranks, self.rank, self.bc = nranks, rank, bc
        self.l = (dims[0], dims[1], dims[2] // nranks)
        self.n = tuple(self.l[a] // self.t[a] for a in range(3))
        self.ntiles = self.n[0] * self.n[1] * self.n[2]
        self.zoff = self.l[2] * rank

    def coords(self, k):
        return k % self.n[0], (k // self.n[0]) % self.n[1], k // (self.n[0] * self.n[1])

    def tid(self, ix, iy, iz):
        return (iz * self.n[1] + iy) * self.n[0] + ix

    def neighbour(self, k, f):
        """('tile', id) | ('dirichlet', None) | ('halo', 0|1, pos)."""
        c = list(self.coords(k))
        axis, step = f // 2, (1 if f & 1 else -1)
        c[axis] += step
        if 0 <= c[axis] < self.n[axis]:
            return ("tile", self.tid(*c))
        if axis < 2 or self.nranks == 1:
            if self.bc == 1:
                return ("dirichlet", None)
            c[axis] %= self.n[axis]
            return ("tile", self.tid(*c))
        pos = c[1] * self.n[0] + c[0]
        if step < 0:
            if self.rank == 0 and self.bc == 1:
                return ("dirichlet", None)
            return ("halo", 0, pos)
        if self.rank == self.nranks - 1 and self.bc == 1:
            return ("dirichlet", None)
        return ("halo", 1, pos)


def wsweep_range(c):
    """lo, hi of a TILE_OP_WSWEEP (two signed 32-bit halves of c)."""
    cu = c & 0xFFFFFFFFFFFFFFFF
    s32 = lambda v: v - (1 << 32) if v & 0x80000000 else v
    return s32(cu & 0xFFFFFFFF), s32(cu >> 32)


def faces_of(u, D=1):
    """The D boundary layers of a tile per face, in increasing coordinate
    order: x-faces (tz,ty,D), y-faces (tz,D,tx), z-faces (D,ty,tx)."""
    return [u[:, :, :D].copy(), u[:, :, -D:].copy(), u[:, :D, :].copy(), u[:, -D:, :].copy(),
            u[:D].copy(), u[-D:].copy()]


def nearest(plane_stack, f):
    """Layer of a neighbour's export adjacent to the reading tile's face f
    (the export is of the opposite face): f = x- reads the last layer of the
    x+ export, f = x+ the first layer of the x- export, etc."""
    last = (f & 1) == 0
    if f <= 1:
        return plane_stack[:, :, -1] if last else plane_stack[:, :, 0]
    if f <= 3:
        return plane_stack[:, -1, :] if last else plane_stack[:, 0, :]
    return plane_stack[-1] if last else plane_stack[0]


class Replayer:
    def __init__(self, geo, host_tiles, alpha, ext=None, comm=None):
        """host_tiles: list of (tz,ty,tx) arrays (the pinned store); ext: the
        Dirichlet extended input of this rank's slab; comm: halo callback."""
        self.G = geo
        self.host = [h.copy() for h in host_tiles]
        self.alpha = alpha
        self.ext = ext
        self.slots = {}
        self.slabs = {}
        self.sub = {}      # packed unit results: (base slot, tile-in-layer) -> (np, ty, tx)
        self.loc = {}      # tile -> device slot of its last H2D
        self.faces = {}
        self.halo = {}
        self.comm = comm
        self.peers = {}    # rank -> Replayer (joint multi-rank replay, fused pushes)
        # multi-rank stream-through (comm_peer.cu peer_st_halo): halo layers
        # [0] lo (the lower rank's top planes), [1] hi (the upper rank's bottom
        # planes) and their counters: S (arrived epoch) and CR (credit: the
        # receiver on that side released the epoch's layer I pushed)
        self.pending2 = {}  # stream -> parameters of a two-level sweep (TILE_OP_WSWEEP2)
        self.st = {0: None, 1: None}
        self.st_arrived = {0: 0, 1: 0}
        self.st_credit = {0: 0, 1: 0}

    def dirichlet_face(self, k, f):
        G = self.G
        ix, iy, iz = G.coords(k)
        tx, ty, tz = G.t
        ox, oy, oz = ix * tx + 1, iy * ty + 1, iz * tz + 1
        e = self.ext
        if f == XM:
            return e[oz:oz + tz, oy:oy + ty, ox - 1]
        if f == XP:
            return e[oz:oz + tz, oy:oy + ty, ox + tx]
        if f == YM:
            return e[oz:oz + tz, oy - 1, ox:ox + tx]
        if f == YP:
            return e[oz:oz + tz, oy + ty, ox:ox + tx]
        if f == ZM:
            return e[oz - 1, oy:oy + ty, ox:ox + tx]
        return e[oz + tz, oy:oy + ty, ox:ox + tx]

    def ghost(self, k, f, par):
        src = self.G.neighbour(k, f)
        if src[0] == "tile":
            return nearest(self.faces[(src[1], f ^ 1, par)], f)
        if src[0] == "dirichlet":
            return self.dirichlet_face(k, f)
        return nearest(self.halo[(src[1], par)][src[2]], f)

    def kernel(self, k, sin, sout, par):
        u = self.slots[sin]
        tz, ty, tx = u.shape
        e = np.zeros((tz + 2, ty + 2, tx + 2))
        e[1:-1, 1:-1, 1:-1] = u
        e[1:-1, 1:-1, 0] = self.ghost(k, XM, par)
        e[1:-1, 1:-1, -1] = self.ghost(k, XP, par)
        e[1:-1, 0, 1:-1] = self.ghost(k, YM, par)
        e[1:-1, -1, 1:-1] = self.ghost(k, YP, par)
        e[0, 1:-1, 1:-1] = self.ghost(k, ZM, par)
        e[-1, 1:-1, 1:-1] = self.ghost(k, ZP, par)
        v = oracle.heat_np(e, self.alpha, 1, oracle.BC_DIRICHLET)[1:-1, 1:-1, 1:-1]
        self.slots[sout] = v
        for f, plane in enumerate(faces_of(v, self.G.depth)):
            self.faces[(k, f, par ^ 1)] = plane

    def kernel_direct(self, k, sin, sout, par, push=False):
        """Single step with direct ghosts (TILE_OP_KERNELD): y/z ghosts of a
        neighbour tile of this rank come from that tile's interior in the
        same buffer array as `sin` (resident layout: tile j in slot base + j),
        everything else from faces as in `kernel`. Exports the x faces and,
        multi-rank, the z- face of layer 0 and the z+ face of the top layer;
        the other exports of parity par^1 become NaN (stale), so a later read
        of them poisons the grid."""
        G = self.G
        base = sin - k
        u = self.slots[sin]
        tz, ty, tx = u.shape

        def g(f):
            src = G.neighbour(k, f)
            if f >= YM and src[0] == "tile":
                nb = self.slots[base + src[1]]
                return {YM: nb[:, -1, :], YP: nb[:, 0, :], ZM: nb[-1], ZP: nb[0]}[f]
            return self.ghost(k, f, par)
        e = np.zeros((tz + 2, ty + 2, tx + 2))
        e[1:-1, 1:-1, 1:-1] = u
        e[1:-1, 1:-1, 0] = g(XM)
        e[1:-1, 1:-1, -1] = g(XP)
        e[1:-1, 0, 1:-1] = g(YM)
        e[1:-1, -1, 1:-1] = g(YP)
        e[0, 1:-1, 1:-1] = g(ZM)
        e[-1, 1:-1, 1:-1] = g(ZP)
        v = oracle.heat_np(e, self.alpha, 1, oracle.BC_DIRICHLET)[1:-1, 1:-1, 1:-1]
        self.slots[sout] = v
        lt = G.n[0] * G.n[1]
        multi = G.nranks > 1
        keep = {XM, XP}
        if multi and k < lt:
            keep.add(ZM)
        if multi and k >= G.ntiles - lt:
            keep.add(ZP)
        for f, plane in enumerate(faces_of(v, G.depth)):
            self.faces[(k, f, par ^ 1)] = plane if f in keep else np.full(plane.shape, np.nan)
        if push:  # fused halo push straight into the neighbour ranks' receive buffers
            up, dn = halo_peers(G)
            fz = faces_of(v, G.depth)
            if dn is not None and k < lt:
                self.peers[dn].push((1, par ^ 1), k, fz[ZM])
            if up is not None and k >= G.ntiles - lt:
                self.peers[up].push((0, par ^ 1), k - (G.ntiles - lt), fz[ZP])

    def push(self, key, pos, plane):
        G = self.G
        lt = G.n[0] * G.n[1]
        cur = list(self.halo.get(key, [None] * lt))
        cur[pos] = plane.copy()
        self.halo[key] = cur

    # ------------------------------------------------ two-step pass (ghost 2)
    def edge_value(self, k, x, y, z, par):
        """Value of tile-local cell (x, y, z) of tile k (outside the tile in
        two axes) at the read parity, taken from the owning tile's exported
        depth-2 faces, or the Dirichlet halo; NaN if never needed."""
        G = self.G
        tx, ty, tz = G.t
        ix, iy, iz = G.coords(k)
        gc = [ix * tx + x, iy * ty + y, G.zoff + iz * tz + z]
        out = [not (0 <= gc[a] < G.g[a]) for a in range(3)]
        if any(out):
            if G.bc == 1:
                if sum(out) >= 2:
                    return np.nan
                return self.ext[gc[2] - G.zoff + 1, gc[1] + 1, gc[0] + 1]
            gc = [gc[a] % G.g[a] for a in range(3)]
        gz = gc[2] - G.zoff
        owner = G.tid(gc[0] // tx, gc[1] // ty, gz // tz)
        lx, ly, lz = gc[0] % tx, gc[1] % ty, gz % tz
        if lx < 2:
            return self.faces[(owner, XM, par)][lz, ly, lx]
        if lx >= tx - 2:
            return self.faces[(owner, XP, par)][lz, ly, lx - (tx - 2)]
        if ly < 2:
            return self.faces[(owner, YM, par)][lz, ly, lx]
        if ly >= ty - 2:
            return self.faces[(owner, YP, par)][lz, ly - (ty - 2), lx]
        raise AssertionError("edge cell is not a boundary cell of its owner")

    def kernel2(self, k, sin, sout, par):
        G = self.G
        u = self.slots[sin]
        tz, ty, tx = u.shape
        e = np.full((tz + 4, ty + 4, tx + 4), np.nan)
        e[2:-2, 2:-2, 2:-2] = u
        dirichlet = {}
        for f in range(6):
            src = G.neighbour(k, f)
            if src[0] == "tile":
                slab = self.faces[(src[1], f ^ 1, par)]
            elif src[0] == "dirichlet":
                dirichlet[f] = self.dirichlet_face(k, f)
                continue
            else:
                raise AssertionError("two-step passes are single-rank")
            if f == XM:
                e[2:-2, 2:-2, 0:2] = slab
            elif f == XP:
                e[2:-2, 2:-2, -2:] = slab
            elif f == YM:
                e[2:-2, 0:2, 2:-2] = slab
            elif f == YP:
                e[2:-2, -2:, 2:-2] = slab
            elif f == ZM:
                e[0:2, 2:-2, 2:-2] = slab
            else:
                e[-2:, 2:-2, 2:-2] = slab

        def set_ring(arr):
            for f, plane in dirichlet.items():
                if f == XM:
                    arr[2:-2, 2:-2, 1] = plane
                elif f == XP:
                    arr[2:-2, 2:-2, -2] = plane
                elif f == YM:
                    arr[2:-2, 1, 2:-2] = plane
                elif f == YP:
                    arr[2:-2, -2, 2:-2] = plane
                elif f == ZM:
                    arr[1, 2:-2, 2:-2] = plane
                else:
                    arr[-2, 2:-2, 2:-2] = plane
        set_ring(e)
        # edge lines: one cell outside in two axes
        for a, b in ((0, 1), (0, 2), (1, 2)):
            line = 3 - a - b
            n_line = (tx, ty, tz)[line]
            for va in (-1, (tx, ty, tz)[a]):
                for vb in (-1, (tx, ty, tz)[b]):
                    for i in range(n_line):
                        c = [0, 0, 0]
                        c[a], c[b], c[line] = va, vb, i
                        e[c[2] + 2, c[1] + 2, c[0] + 2] = self.edge_value(k, c[0], c[1], c[2], par)
        with np.errstate(invalid="ignore"):
            e1 = oracle.heat_np(e, self.alpha, 1, oracle.BC_DIRICHLET)
            set_ring(e1)
            e2 = oracle.heat_np(e1, self.alpha, 1, oracle.BC_DIRICHLET)
        v = e2[2:-2, 2:-2, 2:-2]
        assert not np.isnan(v).any(), "two-step pass read a ghost cell it was not given"
        self.slots[sout] = v
        for f, plane in enumerate(faces_of(v, G.depth)):
            self.faces[(k, f, par ^ 1)] = plane

    def execute(self, op, snapshot_faces):
        name, st, a, b, c, d = op
        if name == "h2d":
            for i in range(c):
                self.slots[b + i] = self.host[a + i].copy()
                self.loc[a + i] = b + i
        elif name == "d2h":
            for i in range(c):
                self.host[a + i] = self.slots[b + i].copy()
        elif name == "kernel":
            self.kernel(a, b, c, d)
        elif name == "kernel2":
            self.kernel2(a, b, c, d)
        elif name == "kerneld":
            self.kernel_direct(a, b, c, d & 0xff, bool(d & 0x100))
        elif name == "extract":
            for f, plane in enumerate(faces_of(self.slots[b], self.G.depth)):
                self.faces[(a, f, d)] = plane
        elif name == "faces_h2d":
            if d >= 0:
                for (k, f), plane in snapshot_faces.items():
                    self.faces[(k, f, d)] = plane.copy()
        elif name == "pointwise":
            self.slots[b] = oracle.sincos_c(self.slots[b], c, 1)
        elif name == "halo":
            self.comm(self, d)
        elif name == "copy":
            for i in range(c):
                self.slots[b + i] = self.slots[a + i].copy()
            for t, sl in list(self.loc.items()):
                if b <= sl < b + c:
                    pass
        elif name == "sweep":
            # a: slab slot, or -1-bit = the resident array with slab plane 0
            # at local z = d; b: slab slot, or -1-slot = packed sub-tiles
            # receiving planes [lo, hi)
            lo, hi = c & 0xffffffff, c >> 32
            src = self.slabs[a] if a >= 0 else self.gather(hi + 1, d)
            if b >= 0:
                self.slabs[b] = self.sweep(src, self.slabs.get(b), lo, hi)
            else:
                new = self.sweep(src, None, lo, hi)
                G = self.G
                tx, ty, tz = G.t
                for i in range(G.n[0] * G.n[1]):
                    ix, iy = i % G.n[0], i // G.n[0]
                    self.sub[(-b - 1, i)] = new[lo:hi, iy * ty:(iy + 1) * ty, ix * tx:(ix + 1) * tx].copy()
        elif name == "sweep2s":
            # two sweeps in one kernel: level 1 on [lo, hi) (not stored),
            # level 2 on [lo+1, hi-1) into b (codes as for "sweep")
            lo, hi = c & 0xffffffff, c >> 32
            src = self.slabs[a] if a >= 0 else self.gather(hi + 1, d)
            assert a < 0 or a != b, "two-sweep kernel writes the slab it reads"
            lev1 = self.sweep(src, None, lo, hi)
            lo2, hi2 = lo + 1, hi - 1
            if b >= 0:
                self.slabs[b] = self.sweep(lev1, self.slabs.get(b), lo2, hi2)
            else:
                new = self.sweep(lev1, None, lo2, hi2)
                G = self.G
                tx, ty, tz = G.t
                for i in range(G.n[0] * G.n[1]):
                    ix, iy = i % G.n[0], i // G.n[0]
                    self.sub[(-b - 1, i)] = new[lo2:hi2, iy * ty:(iy + 1) * ty, ix * tx:(ix + 1) * tx].copy()
        elif name == "sweep_u":
            # source: units u-1, u, u+1 as packed sub-tiles (slots in b);
            # a: destination code as for "sweep"
            lo, hi = c & 0xffffffff, c >> 32
            u, un = d & 0xffffffff, d >> 32
            slots = (b & 0x1fffff, (b >> 21) & 0x1fffff, b >> 42)
            G = self.G
            tx, ty, tz = G.t
            nz, U = G.l[2], G.l[2] // un
            k = (hi + 1 - un) // 2
            src = np.empty((hi + 1, G.l[1], G.l[0]))
            for p in range(hi + 1):
                gz = (u * un - k + p) % nz
                iu = gz // un
                slot = slots[(iu - u + 1) % U if U > 2 else (0 if iu != u else 1)]
                for i in range(G.n[0] * G.n[1]):
                    ix, iy = i % G.n[0], i // G.n[0]
                    src[p, iy * ty:(iy + 1) * ty, ix * tx:(ix + 1) * tx] = self.sub[(slot, i)][gz - iu * un]
            if a >= 0:
                self.slabs[a] = self.sweep(src, self.slabs.get(a), lo, hi)
            else:
                new = self.sweep(src, None, lo, hi)
                for i in range(G.n[0] * G.n[1]):
                    ix, iy = i % G.n[0], i // G.n[0]
                    self.sub[(-a - 1, i)] = new[lo:hi, iy * ty:(iy + 1) * ty, ix * tx:(ix + 1) * tx].copy()
        elif name == "wsweep":
            lo, hi = wsweep_range(c)
            G = self.G
            # one kernel reads [lo-1, hi+1) and writes [lo, hi) with all its CTAs
            # at once: the two must not share memory (an in-kernel WAR race the
            # op-level replay could not otherwise see)
            rd = {self._wave_loc(a, p, d) for p in range(lo - 1, hi + 1)}
            wr = {self._wave_loc(b, p, d) for p in range(lo, hi)}
            assert not rd & wr, "sweep writes planes it reads (in-kernel race)"
            blk = np.stack([self.wave_get(a, p, d) for p in range(lo - 1, hi + 1)])
            new = self.sweep(blk, None, 1, hi - lo + 1)
            for p in range(lo, hi):
                self.wave_set(b, p, d, new[p - lo + 1])
        elif name == "wsweep2":  # parameters of a two-level pass; executed at its _dst record
            self.pending2[st] = (a, b, c, d)
        elif name == "wsweep2_dst":
            # level s on [lo, hi) from view src, written to view mid only at
            # hi-2, hi-1 (mid's planes lo-2, lo-1 are read); level s+1 on
            # [lo-1, hi-1) into view a
            src, mid, cc, nlo = self.pending2.pop(st)
            lo, hi = wsweep_range(cc)
            rd = {self._wave_loc(src, p, nlo) for p in range(lo - 1, hi + 1)} | \
                 {self._wave_loc(mid, p, nlo) for p in (lo - 2, lo - 1)}
            wr = {self._wave_loc(a, p, nlo) for p in range(lo - 1, hi - 1)} | \
                 {self._wave_loc(mid, p, nlo) for p in (hi - 2, hi - 1)}
            assert not rd & wr, "two-level sweep writes memory it reads (in-kernel race)"
            blk = np.stack([self.wave_get(src, p, nlo) for p in range(lo - 1, hi + 1)])
            lev = self.sweep(blk, None, 1, hi - lo + 1)[1:hi - lo + 1]  # level s, planes lo..hi-1
            blk2 = np.concatenate([np.stack([self.wave_get(mid, lo - 2, nlo), self.wave_get(mid, lo - 1, nlo)]), lev])
            lev2 = self.sweep(blk2, None, 1, hi - lo + 1)[1:hi - lo + 1]  # level s+1, planes lo-1..hi-2
            for p in (hi - 2, hi - 1):
                self.wave_set(mid, p, nlo, lev[p - lo])
            for p in range(lo - 1, hi - 1):
                self.wave_set(a, p, nlo, lev2[p - lo + 1])
        elif name == "band2":
            # two steps of the whole periodic grid: u^{s+2} (view b) from u^s
            # (view a), two resident arrays coded as for wsweep
            nz = c >> 32
            assert (a >> 1) & 1 != (b >> 1) & 1, "heat2_band reads and writes one array"
            blk = np.stack([self.wave_get(a, p, 0) for p in range(-2, nz + 2)])
            lev1 = self.sweep(blk, None, 1, nz + 3)      # planes -1 .. nz
            lev2 = self.sweep(lev1, None, 2, nz + 2)     # planes 0 .. nz-1
            for p in range(nz):
                self.wave_set(b, p, 0, lev2[p + 2])
        elif name == "d2h_planes":
            p0, np_ = d & 0xffffffff, d >> 32
            for i in range(c):
                self.host[a + i] = self.host[a + i].copy()
                self.host[a + i][p0:p0 + np_] = self.slots[b + i][p0:p0 + np_]
        elif name == "copy_planes":
            p0, np_ = d & 0xffffffff, d >> 32
            for i in range(c):
                src = self.slots[a + i][p0:p0 + np_].copy()
                if b + i not in self.slots:
                    self.slots[b + i] = np.full(self.host[0].shape, np.nan)
                else:
                    self.slots[b + i] = self.slots[b + i].copy()
                self.slots[b + i][p0:p0 + np_] = src
        elif name == "h2d_pack":
            p0, np_ = d & 0xffffffff, d >> 32
            for i in range(c):
                self.sub[(b, i)] = self.host[a + i][p0:p0 + np_].copy()
        elif name in ("h2d_part", "d2h_part", "copy_part"):
            p0, np_ = d & 0xffffffff, d >> 32
            for i in range(c):
                if name == "h2d_part":
                    if b + i not in self.slots:
                        self.slots[b + i] = np.full(self.host[a + i].shape, np.nan)
                    self.slots[b + i][p0:p0 + np_] = self.host[a + i][p0:p0 + np_]
                    self.loc[a + i] = b + i
                elif name == "d2h_part":
                    self.host[a + i] = self.host[a + i].copy()
                    self.host[a + i][p0:p0 + np_] = self.sub[(b, i)]
                else:
                    self.slots[b + i] = self.slots[b + i].copy()
                    self.slots[b + i][p0:p0 + np_] = self.sub[(a, i)]
        # record / wait / hit / drop: no data movement

    # ------------------------------------------------- stream-through slabs
    def gather(self, planes, zbase):
        G = self.G
        tx, ty, tz = G.t
        nz = G.l[2]
        out = np.empty((planes, G.l[1], G.l[0]))
        for p in range(planes):
            gz = zbase + p
            if G.nranks > 1 and (gz < 0 or gz >= nz):  # beyond the slab: the neighbours' planes
                side = 0 if gz < 0 else 1
                layer = self.st[side]
                assert layer is not None, "stream-through read a halo layer that never arrived"
                out[p] = layer[gz + layer.shape[0]] if side == 0 else layer[gz - nz]
                continue
            gz %= nz
            iz, lz = gz // tz, gz % tz
            for iy in range(G.n[1]):
                for ix in range(G.n[0]):
                    t = G.tid(ix, iy, iz)
                    out[p, iy * ty:(iy + 1) * ty, ix * tx:(ix + 1) * tx] = self.slots[self.loc[t]][lz]
        return out

    # ------------------------------------------------------------ wavefront
    def _wave_loc(self, code, p, nlo):
        """(first slot of the tile layer, plane in the tiles) of unwrapped
        plane p in a TILE_OP_WSWEEP view: bit 0 set and p < 0: the scratch
        tile layers at slot code >> 32 (nlo of them, planes [-nlo*tz, 0));
        bit 0 set, p >= 0: the array starting at slot (code >> 1) & 0x7fffffff;
        bit 0 clear: resident array (code >> 1) & 1, wrapped."""
        G = self.G
        tz, lt, nz = G.t[2], G.n[0] * G.n[1], G.l[2]
        if code & 1 and p < 0:
            q = p + nlo * tz
            assert q >= 0, "wavefront read below its scratch"
            return (code >> 32) + (q // tz) * lt, q % tz
        if code & 1:
            assert p < nz, "wavefront view read past the ring"
            return ((code >> 1) & 0x7FFFFFFF) + (p // tz) * lt, p % tz
        gz = p % nz
        return ((code >> 1) & 1) * G.ntiles + (gz // tz) * lt, gz % tz

    def wave_get(self, code, p, nlo):
        G = self.G
        tx, ty = G.t[0], G.t[1]
        base, lz = self._wave_loc(code, p, nlo)
        plane = np.full((G.l[1], G.l[0]), np.nan)
        for i in range(G.n[0] * G.n[1]):
            t = self.slots.get(base + i)
            if t is not None:
                ix, iy = i % G.n[0], i // G.n[0]
                plane[iy * ty:(iy + 1) * ty, ix * tx:(ix + 1) * tx] = t[lz]
        return plane

    def wave_set(self, code, p, nlo, plane):
        G = self.G
        tx, ty = G.t[0], G.t[1]
        base, lz = self._wave_loc(code, p, nlo)
        for i in range(G.n[0] * G.n[1]):
            s = base + i
            t = self.slots[s].copy() if s in self.slots else np.full(self.host[0].shape, np.nan)
            ix, iy = i % G.n[0], i // G.n[0]
            t[lz] = plane[iy * ty:(iy + 1) * ty, ix * tx:(ix + 1) * tx]
            self.slots[s] = t

    def sweep(self, src, dst, lo, hi):
        """One oracle step on planes [lo, hi), periodic in x and y; planes
        lo-1 and hi are the z neighbours (oracle.heat_np on a block whose
        x/y halo is the periodic wrap and whose z halo is fixed)."""
        blk = np.pad(src[lo - 1:hi + 1], ((0, 0), (1, 1), (1, 1)), mode="wrap")
        new = oracle.heat_np(blk, self.alpha, 1, oracle.BC_DIRICHLET)[1:-1, 1:-1, 1:-1]
        n = max(src.shape[0], hi, 0 if dst is None else dst.shape[0])
        out = np.full((n,) + src.shape[1:], np.nan)  # slabs of different units differ in depth
        if dst is not None:
            out[:dst.shape[0]] = dst
        out[lo:hi] = new
        return out

    def replay(self, trace, seed, st_ready=None, st_exec=None, timeout=120.0, lazy=()):
        """Random valid order of one rank's trace; ops named in `lazy` run
        only when nothing else can (adversarial orders). st_ready / st_exec: the
        multi-process transport of stream-through halo ops (an op is runnable
        when st_ready(self, op); st_exec(self, op) performs it); while only
        such ops remain blocked the replay polls instead of failing."""
        import time
        t_end = time.time() + timeout
        rng = random.Random(seed)
        snapshot = {(k, f): p for k in range(self.G.ntiles)
                    for f, p in enumerate(faces_of(self.host[k], self.G.depth))}
        # bind each wait to the latest preceding record of its event
        last_rec = {}
        bound = {}
        for i, op in enumerate(trace):
            if op[0] == "record":
                last_rec[op[2]] = i
            elif op[0] == "wait":
                bound[i] = last_rec.get(op[2])
        queues = {}
        for i, op in enumerate(trace):
            queues.setdefault(op[1], []).append(i)
        pos = {s: 0 for s in queues}
        done = set()
        remaining = len(trace)
        syncs = [i for i, op in enumerate(trace) if op[0] == "sync"]
        while remaining:
            ready = []
            # host sync (TILE_OP_SYNC): a barrier over every stream
            barrier = next((i for i in syncs if i not in done), len(trace))
            for s, q in queues.items():
                if pos[s] < len(q):
                    i = q[pos[s]]
                    op = trace[i]
                    if i > barrier or (i == barrier and len(done) < barrier):
                        continue
                    if op[0] == "wait" and bound[i] is not None and bound[i] not in done:
                        continue
                    if op[0] == "st_halo" and st_ready is not None and not st_ready(self, op):
                        continue
                    ready.append(s)
            if not ready:
                if st_ready is not None and time.time() < t_end:
                    time.sleep(0.002)  # a neighbour's halo layer is in flight
                    continue
                raise RuntimeError("replay deadlock: no stream can make progress")
            eager = [x for x in ready if trace[queues[x][pos[x]]][0] not in lazy]
            s = rng.choice(eager or ready)
            i = queues[s][pos[s]]
            if trace[i][0] == "st_halo" and st_exec is not None:
                st_exec(self, trace[i])
            elif trace[i][0] == "sync":  # host-side face extraction reads the store now
                snapshot = {(k, f): p for k in range(self.G.ntiles)
                            for f, p in enumerate(faces_of(self.host[k], self.G.depth))}
            else:
                self.execute(trace[i], snapshot)
            done.add(i)
            pos[s] += 1
            remaining -= 1

    def grid(self):
        G = self.G
        tx, ty, tz = G.t
        out = np.empty((G.l[2], G.l[1], G.l[0]))
        for k in range(G.ntiles):
            ix, iy, iz = G.coords(k)
            out[iz * tz:(iz + 1) * tz, iy * ty:(iy + 1) * ty, ix * tx:(ix + 1) * tx] = self.host[k]
        return out


def split_tiles(geo, u):
    tx, ty, tz = geo.t
    out = []
    for k in range(geo.ntiles):
        ix, iy, iz = geo.coords(k)
        out.append(u[iz * tz:(iz + 1) * tz, iy * ty:(iy + 1) * ty, ix * tx:(ix + 1) * tx].copy())
    return out


# ------------------------------------------------------------ multi-rank
def halo_payload(rep, par):
    """Faces a rank sends in the halo exchange of parity `par`: its top
    layer's z+ exports and bottom layer's z- exports (layer-position order)."""
    G = rep.G
    lt = G.n[0] * G.n[1]
    top = [rep.faces[((G.n[2] - 1) * lt + pos, ZP, par)] for pos in range(lt)]
    bot = [rep.faces[(pos, ZM, par)] for pos in range(lt)]
    return top, bot


def halo_peers(G):
    R, r = G.nranks, G.rank
    per = G.bc == 0
    up = (r + 1) % R if (per or r < R - 1) else None
    dn = (r - 1) % R if (per or r > 0) else None
    return up, dn


def replay_ranks(reps, traces, seed, lazy=()):
    """Joint random replay of several ranks' traces; the k-th halo op of
    every rank executes together (a collective). Ops named in `lazy` run only
    when nothing else can (adversarial order: e.g. halo pushes as late as
    their dependencies allow)."""
    rng = random.Random(seed)
    for rep in reps:
        rep.peers = {r: x for r, x in enumerate(reps)}
    state = []
    for rep, tr in zip(reps, traces):
        last_rec, bound = {}, {}
        for i, op in enumerate(tr):
            if op[0] == "record":
                last_rec[op[2]] = i
            elif op[0] == "wait":
                bound[i] = last_rec.get(op[2])
        queues = {}
        for i, op in enumerate(tr):
            queues.setdefault(op[1], []).append(i)
        snapshot = {(k, f): p for k in range(rep.G.ntiles)
                    for f, p in enumerate(faces_of(rep.host[k], rep.G.depth))}
        state.append({"bound": bound, "queues": queues, "pos": {s: 0 for s in queues}, "done": set(),
                      "snap": snapshot, "syncs": [i for i, op in enumerate(tr) if op[0] == "sync"]})
    remaining = sum(len(t) for t in traces)
    while remaining:
        ready, halo_heads = [], {}
        for r, (st, tr) in enumerate(zip(state, traces)):
            barrier = next((i for i in st["syncs"] if i not in st["done"]), len(tr))
            for s, q in st["queues"].items():
                if st["pos"][s] >= len(q):
                    continue
                i = q[st["pos"][s]]
                op = tr[i]
                if i > barrier or (i == barrier and len(st["done"]) < barrier):
                    continue
                if op[0] == "wait" and st["bound"][i] is not None and st["bound"][i] not in st["done"]:
                    continue
                if op[0] in ("halo", "halo_signal"):
                    halo_heads[r] = (s, i)
                elif op[0] == "st_halo":
                    # stream-through halo op (a = 0 push, 1 wait, 2 release; b =
                    # side; c = T; d = epoch): ready when its counter condition holds
                    _, _, a, side, _, e = op
                    if (a == 0 and reps[r].st_credit[side] >= e - 1) or \
                            (a == 1 and reps[r].st_arrived[side] >= e) or a == 2:
                        ready.append((r, s, i))
                else:
                    ready.append((r, s, i))
        if len(halo_heads) == len(reps):
            ready.append(("halo", None, None))
        if not ready:
            raise RuntimeError("multi-rank replay deadlock")
        eager = [x for x in ready if x[0] == "halo" or traces[x[0]][x[2]][0] not in lazy]
        pick = rng.choice(eager or ready)
        if pick[0] == "halo":
            par = traces[0][halo_heads[0][1]][5]
            kind = traces[0][halo_heads[0][1]][0]
            payload = [halo_payload(rep, par) for rep in reps]
            for r, rep in enumerate(reps):
                assert traces[r][halo_heads[r][1]][5] == par
                assert traces[r][halo_heads[r][1]][0] == kind
                up, dn = halo_peers(rep.G)
                if kind == "halo_signal":
                    # fused: the kernels pushed the layers; the collective only orders
                    for key in ((0, par), (1, par)):
                        if (key == (0, par) and dn is not None) or (key == (1, par) and up is not None):
                            assert key in rep.halo and all(x is not None for x in rep.halo[key]), \
                                "fused halo: a boundary layer was not pushed before the signal"
                elif dn is not None:
                    rep.halo[(0, par)] = payload[dn][0]   # rank below's top layer
                if kind == "halo" and up is not None:
                    rep.halo[(1, par)] = payload[up][1]   # rank above's bottom layer
                s, i = halo_heads[r]
                state[r]["done"].add(i)
                state[r]["pos"][s] += 1
                remaining -= 1
            continue
        r, s, i = pick
        op = traces[r][i]
        if op[0] == "st_halo":
            _, _, a, side, T, e = op
            up, dn = halo_peers(reps[r].G)
            peer = reps[up if side == 1 else dn]
            if a == 0:  # my slab-end T planes of the current resident data -> the peer's layer
                nz = reps[r].G.l[2]
                peer.st[1 - side] = reps[r].gather(T, nz - T if side == 1 else 0)
                peer.st_arrived[1 - side] = e
            elif a == 2:  # released: its sender may overwrite it from now on
                reps[r].st[side] = np.full_like(reps[r].st[side], np.nan)
                peer.st_credit[1 - side] = e
        elif op[0] == "sync":
            rp = reps[r]
            state[r]["snap"] = {(k, f): p for k in range(rp.G.ntiles)
                                for f, p in enumerate(faces_of(rp.host[k], rp.G.depth))}
        else:
            reps[r].execute(op, state[r]["snap"])
        state[r]["done"].add(i)
        state[r]["pos"][s] += 1
        remaining -= 1
