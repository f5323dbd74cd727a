// domain.cpp — tile decomposition, ghost-source bookkeeping and host-side
// face extraction (CPU only; no CUDA).
//
// Regions are "partitions of data ... physically separated in memory"
// (§IV.A), "expanded to accommodate ghost cells" (§III). The paper
// computes ghost source/destination indices on the host; here
// they are computed once per domain as 6 face descriptors per tile, because
// the decomposition is static (difference D2).
#include <algorithm>
#include <thread>

#include "runtime.hpp"

namespace tiles {

Status make_err(tile_status c, const std::string& m) {
  Status s;
  s.code = c;
  s.msg = m;
  return s;
}

Status make_geometry(const int64_t dims[3], const int64_t td[3], int ghost, tile_bc bc,
                     int nranks, int rank, Geometry* out) {
  Geometry G{};
  for (int a = 0; a < 3; ++a) {
    if (dims[a] < 1 || td[a] < 1) return make_err(TILE_EINVAL, "dims and tile_dims must be >= 1");
    G.g[a] = dims[a];
    G.t[a] = td[a];
  }
  if (nranks < 1 || rank < 0 || rank >= nranks)
    return make_err(TILE_EINVAL, "need 0 <= rank < nranks");
  if (dims[2] % nranks) return make_err(TILE_EINVAL, "nz must be divisible by nranks");
  G.l[0] = dims[0];
  G.l[1] = dims[1];
  G.l[2] = dims[2] / nranks;
  G.zoff = G.l[2] * rank;
  for (int a = 0; a < 3; ++a) {
    if (G.l[a] % td[a])
      return make_err(TILE_EINVAL,
                      "dims (per rank) must be multiples of tile_dims (ragged tiles rejected)");
    G.n[a] = G.l[a] / td[a];
  }
  if ((td[0] & 1) || (td[1] & 1))
    return make_err(TILE_EINVAL, "tile_dims x and y must be even (128-bit vector access)");
  const int64_t tmin = std::min(td[0], std::min(td[1], td[2]));
  if (ghost < 1 || ghost > tmin) return make_err(TILE_EINVAL, "need 1 <= ghost <= min(tile_dims)");
  if (bc != TILE_BC_PERIODIC && bc != TILE_BC_DIRICHLET) return make_err(TILE_EINVAL, "bad bc");
  G.ghost = ghost;
  G.bc = bc;
  G.nranks = nranks;
  G.rank = rank;
  G.ntiles = G.n[0] * G.n[1] * G.n[2];
  G.tile_elems = td[0] * td[1] * td[2];
  // Faces are D = min(ghost, 2) layers deep, layers in increasing
  // coordinate order: x-faces [z][y][D], y-faces [z][D][x], z-faces [D][y][x].
  G.depth = ghost < 2 ? 1 : 2;
  if (G.depth > std::min(td[0], std::min(td[1], td[2])))
    return make_err(TILE_EINVAL, "ghost 2 needs tiles at least 2 cells deep");
  G.face_elems[XM] = G.face_elems[XP] = td[2] * td[1] * G.depth;
  G.face_elems[YM] = G.face_elems[YP] = td[2] * td[0] * G.depth;
  G.face_elems[ZM] = G.face_elems[ZP] = td[1] * td[0] * G.depth;
  G.layer_tiles = G.n[0] * G.n[1];
  *out = G;
  return Status::ok();
}

FaceSrc face_source(const Geometry& G, int64_t id, int f) {
  int64_t c[3];
  G.tile_coords(id, &c[0], &c[1], &c[2]);
  const int axis = f / 2;
  const int dir = (f & 1) ? +1 : -1;
  int64_t nc[3] = {c[0], c[1], c[2]};
  nc[axis] += dir;
  const bool inside = nc[axis] >= 0 && nc[axis] < G.n[axis];
  if (inside) return {0, G.tile_id(nc[0], nc[1], nc[2])};
  if (axis < 2 || G.nranks == 1) {
    // global boundary along x / y, or along z on a single rank
    if (G.bc == TILE_BC_DIRICHLET) return {1, id};
    nc[axis] = (nc[axis] + G.n[axis]) % G.n[axis];
    return {0, G.tile_id(nc[0], nc[1], nc[2])};
  }
  // slab seam along z
  const int64_t pos = c[1] * G.n[0] + c[0];
  if (dir < 0) {
    if (G.rank == 0 && G.bc == TILE_BC_DIRICHLET) return {1, id};
    return {2, pos};
  }
  if (G.rank == G.nranks - 1 && G.bc == TILE_BC_DIRICHLET) return {1, id};
  return {3, pos};
}

void ghost_map(const Geometry& G, int64_t id, int64_t* out) {
  int64_t c[3];
  G.tile_coords(id, &c[0], &c[1], &c[2]);
  const int64_t g = G.ghost;
  const int64_t ex = G.t[0] + 2 * g, ey = G.t[1] + 2 * g, ez = G.t[2] + 2 * g;
  const int64_t ox = c[0] * G.t[0], oy = c[1] * G.t[1], oz = G.zoff + c[2] * G.t[2];
  int64_t* o = out;
  for (int64_t k = 0; k < ez; ++k) {
    const int64_t z = oz + k - g;
    for (int64_t j = 0; j < ey; ++j) {
      const int64_t y = oy + j - g;
      for (int64_t i = 0; i < ex; ++i) {
        const int64_t x = ox + i - g;
        const bool out_of = x < 0 || x >= G.g[0] || y < 0 || y >= G.g[1] || z < 0 || z >= G.g[2];
        if (out_of && G.bc == TILE_BC_DIRICHLET) {
          *o++ = -1;
          continue;
        }
        const int64_t wx = (x % G.g[0] + G.g[0]) % G.g[0];
        const int64_t wy = (y % G.g[1] + G.g[1]) % G.g[1];
        const int64_t wz = (z % G.g[2] + G.g[2]) % G.g[2];
        *o++ = (wz * G.g[1] + wy) * G.g[0] + wx;
      }
    }
  }
}

void host_parallel_for(int64_t n, const std::function<void(int64_t, int64_t)>& fn) {
  unsigned hw = std::thread::hardware_concurrency();
  int64_t nt = std::max<int64_t>(1, std::min<int64_t>(hw ? hw : 4, n));
  if (nt == 1) {
    fn(0, n);
    return;
  }
  std::vector<std::thread> th;
  for (int64_t i = 0; i < nt; ++i) {
    int64_t b = n * i / nt, e = n * (i + 1) / nt;
    th.emplace_back([&fn, b, e] { fn(b, e); });
  }
  for (auto& t : th) t.join();
}

// Export every tile's D boundary layers from the host store (layouts as the
// device faces: x-faces [z][y][D], y-faces [z][D][x], z-faces [D][y][x], the
// D layers in increasing coordinate order).
void host_extract_faces(const Geometry& G, const double* host, double* const faces[6]) {
  const int64_t tx = G.t[0], ty = G.t[1], tz = G.t[2], D = G.depth;
  host_parallel_for(G.ntiles, [&](int64_t b, int64_t e) {
    for (int64_t k = b; k < e; ++k) {
      const double* u = host + k * G.tile_elems;
      double* fxm = faces[XM] + k * G.face_elems[XM];
      double* fxp = faces[XP] + k * G.face_elems[XP];
      double* fym = faces[YM] + k * G.face_elems[YM];
      double* fyp = faces[YP] + k * G.face_elems[YP];
      double* fzm = faces[ZM] + k * G.face_elems[ZM];
      double* fzp = faces[ZP] + k * G.face_elems[ZP];
      for (int64_t z = 0; z < tz; ++z)
        for (int64_t y = 0; y < ty; ++y) {
          const double* row = u + (z * ty + y) * tx;
          for (int64_t l = 0; l < D; ++l) {
            fxm[(z * ty + y) * D + l] = row[l];
            fxp[(z * ty + y) * D + l] = row[tx - D + l];
          }
        }
      for (int64_t z = 0; z < tz; ++z)
        for (int64_t l = 0; l < D; ++l) {
          const double* lo = u + (z * ty + l) * tx;
          const double* hi = u + (z * ty + ty - D + l) * tx;
          std::copy(lo, lo + tx, fym + (z * D + l) * tx);
          std::copy(hi, hi + tx, fyp + (z * D + l) * tx);
        }
      std::copy(u, u + D * ty * tx, fzm);
      std::copy(u + (tz - D) * ty * tx, u + tz * ty * tx, fzp);
    }
  });
}

// Global coordinates of the tile-local cell (x, y, z) of tile id.
static void local_to_tile(const Geometry& G, int64_t c[3], int64_t* tile, bool* inside_all,
                          int out_axis[3]) {
  // c is in units of tile-local cells relative to tile `*tile`; wrap
  // periodically per axis (single rank) and report axes leaving the domain
  int64_t t[3];
  G.tile_coords(*tile, &t[0], &t[1], &t[2]);
  *inside_all = true;
  for (int a = 0; a < 3; ++a) {
    out_axis[a] = 0;
    int64_t off = 0;
    if (c[a] < 0) off = -1;
    if (c[a] >= G.t[a]) off = +1;
    int64_t nt = t[a] + off;
    if (nt < 0 || nt >= G.n[a]) {
      if (G.bc == TILE_BC_DIRICHLET || (a == 2 && G.nranks > 1)) {
        out_axis[a] = off;
        *inside_all = false;
        nt = t[a];  // stay on this tile along a (the cell is in its ghost layer)
        continue;   // keep c[a] as a ghost coordinate
      }
      nt = (nt + G.n[a]) % G.n[a];
    }
    t[a] = nt;
    c[a] -= off * G.t[a];
  }
  *tile = G.tile_id(t[0], t[1], t[2]);
}

EdgeSrc edge_source(const Geometry& G, int64_t id, int e) {
  static const int axes[3][2] = {{0, 1}, {0, 2}, {1, 2}};
  const int grp = e >> 2, ga = (e >> 1) & 1, gb = e & 1;
  const int a = axes[grp][0], b = axes[grp][1], line = 3 - a - b;
  int64_t c[3] = {0, 0, 0};  // tile-local coords of the line's cell 0
  c[a] = ga ? G.t[a] : -1;
  c[b] = gb ? G.t[b] : -1;
  c[line] = 0;
  int64_t tile = id;
  bool inside = true;
  int out[3];
  local_to_tile(G, c, &tile, &inside, out);
  if (G.nranks > 1 && (out[2] != 0 || (a == 2 || b == 2))) {
    // z edges of slab tiles may cross the seam: two-step passes are single-rank only
    if (out[2] != 0 || G.n[2] == 1) return {-2, 0, 0, 0, 0};
  }
  const int nout = (out[a] != 0) + (out[b] != 0);
  if (nout == 2) return {-1, 0, 0, 0, 0};
  const int64_t D = G.depth, tx = G.t[0], ty = G.t[1];
  // the cell is in-domain along the axis that does not leave the domain: it
  // is an interior cell of `tile` (nout == 0) or a Dirichlet ghost of `tile`
  // across the leaving axis (nout == 1). Pick a face array that holds it.
  EdgeSrc s{nout == 0 ? 0 : 1, tile, 0, 0, 1};
  // the face to read: across the leaving axis if any, else the first axis
  const int fa = nout == 1 ? (out[a] != 0 ? a : b) : a;
  const int64_t cf = c[fa];
  int face;
  int64_t layer;
  if (nout == 0) {  // export of the tile's own boundary layers
    face = 2 * fa + (cf == 0 ? 0 : 1);
    layer = cf == 0 ? 0 : D - 1;  // cell at coordinate 0 or t-1
  } else {          // Dirichlet fixed face; the halo value is the nearest layer
    face = 2 * fa + (cf < 0 ? 0 : 1);
    layer = cf < 0 ? D - 1 : 0;
  }
  s.face = face;
  // element offset of cell (c) within the face array and stride along `line`
  auto off_of = [&](int64_t x, int64_t y, int64_t z) -> int64_t {
    if (face <= XP) return ((z * ty) + y) * D + layer;                // [z][y][D]
    if (face <= YP) return ((z * D) + layer) * tx + x;                // [z][D][x]
    return ((layer * ty) + y) * tx + x;                               // [D][y][x]
  };
  const int64_t cx = fa == 0 ? 0 : c[0], cy = fa == 1 ? 0 : c[1], cz = fa == 2 ? 0 : c[2];
  s.offset = off_of(cx, cy, cz);
  int64_t d1[3] = {cx, cy, cz};
  d1[line] += 1;
  s.stride = off_of(d1[0], d1[1], d1[2]) - s.offset;
  return s;
}

EdgePtr Domain::edge_src_ptr(int64_t id, int e, int parity) const {
  const EdgeSrc s = edge_source(G, id, e);
  if (s.kind < 0) return {nullptr, 0};
  const double* base = s.kind == 0 ? faces[s.face][parity] : dir_faces[s.face];
  return {base + s.tile * G.face_elems[s.face] + s.offset, s.stride};
}

const double* Domain::face_src_ptr(int64_t id, int f, int parity) const {
  const FaceSrc s = face_source(G, id, f);
  switch (s.kind) {
    case 0:
      return faces[f ^ 1][parity] + s.val * G.face_elems[f ^ 1];
    case 1:
      return dir_faces[f] + id * G.face_elems[f];
    case 2:
      return halo[0][parity] + s.val * G.face_elems[ZM];
    default:
      return halo[1][parity] + s.val * G.face_elems[ZP];
  }
}

// Direct ghost sources (HeatParams::gdir): x ghosts from the
// exported x faces; y and z ghosts from the nearest ghost layer itself — the
// neighbour tile's boundary row / plane inside its interior in buffer array
// `bit` when the neighbour is a tile of this rank (resident mode: tile k lives
// in slot k or ntiles + k), else the nearest layer of the face source.
const double* Domain::direct_src_ptr(int64_t id, int f, int bit, int parity) const {
  if (f <= XP) return face_src_ptr(id, f, parity);
  const int64_t tx = G.t[0], ty = G.t[1], tz = G.t[2], D = G.depth;
  const FaceSrc s = face_source(G, id, f);
  if (s.kind == 0) {
    const double* nb = slot_ptr(bit ? (int)(G.ntiles + s.val) : (int)s.val);
    switch (f) {
      case YM: return nb + (ty - 1) * tx;
      case YP: return nb;
      case ZM: return nb + (tz - 1) * ty * tx;
      default: return nb;
    }
  }
  const double* base = face_src_ptr(id, f, parity);
  switch (f) {
    case YM: return base + (D - 1) * tx;
    case YP: return base;
    case ZM: return base + (D - 1) * ty * tx;
    default: return base;
  }
}

// z-stride of the direct y ghost row of tile `id` (f = YM or YP).
int64_t Domain::direct_ystride(int64_t id, int f) const {
  return face_source(G, id, f).kind == 0 ? G.t[1] * G.t[0] : (int64_t)G.depth * G.t[0];
}

}  // namespace tiles
