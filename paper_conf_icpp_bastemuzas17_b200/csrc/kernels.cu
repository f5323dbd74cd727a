// kernels.cu — hand-written sm_100a kernels of the tiled hot path.
//
//  heat7_tma      7-point Jacobi heat step over a batch of tiles
//                 (§VI.A; update = DESIGN.md reading R1), with the
//                 ghost update of P:L61/P:L96 fused in: ghost cells are read
//                 straight from the neighbours' exported boundary faces, and
//                 every tile exports its new boundary faces in the epilogue.
//  sincos_iter    compute-intensive kernel, listing P:L219-L224 §VI.B.
//  extract_faces  exports a tile's boundary layers (initial ghost sources).
//
// Design: a tile is stored contiguously ([tz][ty][tx], x
// fastest), so a band of rows of one z-plane is ONE contiguous range. Each
// CTA is persistent over a contiguous range of (tile, band, z) planes and
// marches in z. Planes are staged into a ring of shared-memory stages by
// one thread with 1-D TMA bulk copies (cp.async.bulk ... mbarrier::complete_tx)
// — the band rows, the two y-halo rows and the two x-ghost columns are five
// contiguous ranges — and consumed by all threads from shared memory. All
// arithmetic uses explicit round-to-nearest intrinsics in the order of
// reading R1, so the result is bit-identical to the no-FMA CPU oracle.
#include "kernels.cuh"
#include "ptx.cuh"

#include <algorithm>
#include <cstdlib>

namespace tiles {

// ---------------------------------------------------------------- heat7
// Producer (one thread): stage plane z of band [y0, y0+BY) of tile `in` into
// `dst` ((BY+2) rows of tx + 2 x-ghost columns of BY), completion on `bar`.
// z outside [0, tz) stages the band rows of the z- / z+ ghost plane.
// Stage layout: rows [0, BY+2) of tx (y-halo row, BY band rows, y-halo row),
// then the x- ghost columns (D per row, 2*BY reserved) and the x+ ghost
// columns (D per row). Faces are D layers deep; a single step reads the layer
// nearest the tile (x-: last, x+: first; likewise y and z).
// Ghost sources gs[f]: with ys == nullptr exported-face bases (layouts of
// HeatParams::fexp); with ys != nullptr the direct convention of
// HeatParams::gdir (y/z entries point at the nearest ghost layer, ys[0/1] the
// z-stride of the y-/y+ source rows).
__device__ __forceinline__ void stage_plane(double* dst, uint64_t* bar, const double* in,
                                            const double* const* gs, const int64_t* ys, int z,
                                            int tx, int ty, int tz, int y0, int BY, int flags,
                                            int D) {
  // interior and ghost faces are read once: optionally evict_first
  const uint64_t pol = (flags & 1) ? policy_evict_first() : policy_evict_normal();
  fence_proxy_async();
  if (z < 0 || z >= tz) {
    const uint32_t bytes = (uint32_t)BY * tx * 8;
    mbar_expect_tx(bar, bytes);
    const double* src;
    if (ys)
      src = (z < 0 ? gs[ZM] : gs[ZP]) + (size_t)y0 * tx;
    else
      src = z < 0 ? gs[ZM] + ((size_t)(D - 1) * ty + y0) * tx : gs[ZP] + (size_t)y0 * tx;
    bulk_g2s_hint(dst + tx, src, bytes, bar, pol);
    return;
  }
  const int rows = BY + 2;
  const uint32_t row_b = (uint32_t)tx * 8;
  mbar_expect_tx(bar, ((uint32_t)rows * tx + 2u * D * BY) * 8u);
  const double* plane = in + (size_t)z * ty * tx;
  bulk_g2s_hint(dst + tx, plane + (size_t)y0 * tx, row_b * BY, bar, pol);
  const double* lo;
  const double* hi;
  if (y0 > 0)
    lo = plane + (size_t)(y0 - 1) * tx;
  else
    lo = ys ? gs[YM] + (size_t)z * ys[0] : gs[YM] + ((size_t)z * D + D - 1) * tx;
  if (y0 + BY < ty)
    hi = plane + (size_t)(y0 + BY) * tx;
  else
    hi = ys ? gs[YP] + (size_t)z * ys[1] : gs[YP] + (size_t)z * D * tx;
  bulk_g2s_hint(dst, lo, row_b, bar, pol);
  bulk_g2s_hint(dst + (size_t)(BY + 1) * tx, hi, row_b, bar, pol);
  const uint32_t xb = (uint32_t)(D * BY) * 8;
  bulk_g2s_hint(dst + (size_t)rows * tx, gs[XM] + ((size_t)z * ty + y0) * D, xb, bar, pol);
  bulk_g2s_hint(dst + (size_t)rows * tx + 2 * BY, gs[XP] + ((size_t)z * ty + y0) * D, xb, bar, pol);
}

__device__ __forceinline__ TileItem item_at(const HeatParams& p, int i) {
  return p.items ? p.items[i] : p.inline_items[i];
}

// Contiguous range of (column, plane) pairs owned by this CTA. A column is an
// item column c < lt and a band; its planes g < NZ = nstack*tz run through
// the stacked tiles items[L*lt + c], L = g / tz (nstack = 1: one tile).
struct PlaneRange {
  int64_t pb, pe, P;
  int NZ;
  __device__ PlaneRange(const HeatParams& p) {
    P = (int64_t)p.nitems * p.nbands * p.tz;
    pb = P * blockIdx.x / gridDim.x;
    pe = P * (blockIdx.x + 1) / gridDim.x;
    NZ = p.nstack * p.tz;
  }
};


// Runs (column, first plane, planes) of this CTA for the specialised kernel:
// round-robin whole columns first (HeatParams::rr_rounds), then a contiguous
// share of the remaining columns' planes.
struct Runs {
  // items: (z chunk of ZC planes, column), chunk-major, ZC = HeatParams::zchunk
  // (0: the whole column depth NZ, one item per column)
  int64_t c, cend, pp, pe, total, ncols;
  int NZ, ZC;
  bool rev;  // snake order: the same runs in reverse, each run's planes descending
  __device__ Runs(const HeatParams& p, bool reverse) {
    NZ = p.nstack * p.tz;
    ZC = p.zchunk > 0 ? p.zchunk : NZ;
    rev = reverse;
    ncols = (int64_t)p.lt * p.nbands;
    const int64_t nitems = ncols * (NZ / ZC);
    cend = (int64_t)p.rr_rounds * gridDim.x;
    const int64_t P = (nitems - cend) * ZC;
    pp = cend * ZC + P * blockIdx.x / gridDim.x;
    pe = cend * ZC + P * (blockIdx.x + 1) / gridDim.x;
    const int64_t mine = cend > (int64_t)blockIdx.x ? (cend - 1 - blockIdx.x) / gridDim.x + 1 : 0;
    total = mine * ZC + (pe - pp);
    c = !rev ? (int64_t)blockIdx.x : mine ? (int64_t)blockIdx.x + (mine - 1) * gridDim.x : -1;
  }
  __device__ __forceinline__ void item(int64_t it, int64_t& col, int& gbase) const {
    const int64_t j = it / ncols;
    col = it - j * ncols;
    gbase = (int)(j * ZC);
  }
  __device__ __forceinline__ bool next(int64_t& col, int& g0, int& n) {
    int gb;
    if (rev) {
      if (pe > pp) {
        const int64_t it = (pe - 1) / ZC;
        const int64_t start = pp > it * ZC ? pp : it * ZC;
        item(it, col, gb);
        g0 = gb + (int)(start - it * ZC);
        n = (int)(pe - start);
        pe = start;
        return true;
      }
      if (c < (int64_t)blockIdx.x) return false;
      item(c, col, gb);
      g0 = gb;
      n = ZC;
      c -= gridDim.x;
      return true;
    }
    if (c < cend) {
      item(c, col, gb);
      g0 = gb;
      n = ZC;
      c += gridDim.x;
      return true;
    }
    if (pp >= pe) return false;
    const int64_t it = pp / ZC;
    const int off = (int)(pp - it * ZC);
    item(it, col, gb);
    g0 = gb + off;
    n = (int)(pe - pp < (int64_t)(ZC - off) ? pe - pp : ZC - off);
    pp += n;
    return true;
  }
};

// ---- specialised kernel: compile-time tile width TX, band height BY and
// ring depth S. Each thread owns column pair c2 and rows r0 + j*RPP
// (j < NR) of the band in EVERY plane (register z-march: z-1 and z values
// stay in registers, 5 shared loads per pair and plane). All shared and
// global offsets are compile-time immediates off two per-thread bases.
// The march continues through stacked tiles (HeatParams::nstack): the plane
// below a tile's first plane is the previous tile's last plane, already in
// registers, so only the two ends of a CTA's run read a ghost plane.
template <int TX, int BY, int S>
struct Fixed {
  static constexpr int HALF = TX / 2;
  static constexpr int RPP = (BY < 512 / HALF) ? BY : 512 / HALF;
  static constexpr int NT = RPP * HALF;
  static constexpr int NR = BY / RPP;
  static constexpr int ROWS = BY + 2;
  static constexpr int STAGE_ELEMS = ROWS * TX + 4 * BY;  // x columns: 2 sides x D <= 2
  static constexpr uint32_t STAGE_BYTES = STAGE_ELEMS * 8;
  static constexpr size_t SMEM = (size_t)S * STAGE_BYTES + (size_t)S * 16;  // + full/empty
  static_assert(BY % RPP == 0 && NR >= 1 && NR <= 8, "bad fixed config");
};

template <int TX, int BY, int S, int D>
__global__ void __launch_bounds__(Fixed<TX, BY, S>::NT + 32)
    heat7_fixed(const __grid_constant__ HeatParams p) {
  // Warp-specialised: warps 0..NT/32-1 compute, warp NT/32 is the TMA
  // producer. full[s] completes when stage s has landed (expect_tx bytes);
  // empty[s] completes when every consumer warp has released it. No
  // block-wide barrier in the main loop; the producer runs up to S planes
  // ahead, across column (run) boundaries.
  using C = Fixed<TX, BY, S>;
  constexpr int NCW = C::NT / 32;  // consumer warps
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double* stage_base = reinterpret_cast<double*>(smem_raw);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw + (size_t)S * C::STAGE_BYTES);
  uint64_t* empty = full + S;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], TILES_ARRIVE_PER_THREAD ? NCW * 32 : NCW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  const int ty = p.ty, tz = p.tz;
  const int nsteps = p.nsteps > 1 ? p.nsteps : 1;

  if ((int)threadIdx.x >= C::NT) {  // ---------------- producer warp
    if (threadIdx.x != C::NT) return;
    uint32_t g = 0;
    for (int s = 0; s < nsteps; ++s) {
      const bool odd = s & 1;
      const bool rev = p.snake && odd;
      const TileItem* items = odd ? p.items_odd : p.items;
      const double* const* gtab = odd ? p.gdir_odd : (p.gdir ? p.gdir : p.gsrc);
      Runs W(p, rev);
      int64_t col;
      int g0, n;
      const int NZ = W.NZ;
      while (W.next(col, g0, n)) {
        const int icol = (int)(col / p.nbands);
        const int y0 = (int)(col - (int64_t)icol * p.nbands) * BY;
        // planes g0-1 .. g0+n in march order (descending when rev): stacked
        // tile L, local plane z (z = -1 / tz at the stack ends stage the z
        // ghost planes)
        auto locate = [&](int gp, int& L, int& z) {
          if (gp < 0) L = 0, z = -1;
          else if (gp >= NZ) L = p.nstack - 1, z = tz;
          else L = gp / tz, z = gp - L * tz;
        };
        int L, z;
        locate(rev ? g0 + n : g0 - 1, L, z);
        TileItem it = items ? items[L * p.lt + icol] : p.inline_items[L * p.lt + icol];
        for (int q = 0; q < n + 2; ++q, ++g) {
          if (q) {
            int L2;
            locate(rev ? g0 + n - q : g0 - 1 + q, L2, z);
            if (L2 != L) {  // next stacked tile
              L = L2;
              it = items ? items[L * p.lt + icol] : p.inline_items[L * p.lt + icol];
            }
          }
          const int st = (int)(g % S);
          mbar_wait(&empty[st], ((g / S) & 1u) ^ 1u);
          const double* const* gs = gtab + (size_t)it.tile * 6;
          const int64_t* ys = p.gdir ? p.ystr + (size_t)it.tile * 2 : nullptr;
          stage_plane(stage_base + (size_t)st * C::STAGE_ELEMS, &full[st], it.in, gs, ys, z, TX, ty, tz,
                      y0, BY, p.cache_flags, D);
        }
      }
      if (s + 1 < nsteps) {
        // step barrier: every consumer of this CTA done with step s (drain the
        // ring; mbarrier acquire), their stores released at gpu scope, then
        // one arrival on the grid counter and a wait for all gridDim.x of them.
        // Only this thread waits: the consumers block on the ring as usual.
        for (int i = 0; i < S; ++i) {
          const uint32_t j = g + (uint32_t)i;
          mbar_wait(&empty[j % S], ((j / S) & 1u) ^ 1u);
        }
        fence_acq_rel_gpu();
        red_add_release_gpu(p.prog, 1ull);
        const unsigned long long target = ((unsigned long long)p.epoch + (unsigned long long)s + 1) * gridDim.x;
        while (ld_acquire_gpu(p.prog) < target) __nanosleep(32);
        fence_proxy_async_all();  // other CTAs' generic stores -> this thread's TMA reads
      }
    }
    return;
  }

  // ------------------------------------------------------- consumer warps
  const int lane = (int)threadIdx.x & 31;
  const uint64_t keep = (p.cache_flags & 2) ? policy_evict_last() : policy_evict_normal();
  const int c2 = (int)threadIdx.x % C::HALF;
  const int r0 = (int)threadIdx.x / C::HALF;
  const int x = c2 * 2;
  const bool xlo_edge = c2 == 0, xhi_edge = c2 == C::HALF - 1;
  const double alpha = p.alpha;
  const char* sm = reinterpret_cast<const char*>(smem_raw);
  const int coff = ((r0 + 1) * TX + x) * 8;
  // x ghosts: every thread reads its row neighbours (immediate offsets off
  // cc); the two edge lanes of a warp then overwrite theirs from the staged
  // x-ghost columns (a predicated load at an immediate offset off gcol), so
  // no thread-dependent stride lives in the march
  const int goff = xlo_edge ? (C::ROWS * TX + r0 * D + D - 1) * 8 : (C::ROWS * TX + 2 * BY + r0 * D) * 8;
  auto wait_g = [&](uint32_t g) { mbar_wait(&full[g % S], (g / S) & 1u); };
  auto release_g = [&](uint32_t g) {
    if (TILES_ARRIVE_PER_THREAD) {
      mbar_arrive(&empty[g % S]);
    } else {
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[g % S]);
    }
  };
  uint32_t seq = 0;
  const size_t plane = (size_t)ty * TX;
  const bool xedge = xlo_edge || xhi_edge;
  const int xf = xlo_edge ? XM : XP;  // the x face this thread exports, if any
  bool pushed = false;  // this thread stored halo layers into a neighbour rank's window

  for (int s = 0; s < nsteps; ++s) {
  const bool odd = s & 1;
  const bool rev = p.snake && odd;
  const TileItem* items = odd ? p.items_odd : p.items;
  auto fexp = [&](int f) { return odd ? p.fexp_odd[f] : p.fexp[f]; };
  Runs W(p, rev);
  int64_t left = W.total;  // planes of this step still to store (march order)
  const int64_t dz = rev ? -1 : 1;
  int64_t col;
  int g0, n;
  while (W.next(col, g0, n)) {
    const int icol = (int)(col / p.nbands);
    const int yb = (int)(col - (int64_t)icol * p.nbands) * BY + r0;

    double2 zm[C::NR], zc[C::NR];
    wait_g(seq);
    wait_g(seq + 1);
    {
      const char* s0 = sm + (size_t)(seq % S) * C::STAGE_BYTES + coff;
      const char* s1 = sm + (size_t)((seq + 1) % S) * C::STAGE_BYTES + coff;
#pragma unroll
      for (int j = 0; j < C::NR; ++j) {
        zm[j] = *reinterpret_cast<const double2*>(s0 + j * C::RPP * TX * 8);
        zc[j] = *reinterpret_cast<const double2*>(s1 + j * C::RPP * TX * 8);
      }
    }
    release_g(seq);  // plane g0-1 (g0+n when rev) is in registers now
    const int gfirst = rev ? g0 + n - 1 : g0;
    int L = gfirst / tz, z = gfirst - L * tz;
    int tile = 0;
    double* op = nullptr;  // output cell pair of row yb, plane z
    double* fx = nullptr;  // x-face export of row yb, plane z (edge threads)
    auto enter_tile = [&]() {
      const TileItem it = items ? items[L * p.lt + icol] : p.inline_items[L * p.lt + icol];
      tile = it.tile;
      op = it.out + ((size_t)z * ty + yb) * TX + x;
      if (xedge) fx = fexp(xf) + (int64_t)tile * p.face_elems[xf] + ((size_t)z * ty + yb) * D;
    };
    enter_tile();
    for (int i = 0; i < n; ++i) {
      if (z == tz || z < 0) {  // next stacked tile in march order (cold)
        L += (int)dz;
        z = rev ? tz - 1 : 0;
        enter_tile();
      }
      wait_g(seq + i + 2);
      const char* cur = sm + (size_t)((seq + i + 1) % S) * C::STAGE_BYTES;
      const char* nxt = sm + (size_t)((seq + i + 2) % S) * C::STAGE_BYTES + coff;
      const char* cc = cur + coff;
      const char* gcol = cur + goff;
      double2 v[C::NR];
#pragma unroll
      for (int j = 0; j < C::NR; ++j) {
        const int jo = j * C::RPP * TX * 8;
        const double2 zp = *reinterpret_cast<const double2*>(nxt + jo);
        const double2 ym = *reinterpret_cast<const double2*>(cc + jo - TX * 8);
        const double2 yp = *reinterpret_cast<const double2*>(cc + jo + TX * 8);
        double xm = *reinterpret_cast<const double*>(cc + jo - 8);
        double xp = *reinterpret_cast<const double*>(cc + jo + 16);
        const double xg = *reinterpret_cast<const double*>(gcol + j * C::RPP * D * 8);
        if (xlo_edge) xm = xg;
        if (xhi_edge) xp = xg;
        const double2 c = zc[j];
        v[j].x = heat_update(c.x, xm, c.y, ym.x, yp.x, zm[j].x, zp.x, alpha);
        v[j].y = heat_update(c.y, c.x, xp, ym.y, yp.y, zm[j].y, zp.y, alpha);
        if (left > p.keep_tail) stg2_stream(op + (size_t)j * C::RPP * TX, v[j]);
        else st2_hint(op + (size_t)j * C::RPP * TX, v[j], keep);  // read first by the next (reversed) step
        zm[j] = c;
        zc[j] = zp;
      }
      --left;
      release_g(seq + i + 1);  // plane z no longer read (its centre is in registers)
      // Epilogue: export the new boundary layers (the neighbours' ghost
      // sources for the next step). x: the two edge lanes of every
      // warp; y (warp-uniform rows) and z (block-uniform planes): rare.
      if (xedge) {
#pragma unroll
        for (int j = 0; j < C::NR; ++j) {
          double* q = fx + (size_t)j * C::RPP * D;
          if (D == 1) st_hint(q, xlo_edge ? v[j].x : v[j].y, keep);
          else st2_hint(q, v[j], keep);
        }
      }
      if (p.exp_y) {
#pragma unroll
        for (int j = 0; j < C::NR; ++j) {
          const int y = yb + j * C::RPP;
          if (y < D) st2_hint(fexp(YM) + (int64_t)tile * p.face_elems[YM] + ((size_t)z * D + y) * TX + x, v[j], keep);
          if (y >= ty - D)
            st2_hint(fexp(YP) + (int64_t)tile * p.face_elems[YP] + ((size_t)z * D + y - (ty - D)) * TX + x, v[j], keep);
        }
      }
      if (z < D && tile < p.exp_zlo_below) {
        const size_t e = ((size_t)z * ty + yb) * TX + x;
#pragma unroll
        for (int j = 0; j < C::NR; ++j)
          st2_hint(fexp(ZM) + (int64_t)tile * p.face_elems[ZM] + e + (size_t)j * C::RPP * TX, v[j], keep);
        if (p.zpush_lo) {  // fused halo push into the lower rank's window
          pushed = true;
          double* q = p.zpush_lo + (int64_t)tile * p.face_elems[ZM] + e;
#pragma unroll
          for (int j = 0; j < C::NR; ++j) *reinterpret_cast<double2*>(q + (size_t)j * C::RPP * TX) = v[j];
        }
      }
      if (z >= tz - D && tile >= p.exp_zhi_from) {
        const size_t e = ((size_t)(z - (tz - D)) * ty + yb) * TX + x;
#pragma unroll
        for (int j = 0; j < C::NR; ++j)
          st2_hint(fexp(ZP) + (int64_t)tile * p.face_elems[ZP] + e + (size_t)j * C::RPP * TX, v[j], keep);
        if (p.zpush_hi) {  // fused halo push into the upper rank's window
          pushed = true;
          double* q = p.zpush_hi + (int64_t)(tile - p.exp_zhi_from) * p.face_elems[ZP] + e;
#pragma unroll
          for (int j = 0; j < C::NR; ++j) *reinterpret_cast<double2*>(q + (size_t)j * C::RPP * TX) = v[j];
        }
      }
      op += dz * (int64_t)plane;
      fx += dz * (int64_t)ty * D;
      z += (int)dz;
    }
    release_g(seq + n + 1);  // plane g0+n (last z+1 neighbour)
    seq += (uint32_t)(n + 2);
  }
  }
  // pushed halo layers visible system-wide (the neighbour ranks' GPUs) before
  // the halo stream's arrival counter, written after this kernel, is
  if (pushed) asm volatile("fence.acq_rel.sys;" ::: "memory");
}

// ---- general kernel: any even tile width / band (runtime shape). Every
// plane is read from shared memory (7 loads per pair). Used when no
// specialisation matches.
template <int NT>
__global__ void __launch_bounds__(NT) heat7_generic(const __grid_constant__ HeatParams p,
                                                    const int stages) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  const int tx = p.tx, ty = p.ty, tz = p.tz, BY = p.band, D = p.depth;
  const int rows = BY + 2;
  const int stage_elems = rows * tx + 4 * BY;
  double* stage_base = reinterpret_cast<double*>(smem_raw);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem_raw + (size_t)stages * stage_elems * 8);
  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) mbar_init(&bars[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const PlaneRange R(p);
  const int half = tx >> 1;
  const double alpha = p.alpha;
  uint32_t seq = 0;
  for (int64_t pp = R.pb; pp < R.pe;) {
    const int64_t col = pp / tz;
    const int z0 = (int)(pp - col * tz);
    const int z1 = (int)(R.pe - pp < (int64_t)(tz - z0) ? z0 + (R.pe - pp) : tz);
    const int item_i = (int)(col / p.nbands);
    const int y0 = (int)(col - (int64_t)item_i * p.nbands) * BY;
    const TileItem it = p.items ? p.items[item_i] : p.inline_items[item_i];
    const double* const* gs = p.gsrc + (size_t)it.tile * 6;
    const int nq = z1 - z0 + 2;
    auto issue = [&](int q) {
      const uint32_t g = seq + q;
      stage_plane(stage_base + (size_t)(g % stages) * stage_elems, &bars[g % stages], it.in, gs,
                  nullptr, z0 - 1 + q, tx, ty, tz, y0, BY, p.cache_flags, D);
    };
    auto wait_q = [&](int q) {
      const uint32_t g = seq + q;
      mbar_wait(&bars[g % stages], (g / stages) & 1u);
    };
    if (threadIdx.x == 0)
      for (int q = 0; q < min(stages, nq); ++q) issue(q);
    const int64_t tile = it.tile;
    double* fxm = p.fexp[XM] + tile * p.face_elems[XM];
    double* fxp = p.fexp[XP] + tile * p.face_elems[XP];
    double* fym = p.fexp[YM] + tile * p.face_elems[YM];
    double* fyp = p.fexp[YP] + tile * p.face_elems[YP];
    double* fzm = p.fexp[ZM] + tile * p.face_elems[ZM];
    double* fzp = p.fexp[ZP] + tile * p.face_elems[ZP];
    wait_q(0);
    wait_q(1);
    for (int i = 0; i < z1 - z0; ++i) {
      wait_q(i + 2);
      const int z = z0 + i;
      const double* prv = stage_base + (size_t)((seq + i) % stages) * stage_elems;
      const double* cur = stage_base + (size_t)((seq + i + 1) % stages) * stage_elems;
      const double* nxt = stage_base + (size_t)((seq + i + 2) % stages) * stage_elems;
      const double* xlo = cur + (size_t)rows * tx;      // [r][D], nearest layer D-1
      const double* xhi = xlo + 2 * BY;                  // [r][D], nearest layer 0
      double* out_plane = it.out + (size_t)z * ty * tx;
      const int npairs = BY * half;
      for (int e = threadIdx.x; e < npairs; e += NT) {
        const int r = e / half, x = (e % half) << 1;
        const double* crow = cur + (size_t)(r + 1) * tx;
        const double2 c = *reinterpret_cast<const double2*>(crow + x);
        const double2 ym = *reinterpret_cast<const double2*>(cur + (size_t)r * tx + x);
        const double2 yp = *reinterpret_cast<const double2*>(cur + (size_t)(r + 2) * tx + x);
        const double2 zm = *reinterpret_cast<const double2*>(prv + (size_t)(r + 1) * tx + x);
        const double2 zp = *reinterpret_cast<const double2*>(nxt + (size_t)(r + 1) * tx + x);
        const double xm = x == 0 ? xlo[r * D + D - 1] : crow[x - 1];
        const double xp = x + 2 == tx ? xhi[r * D] : crow[x + 2];
        double2 v;
        v.x = heat_update(c.x, xm, c.y, ym.x, yp.x, zm.x, zp.x, alpha);
        v.y = heat_update(c.y, c.x, xp, ym.y, yp.y, zm.y, zp.y, alpha);
        const int y = y0 + r;
        stg2_stream(out_plane + (size_t)y * tx + x, v);
        if (x == 0) {
          if (D == 1) fxm[(size_t)z * ty + y] = v.x;
          else *reinterpret_cast<double2*>(fxm + ((size_t)z * ty + y) * 2) = v;
        }
        if (x + 2 == tx) {
          if (D == 1) fxp[(size_t)z * ty + y] = v.y;
          else *reinterpret_cast<double2*>(fxp + ((size_t)z * ty + y) * 2) = v;
        }
        if (y < D) *reinterpret_cast<double2*>(fym + ((size_t)z * D + y) * tx + x) = v;
        if (y >= ty - D) *reinterpret_cast<double2*>(fyp + ((size_t)z * D + y - (ty - D)) * tx + x) = v;
        if (z < D) *reinterpret_cast<double2*>(fzm + ((size_t)z * ty + y) * tx + x) = v;
        if (z >= tz - D) *reinterpret_cast<double2*>(fzp + ((size_t)(z - (tz - D)) * ty + y) * tx + x) = v;
      }
      __syncthreads();
      if (threadIdx.x == 0 && i + stages < nq) issue(i + stages);
    }
    seq += (uint32_t)nq;
    pp += z1 - z0;
  }
}

constexpr int kGenericThreads = 256;

// Specialisations: (TX, BY) -> kernel. BY is the largest of {64,32,16,8}
// that divides ty and whose 5-stage ring fits in shared memory.
struct FixedEntry {
  int tx, by, stages, depth;
  void (*fn)(HeatParams);
  int nt;
  size_t smem;
};
#define FIXED1(TX, BY, S, D) \
  {TX, BY, S, D, heat7_fixed<TX, BY, S, D>, Fixed<TX, BY, S>::NT + 32, Fixed<TX, BY, S>::SMEM}
#define FIXED(TX, BY, S) FIXED1(TX, BY, S, 1), FIXED1(TX, BY, S, 2)
static const FixedEntry kFixed[] = {
    FIXED(32, 32, 6),  FIXED(32, 16, 6),  FIXED(32, 8, 6),   FIXED(64, 64, 4),
    FIXED(64, 64, 6),  FIXED(64, 64, 5),  FIXED(64, 32, 4),  FIXED(64, 32, 3),
    FIXED(64, 32, 6),  FIXED(64, 16, 6),  FIXED(64, 8, 6),   FIXED(128, 32, 6),
    FIXED(128, 16, 6), FIXED(128, 8, 6),  FIXED(256, 16, 6), FIXED(256, 8, 6),
    FIXED(512, 8, 5)};
#undef FIXED

static const FixedEntry* find_fixed(int tx, int by) {
  for (const auto& e : kFixed)
    if (e.tx == tx && e.by == by) return &e;
  return nullptr;
}

static const FixedEntry* find_fixed_s(int tx, int by, int st, int depth = 1) {
  for (const auto& e : kFixed)
    if (e.tx == tx && e.by == by && e.stages == st && e.depth == depth) return &e;
  return nullptr;
}

bool heat_plan(int tx, int ty, int max_smem, int* band, int* stages, size_t* smem) {
  if (tx < 2 || (tx & 1) || ty < 2 || (ty & 1)) return false;
  // tuning override: TILES_HEAT_BAND / TILES_HEAT_STAGES select a specialisation
  if (const char* eb = std::getenv("TILES_HEAT_BAND")) {
    const char* es = std::getenv("TILES_HEAT_STAGES");
    const int by = std::atoi(eb), st = es ? std::atoi(es) : 0;
    const FixedEntry* e = st ? find_fixed_s(tx, by, st) : find_fixed(tx, by);
    if (e && ty % by == 0 && e->smem <= (size_t)max_smem) {
      *band = by;
      *stages = e->stages;
      *smem = e->smem;
      return true;
    }
  }
  for (int by : {64, 32, 16, 8}) {  // specialised kernels first
    if (ty % by) continue;
    const FixedEntry* e = find_fixed(tx, by);
    if (e && e->smem <= (size_t)max_smem) {
      *band = by;
      *stages = e->stages;
      *smem = e->smem;
      return true;
    }
  }
  // general kernel: largest even divisor of ty (<= 64) whose ring fits;
  // prefer 5 stages, trade stages for bands of >= 16 rows.
  const int want = std::min(ty, 16);
  int best_by = 0, best_s = 0;
  for (int S : {5, 4, 3}) {
    for (int by = std::min(ty, 64); by >= 2; --by) {
      if ((by & 1) || ty % by) continue;
      size_t bytes = (size_t)S * ((size_t)(by + 2) * tx + 4 * by) * 8 + (size_t)S * 8;
      if (bytes > (size_t)max_smem) continue;
      if (by > best_by) { best_by = by; best_s = S; }
      break;
    }
    if (best_by >= want) break;
  }
  if (!best_by) return false;
  *band = best_by;
  *stages = best_s;
  *smem = (size_t)best_s * ((size_t)(best_by + 2) * tx + 4 * best_by) * 8 + (size_t)best_s * 8;
  return true;
}

cudaError_t heat_configure(int tx, int ty, int band, int stages, size_t smem, int* ctas_per_sm) {
  (void)ty;
  const FixedEntry* e = find_fixed_s(tx, band, stages, 1);
  if (e && e->smem == smem) {
    for (int dd = 1; dd <= 2; ++dd) {  // both face depths share the plan
      const FixedEntry* f = find_fixed_s(tx, band, stages, dd);
      cudaError_t r = cudaFuncSetAttribute(f->fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      if (r != cudaSuccess) return r;
    }
    cudaError_t r = cudaFuncSetAttribute(e->fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (r != cudaSuccess) return r;
    return cudaOccupancyMaxActiveBlocksPerMultiprocessor(ctas_per_sm, e->fn, e->nt, smem);
  }
  cudaError_t r = cudaFuncSetAttribute(heat7_generic<kGenericThreads>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (r != cudaSuccess) return r;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(ctas_per_sm, heat7_generic<kGenericThreads>,
                                                       kGenericThreads, smem);
}

cudaError_t launch_heat7(const HeatParams& p, int stages, size_t smem, int grid, cudaStream_t s) {
  const FixedEntry* e = find_fixed_s(p.tx, p.band, stages, p.depth);
  if (e && e->smem == smem) {
    void* args[] = {const_cast<HeatParams*>(&p)};
    if (p.nsteps > 1)  // CTAs wait on each other's progress: all must be co-resident
      return cudaLaunchCooperativeKernel(reinterpret_cast<const void*>(e->fn), dim3(grid), dim3(e->nt),
                                         args, smem, s);
    return cudaLaunchKernel(reinterpret_cast<const void*>(e->fn), dim3(grid), dim3(e->nt), args,
                            smem, s);
  }
  // the general kernel takes independent tiles and exported faces only
  if (p.gdir || p.nstack != 1 || p.lt != p.nitems || p.nsteps > 1) return cudaErrorInvalidValue;
  heat7_generic<kGenericThreads><<<grid, kGenericThreads, smem, s>>>(p, stages);
  return cudaGetLastError();
}

bool heat_is_fixed(int tx, int band, int stages, size_t smem) {
  const FixedEntry* e = find_fixed_s(tx, band, stages, 1);
  return e && e->smem == smem;
}

// -------------------------------------------------------------- sincos_iter
// Listing P:L219-L224: per cell, `iters` times: s=sin(x); c=cos(x);
// x = x + sqrt(s*s + c*c). Each thread carries two independent cells (ILP);
// the listing's own operations are rounded one by one (no contraction).
// sin(x)^2 + cos(x)^2 as the listing evaluates it (s*s + c*c, each product
// and the sum rounded, no contraction). With x = q*pi/2 + r (|r| <= pi/4),
// sin x and cos x are +-sin r and +-cos r, swapped when q is odd; the sum of
// the rounded squares does not depend on signs or order, so the quadrant is
// never needed. sin r, cos r: fdlibm's minimax polynomials (max 1 ulp /
// 2 ulp, checked against glibc over 2e7 points), r by a two-constant FMA
// Cody-Waite reduction (exact to ~1 ulp of r for |q| < 2^20). The fast loop
// runs while |x| <= 1e6 is guaranteed for all iterations (x grows by at most
// ~1 per iteration); otherwise libdevice's sincos (Payne-Hanek) is used.
// Polynomial and reduction constants live in constant memory so the DFMAs
// take them as c[][] operands (64-bit immediates would cost two uniform
// moves per use per iteration). TILES_SINCOS_LIBDEVICE=1: libdevice only.
#ifndef TILES_SINCOS_LIBDEVICE
#define TILES_SINCOS_LIBDEVICE 0
#endif
__constant__ double kSC[16] = {
    6.36619772367581382433e-01,   // 0: 2/pi
    1.5707963267948966,           // 1: pi/2 high
    6.123233995736766e-17,        // 2: pi/2 - high
    1.58969099521155010221e-10,   // 3..8: sin S6..S1
    -2.50507602534068634195e-08, 2.75573137070700676789e-06, -1.98412698298579493134e-04,
    8.33333333332248946124e-03, -1.66666666666666324348e-01,
    -1.13596475577881948265e-11,  // 9..14: cos C6..C1
    2.08757232129817482790e-09, -2.75573143513906633035e-07, 2.48015872894767294178e-05,
    -1.38888888888741095749e-03, 4.16666666666666019037e-02,
    0.0};

static __device__ __forceinline__ double sin2_plus_cos2_fast(double x) {
  const double q = rint(__dmul_rn(x, kSC[0]));
  double r = fma(-q, kSC[1], x);
  r = fma(-q, kSC[2], r);
  const double z = __dmul_rn(r, r);
  const double ps = fma(z, fma(z, fma(z, fma(z, kSC[3], kSC[4]), kSC[5]), kSC[6]), kSC[7]);
  const double s = fma(__dmul_rn(r, z), fma(z, ps, kSC[8]), r);
  const double pc = fma(z, fma(z, fma(z, fma(z, fma(z, kSC[9], kSC[10]), kSC[11]), kSC[12]), kSC[13]), kSC[14]);
  const double c = fma(z, fma(z, pc, -0.5), 1.0);
  return __dadd_rn(__dmul_rn(s, s), __dmul_rn(c, c));
}

static __device__ __forceinline__ double sin2_plus_cos2_libdevice(double x) {
  double s, c;
  sincos(x, &s, &c);
  return __dadd_rn(__dmul_rn(s, s), __dmul_rn(c, c));
}

__global__ void __launch_bounds__(256) sincos_iter(const __grid_constant__ SincosParams p) {
  const int item_i = blockIdx.y;
  const TileItem it = p.items ? p.items[item_i] : p.inline_items[item_i];
  double2* data = reinterpret_cast<double2*>(it.out);
  const double2* src = reinterpret_cast<const double2*>(it.in);
  const int64_t npairs = p.tile_elems >> 1;
  for (int64_t j = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; j < npairs;
       j += (int64_t)gridDim.x * blockDim.x) {
    double2 v = src[j];
    double a = v.x, b = v.y;
    const double lim = 1.0e6 - 2.0 * (double)p.iters;  // fast path valid for every iteration
    if (!TILES_SINCOS_LIBDEVICE && fabs(a) <= lim && fabs(b) <= lim) {
      for (int64_t k = 0; k < p.iters; ++k) {
        const double ta = sin2_plus_cos2_fast(a), tb = sin2_plus_cos2_fast(b);
        a = __dadd_rn(a, __dsqrt_rn(ta));
        b = __dadd_rn(b, __dsqrt_rn(tb));
      }
    } else {
      for (int64_t k = 0; k < p.iters; ++k) {
        const double ta = sin2_plus_cos2_libdevice(a), tb = sin2_plus_cos2_libdevice(b);
        a = __dadd_rn(a, __dsqrt_rn(ta));
        b = __dadd_rn(b, __dsqrt_rn(tb));
      }
    }
    data[j] = make_double2(a, b);
  }
}

cudaError_t launch_sincos(const SincosParams& p, int grid, cudaStream_t s) {
  dim3 g(grid, p.nitems);
  sincos_iter<<<g, 256, 0, s>>>(p);
  return cudaGetLastError();
}

// ------------------------------------------------------------ extract_faces
__global__ void extract_faces(const __grid_constant__ ExtractParams p) {
  const int item_i = blockIdx.y;
  const int f = blockIdx.z;
  const TileItem it = p.items ? p.items[item_i] : p.inline_items[item_i];
  const int tx = p.tx, ty = p.ty, tz = p.tz, D = p.depth;
  double* dst = p.fexp[f] + (int64_t)it.tile * p.face_elems[f];
  const int64_t n = p.face_elems[f];
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n;
       e += (int64_t)gridDim.x * blockDim.x) {
    int64_t src;
    if (f <= XP) {  // [z][y][D]
      const int64_t l = e % D, zy = e / D, z = zy / ty, y = zy % ty;
      src = (z * ty + y) * tx + (f == XM ? l : tx - D + l);
    } else if (f <= YP) {  // [z][D][x]
      const int64_t x = e % tx, zl = e / tx, z = zl / D, l = zl % D;
      src = (z * ty + (f == YM ? l : ty - D + l)) * tx + x;
    } else {  // [D][y][x]
      src = (int64_t)(f == ZM ? 0 : tz - D) * ty * tx + e;
    }
    dst[e] = it.in[src];
  }
}

cudaError_t launch_extract(const ExtractParams& p, cudaStream_t s) {
  dim3 g(8, p.nitems, 6);
  extract_faces<<<g, 256, 0, s>>>(p);
  return cudaGetLastError();
}

}  // namespace tiles

namespace tiles {

// ---------------------------------------------------------------- push_rows
// Device -> pinned host copy done by the SMs (the host store is mapped): n
// rows of len double2, row r from src + r * sp to dst + r * dp (in double2
// units). The copy engine then carries only host -> device traffic, and the
// writes leave as posted PCIe writes from a few CTAs.
__global__ void __launch_bounds__(256) push_rows(const double2* __restrict__ src, int64_t sp, double2* dst,
                                                 int64_t dp, int64_t len) {
  const double2* s = src + (int64_t)blockIdx.y * sp;
  double2* d = dst + (int64_t)blockIdx.y * dp;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < len; i += (int64_t)gridDim.x * blockDim.x)
    d[i] = __ldcs(s + i);
}

cudaError_t launch_push_rows(const double* src, int64_t src_pitch, double* dst, int64_t dst_pitch, int64_t rows,
                             int64_t len, int ctas, cudaStream_t st) {
  if (rows <= 0 || len <= 0) return cudaSuccess;
  const int64_t gx = std::max<int64_t>(1, ctas / std::max<int64_t>(1, rows));
  push_rows<<<dim3((unsigned)gx, (unsigned)rows), 256, 0, st>>>(
      reinterpret_cast<const double2*>(src), src_pitch / 2, reinterpret_cast<double2*>(dst), dst_pitch / 2, len / 2);
  return cudaGetLastError();
}

}  // namespace tiles
