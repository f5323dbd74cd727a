// kernels_x2.cu — two Jacobi steps per pass (temporal blocking, §8(f) NEXT
// #2; DESIGN.md §4 "heat7x2"). A tile with a ghost width of 2 can advance two
// steps per residency pass: u^{s+2} on the tile needs u^{s+1} on the tile plus
// its face ring (cells one outside in exactly one axis), which needs u^s on
// the tile, its depth-2 faces and the 12 edge lines (cells one outside in two
// axes). Faces come from the neighbours' depth-2 exports (or Dirichlet fixed
// faces); edge lines are read out of the diagonal neighbours' face exports
// (EdgePtr table), so no extra exports exist. Every cell update uses the same
// rounded operations as the single step (reading R1), so two single steps and
// one double step give bit-identical results.
//
// Per CTA (persistent over a contiguous range of (tile, band, z) columns, as
// heat7_fixed): a producer warp stages u^s planes z0-2 .. z1+1 into a ring of
// S stages (band rows +-2, depth-2 x-ghost columns, edge cells); consumer
// warps compute u^{s+1} for plane m (band rows +-1, x ring columns) into one
// of two shared "mid" planes, then u^{s+2} for plane m-1 from the mid planes
// (register z-march: mid(m-2) of a thread's own cells stays in registers).
#include "kernels.cuh"
#include "ptx.cuh"

#include <cstdio>
#include <cstdlib>

namespace tiles {

template <int TX, int BY, int S_ = 4, int MB_ = 2>
struct X2 {
  static constexpr int MB = MB_;         // mid planes: 2 (phases per plane) or 3 (pipelined)
  static constexpr int HALF = TX / 2;
  static constexpr int RPP = (BY < 512 / HALF) ? BY : 512 / HALF;
  static constexpr int NT = RPP * HALF;  // consumer threads
  static constexpr int NR = BY / RPP;    // output rows per consumer thread
  static constexpr int S = S_;           // input stages
  static constexpr int IROWS = BY + 4;   // staged rows y0-2 .. y0+BY+1
  static constexpr int XOFF = IROWS * TX;
  static constexpr int STAGE_ELEMS = IROWS * TX + 4 * IROWS;  // + x-ghost [2 sides][IROWS][2]
  static constexpr int MROWS = BY + 2;   // mid rows y0-1 .. y0+BY
  static constexpr int MPITCH = TX + 4;  // mid col of x is x + 2 (x = -1 .. TX)
  static constexpr int MID_ELEMS = MROWS * MPITCH;
  static constexpr size_t SMEM = (size_t)S * STAGE_ELEMS * 8 + MB * (size_t)MID_ELEMS * 8 + 2 * S * 8;
  static_assert(BY % RPP == 0 && NR >= 1 && NR <= 8, "bad x2 config");
};

constexpr int kEdgeXY = 0, kEdgeXZ = 4, kEdgeYZ = 8;
__host__ __device__ constexpr uint8_t bit(int f) { return (uint8_t)(1u << f); }

// Producer warp: stage u^s plane z of band y0 of tile `in` into dst.
template <int TX, int BY, int S>
__device__ __forceinline__ void stage_x2(double* dst, uint64_t* bar, const double* in,
                                         const double* const* gs, const EdgePtr* es, int z,
                                         int ty, int tz, int y0, int lane) {
  using C = X2<TX, BY, S, 2>;  // stage layout does not depend on MB
  const int lo = y0 - 2 < 0 ? 0 : y0 - 2;
  const int hi = y0 + BY + 2 > ty ? ty : y0 + BY + 2;
  const int rlo = lo - (y0 - 2);  // staged row of y = lo
  const bool inplane = z >= 0 && z < tz;
  const bool near_ghost = z == -1 || z == tz;
  // 1) edge cells (regular loads by the warp, generic proxy) — written before
  //    the lanes' arrives on `bar`, which release them to the consumers.
  if (inplane) {
    if (lane < 4) {
      const int gx = lane & 1, gy = lane >> 1;
      const bool need = gy == 0 ? y0 == 0 : y0 + BY == ty;
      if (need) {
        const EdgePtr e = es[kEdgeXY + 2 * gx + gy];
        if (e.ptr) {
          const int r = (gy == 0 ? -1 : ty) - (y0 - 2);
          dst[C::XOFF + gx * 2 * C::IROWS + r * 2 + (gx ? 0 : 1)] = e.ptr[(int64_t)z * e.stride];
        }
      }
    }
  } else if (near_ghost) {
    const int gz = z < 0 ? 0 : 1;
    for (int gy = 0; gy < 2; ++gy) {  // rows y = -1 / ty of the ghost plane
      const bool need = gy == 0 ? y0 == 0 : y0 + BY == ty;
      const EdgePtr e = es[kEdgeYZ + 2 * gy + gz];
      if (need && e.ptr) {
        const int r = (gy == 0 ? -1 : ty) - (y0 - 2);
        for (int x = lane; x < TX; x += 32) dst[r * TX + x] = e.ptr[(int64_t)x * e.stride];
      }
    }
    for (int gx = 0; gx < 2; ++gx) {  // x = -1 / TX columns of the ghost plane
      const EdgePtr e = es[kEdgeXZ + 2 * gx + gz];
      if (!e.ptr) continue;
      for (int y = y0 + lane; y < y0 + BY; y += 32)
        dst[C::XOFF + gx * 2 * C::IROWS + (y - (y0 - 2)) * 2 + (gx ? 0 : 1)] =
            e.ptr[(int64_t)y * e.stride];
    }
  }
  if (TILES_ARRIVE_PER_THREAD) {  // every lane releases its own edge writes
    if (lane != 0) {
      mbar_arrive(bar);
      return;
    }
  } else {
    __syncwarp();
    if (lane != 0) return;
  }
  // 2) bulk copies (TMA)
  const uint64_t pol = policy_evict_normal();
  fence_proxy_async();
  uint32_t bytes = 0;
  const uint32_t row_b = TX * 8;
  if (inplane) {
    bytes += (uint32_t)(hi - lo) * row_b + 2u * (uint32_t)(hi - lo) * 16u;
    if (y0 == 0) bytes += 2 * row_b;
    if (y0 + BY == ty) bytes += 2 * row_b;
  } else {
    bytes += (uint32_t)(hi - lo) * row_b;
  }
  mbar_expect_tx(bar, bytes);
  if (inplane) {
    const double* plane = in + (size_t)z * ty * TX;
    bulk_g2s_hint(dst + (size_t)rlo * TX, plane + (size_t)lo * TX, (hi - lo) * row_b, bar, pol);
    if (y0 == 0)  // rows -2, -1: layers 0, 1 of the y- source, plane z ([z][2][x])
      bulk_g2s_hint(dst, gs[YM] + (size_t)z * 2 * TX, 2 * row_b, bar, pol);
    if (y0 + BY == ty)  // rows ty, ty+1: layers 0, 1 of the y+ source
      bulk_g2s_hint(dst + (size_t)(ty - (y0 - 2)) * TX, gs[YP] + (size_t)z * 2 * TX, 2 * row_b, bar,
                    pol);
    const uint32_t xb = (uint32_t)(hi - lo) * 16u;  // [y][2] per side
    bulk_g2s_hint(dst + C::XOFF + rlo * 2, gs[XM] + ((size_t)z * ty + lo) * 2, xb, bar, pol);
    bulk_g2s_hint(dst + C::XOFF + 2 * C::IROWS + rlo * 2, gs[XP] + ((size_t)z * ty + lo) * 2, xb,
                  bar, pol);
  } else {
    const int l = z < 0 ? z + 2 : z - tz;  // layer of the z source ([2][y][x])
    const double* src = (z < 0 ? gs[ZM] : gs[ZP]) + ((size_t)l * ty + lo) * TX;
    bulk_g2s_hint(dst + (size_t)rlo * TX, src, (hi - lo) * row_b, bar, pol);
  }
}

template <int TX, int BY, int S, int MB>
__global__ void __launch_bounds__(X2<TX, BY, S, MB>::NT + 32) heat7x2(const __grid_constant__ Heat2Params P) {
  using C = X2<TX, BY, S, MB>;
  const HeatParams& p = P.h;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double* stage_base = reinterpret_cast<double*>(smem_raw);
  double* mid0 = stage_base + (size_t)C::S * C::STAGE_ELEMS;
  uint64_t* full = reinterpret_cast<uint64_t*>(mid0 + MB * C::MID_ELEMS);
  uint64_t* empty = full + C::S;
  constexpr int NCW = C::NT / 32;
  if (threadIdx.x == 0) {
    for (int s = 0; s < C::S; ++s) {
      mbar_init(&full[s], TILES_ARRIVE_PER_THREAD ? 32 : 1);  // producer lanes (edge cells)
      mbar_init(&empty[s], TILES_ARRIVE_PER_THREAD ? NCW * 32 : NCW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const int ty = p.ty, tz = p.tz;
  const int64_t P_all = (int64_t)p.nitems * p.nbands * tz;
  const int64_t pb = P_all * blockIdx.x / gridDim.x, pe = P_all * (blockIdx.x + 1) / gridDim.x;
  const int lane = (int)threadIdx.x & 31;

  if ((int)threadIdx.x >= C::NT) {  // ---------------------- producer warp
    uint32_t g = 0;
    for (int64_t pp = pb; pp < pe;) {
      const int64_t col = pp / tz;
      const int z0 = (int)(pp - col * tz);
      const int z1 = (int)(pe - pp < (int64_t)(tz - z0) ? z0 + (pe - pp) : tz);
      const int item_i = (int)(col / p.nbands);
      const int y0 = (int)(col - (int64_t)item_i * p.nbands) * BY;
      const TileItem it = p.items ? p.items[item_i] : p.inline_items[item_i];
      const double* const* gs = p.gsrc + (size_t)it.tile * 6;
      const EdgePtr* es = P.esrc + (size_t)it.tile * 12;
      for (int z = z0 - 2; z <= z1 + 1; ++z, ++g) {
        const int s = (int)(g % C::S);
        mbar_wait(&empty[s], ((g / C::S) & 1u) ^ 1u);
        stage_x2<TX, BY, S>(stage_base + (size_t)s * C::STAGE_ELEMS, &full[s], it.in, gs, es, z, ty, tz,
                         y0, lane);
      }
      pp += z1 - z0;
    }
    return;
  }

  // ------------------------------------------------------- consumer warps
  const int tid = (int)threadIdx.x;
  const int c2 = tid % C::HALF, r0 = tid / C::HALF, xo = c2 * 2;
  const bool xlo_edge = c2 == 0, xhi_edge = c2 == C::HALF - 1;
  const double alpha = p.alpha;
  const uint64_t keep = (p.cache_flags & 2) ? policy_evict_last() : policy_evict_normal();
  auto cbar = [] { asm volatile("bar.sync 1, %0;" ::"n"(C::NT) : "memory"); };
  auto wait_g = [&](uint32_t g) { mbar_wait(&full[g % C::S], (g / C::S) & 1u); };
  auto release_g = [&](uint32_t g) {
    if (TILES_ARRIVE_PER_THREAD) {
      mbar_arrive(&empty[g % C::S]);
    } else {
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[g % C::S]);
    }
  };
  uint32_t seq = 0;

  for (int64_t pp = pb; pp < pe;) {
    const int64_t col = pp / tz;
    const int z0 = (int)(pp - col * tz);
    const int z1 = (int)(pe - pp < (int64_t)(tz - z0) ? z0 + (pe - pp) : tz);
    const int item_i = (int)(col / p.nbands);
    const int y0 = (int)(col - (int64_t)item_i * p.nbands) * BY;
    const TileItem it = p.items ? p.items[item_i] : p.inline_items[item_i];
    const int64_t tile = it.tile;
    const uint8_t fm = P.fixed_mask[tile];
    const int nq = z1 - z0 + 4;  // input planes z0-2 .. z1+1

    // input value of plane stage `st` at (x, y), x in [-2, TX+2)
    auto U = [&](const double* st, int x, int y) -> double {
      const int r = y - (y0 - 2);
      if (x < 0) return st[C::XOFF + r * 2 + (x + 2)];
      if (x >= TX) return st[C::XOFF + 2 * C::IROWS + r * 2 + (x - TX)];
      return st[r * TX + x];
    };
    auto U2 = [&](const double* st, int x, int y) -> double2 {
      return *reinterpret_cast<const double2*>(st + (y - (y0 - 2)) * TX + x);
    };
    auto stage = [&](uint32_t q) { return stage_base + (size_t)((seq + q) % C::S) * C::STAGE_ELEMS; };

    // exports of the output (D = 2 faces)
    double* fxm = p.fexp[XM] + tile * p.face_elems[XM];
    double* fxp = p.fexp[XP] + tile * p.face_elems[XP];
    double* fym = p.fexp[YM] + tile * p.face_elems[YM] + xo;
    double* fyp = p.fexp[YP] + tile * p.face_elems[YP] + xo;
    double* fzm = p.fexp[ZM] + tile * p.face_elems[ZM] + xo;
    double* fzp = p.fexp[ZP] + tile * p.face_elems[ZP] + xo;
    const int yb = y0 + r0;
    double* obase = it.out + (size_t)yb * TX + xo;
    const size_t plane_elems = (size_t)ty * TX;

    double2 zmr[C::NR];  // mid(o-1) at this thread's own output cells
    // u^{s+2} of plane o: MB == 2 at iteration mi: o = z0+mi-2 (mid(o), mid(o+1)
    // in buffers (mi-1)%2, mi%2); MB == 3: o = z0+mi-3 (buffers (mi-2)%3, (mi-1)%3)
    auto output_plane = [&](int mi) {
      const int o = z0 + mi - (MB == 3 ? 3 : 2);
      const double* cb = mid0 + (size_t)((mi - (MB == 3 ? 2 : 1)) % MB) * C::MID_ELEMS;  // mid(o)
      const double* nb = mid0 + (size_t)((mi - (MB == 3 ? 1 : 0)) % MB) * C::MID_ELEMS;  // mid(o+1)
      double* op = obase + (size_t)o * plane_elems;
      const bool zlo = o < 2, zhi = o >= tz - 2;
#pragma unroll
      for (int j = 0; j < C::NR; ++j) {
        const int r = r0 + j * C::RPP;  // band row
        const double* crow = cb + (r + 1) * C::MPITCH + xo + 2;
        const double2 c = *reinterpret_cast<const double2*>(crow);
        const double2 ym = *reinterpret_cast<const double2*>(crow - C::MPITCH);
        const double2 yp = *reinterpret_cast<const double2*>(crow + C::MPITCH);
        const double2 zp = *reinterpret_cast<const double2*>(nb + (r + 1) * C::MPITCH + xo + 2);
        const double xm = crow[-1], xp = crow[2];
        double2 v;
        v.x = heat_update(c.x, xm, c.y, ym.x, yp.x, zmr[j].x, zp.x, alpha);
        v.y = heat_update(c.y, c.x, xp, ym.y, yp.y, zmr[j].y, zp.y, alpha);
        stg2_stream(op + (size_t)j * C::RPP * TX, v);
        zmr[j] = c;
        const int y = yb + j * C::RPP;
        if (xlo_edge) st2_hint(fxm + ((size_t)o * ty + y) * 2, v, keep);
        if (xhi_edge) st2_hint(fxp + ((size_t)o * ty + y) * 2, v, keep);
        if (y < 2) st2_hint(fym + ((size_t)o * 2 + y) * TX, v, keep);
        if (y >= ty - 2) st2_hint(fyp + ((size_t)o * 2 + y - (ty - 2)) * TX, v, keep);
        if (zlo) st2_hint(fzm + ((size_t)o * ty + y) * TX, v, keep);
        if (zhi) st2_hint(fzp + ((size_t)(o - (tz - 2)) * ty + y) * TX, v, keep);
      }
    };
    wait_g(seq);
    wait_g(seq + 1);
    const int nmid = z1 - z0 + 2;  // mid planes z0-1 .. z1
    // MB == 3: iteration mi computes mid(m) and, independently, the output
    // of plane m-2 (one barrier per plane); MB == 2: mid(m), barrier,
    // output of plane m-1, barrier.
    for (int mi = 0; mi < nmid + (MB == 3 ? 1 : 0); ++mi) {
      const int m = z0 - 1 + mi;
      if (MB == 3 && mi == nmid) {  // drain: last output only
        output_plane(mi);
        cbar();
        break;
      }
      wait_g(seq + mi + 2);
      const double* prv = stage(mi);
      const double* cur = stage(mi + 1);
      const double* nxt = stage(mi + 2);
      double* mb = mid0 + (size_t)(mi % MB) * C::MID_ELEMS;
      const bool zring = m < 0 || m >= tz;
      const bool zfixed = zring && (fm & bit(m < 0 ? ZM : ZP));
      // --- u^{s+1}: band rows +-1 (band rows only on z-ring planes), x pairs
      const int ry0 = zring ? 1 : 0, ry1 = zring ? C::MROWS - 1 : C::MROWS;
      for (int e = tid; e < (ry1 - ry0) * C::HALF; e += C::NT) {
        const int mr = ry0 + e / C::HALF;
        const int x = (e % C::HALF) * 2;
        const int y = y0 - 1 + mr;
        double2 v;
        const bool yout = y < 0 || y >= ty;
        if (zfixed || (yout && (fm & bit(y < 0 ? YM : YP)))) {
          v = U2(cur, x, y);  // Dirichlet: the ring keeps its fixed value
        } else {
          const double2 c = U2(cur, x, y);
          const double2 ym = U2(cur, x, y - 1), yp = U2(cur, x, y + 1);
          const double2 zm = U2(prv, x, y), zp = U2(nxt, x, y);
          const double xm = U(cur, x - 1, y), xp = U(cur, x + 2, y);
          v.x = heat_update(c.x, xm, c.y, ym.x, yp.x, zm.x, zp.x, alpha);
          v.y = heat_update(c.y, c.x, xp, ym.y, yp.y, zm.y, zp.y, alpha);
        }
        *reinterpret_cast<double2*>(mb + mr * C::MPITCH + x + 2) = v;
      }
      if (!zring) {  // x ring columns x = -1, TX for band rows
        // on warps that did not take an extra row above (load balance)
        constexpr int RB = (C::MROWS * C::HALF) % C::NT == 0 ? 0
                           : (((C::MROWS * C::HALF) % C::NT + 31) / 32) * 32;
        constexpr int R0 = (C::NT - RB >= 2 * BY) ? RB : 0;
        const int e = tid - R0;
        if (e >= 0 && e < 2 * BY) {
          const int side = e / BY;
          const int y = y0 + e % BY;
          const int rr = y - (y0 - 2);
          const double* xb = cur + C::XOFF + side * 2 * C::IROWS + rr * 2;  // [rr][2]
          const int own = side ? 0 : 1, far = side ? 1 : 0;   // layer of x = -1/TX, -2/TX+1
          double v;
          if (fm & bit(side ? XP : XM)) {
            v = xb[own];
          } else {
            const double inner = cur[rr * TX + (side ? TX - 1 : 0)];
            const double xm = side ? inner : xb[far], xp = side ? xb[far] : inner;
            v = heat_update(xb[own], xm, xp, xb[own - 2], xb[own + 2],
                            prv[C::XOFF + side * 2 * C::IROWS + rr * 2 + own],
                            nxt[C::XOFF + side * 2 * C::IROWS + rr * 2 + own], alpha);
          }
          mb[(y - y0 + 1) * C::MPITCH + (side ? TX + 2 : 1)] = v;
        }
      }
      if (MB == 3) {
        if (mi == 2) {  // mid(z0-1) to registers before its buffer is reused
#pragma unroll
          for (int j = 0; j < C::NR; ++j)
            zmr[j] = *reinterpret_cast<const double2*>(mid0 + (r0 + j * C::RPP + 1) * C::MPITCH + xo + 2);
        }
        if (mi >= 3) output_plane(mi);
        cbar();  // mid(m) complete, output(m-2) done; input plane m-1 no longer read
        release_g(seq + mi);
        continue;
      }
      cbar();                // mid plane m complete; input plane m-1 no longer read
      release_g(seq + mi);
      if (mi == 0) {
#pragma unroll
        for (int j = 0; j < C::NR; ++j)
          zmr[j] = *reinterpret_cast<const double2*>(mb + (r0 + j * C::RPP + 1) * C::MPITCH + xo + 2);
      }
      if (mi >= 2) {
        output_plane(mi);
        cbar();  // mid(o) may be overwritten by the next mid plane
      }
    }
    release_g(seq + nq - 2);
    release_g(seq + nq - 1);
    seq += (uint32_t)nq;
    pp += z1 - z0;
  }
}

// ---- heat7x2r: the same two-step pass with a row-owning thread layout
// (TX = 64: one warp spans the tile width, lane l owns the x-pair 2l). 16
// "row warps" own RW = BY/16 consecutive band rows each and keep their mid
// values u^{s+1} of planes m-2, m-1, m in registers, so the second step reads
// shared memory only for the two neighbour rows and, on the edge lanes, the
// x ring; x neighbours come by warp shuffle. A "ring warp" computes the mid
// halo rows (y0-1, y0+BY) and the x-ring columns (x = -1, TX) of each plane.
// One named barrier per plane; mid planes in a ring of 3 shared buffers
// (a buffer is rewritten two barriers after its last read). Same stage
// layout, producer and rounded operations as heat7x2.
template <int BY, int S>
struct X2R {
  static constexpr int TX = 64;
  using L = X2<TX, BY, S, 2>;
  static constexpr int RW = BY / 16;          // band rows per row warp
  static constexpr int NT = 17 * 32;          // 16 row warps + ring warp
  static constexpr size_t SMEM = (size_t)S * L::STAGE_ELEMS * 8 + 3 * (size_t)L::MID_ELEMS * 8 + 2 * S * 8;
  static_assert(BY % 16 == 0 && RW >= 1 && RW <= 4, "bad x2r band");
};

template <int BY, int S>
__global__ void __launch_bounds__(X2R<BY, S>::NT + 32) heat7x2r(const __grid_constant__ Heat2Params P) {
  using R = X2R<BY, S>;
  using C = typename R::L;
  constexpr int TX = 64, RW = R::RW;
  const HeatParams& p = P.h;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double* stage_base = reinterpret_cast<double*>(smem_raw);
  double* mid0 = stage_base + (size_t)S * C::STAGE_ELEMS;
  uint64_t* full = reinterpret_cast<uint64_t*>(mid0 + 3 * C::MID_ELEMS);
  uint64_t* empty = full + S;
  constexpr int NCW = R::NT / 32;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], TILES_ARRIVE_PER_THREAD ? 32 : 1);
      mbar_init(&empty[s], TILES_ARRIVE_PER_THREAD ? NCW * 32 : NCW);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const int ty = p.ty, tz = p.tz;
  const int64_t P_all = (int64_t)p.nitems * p.nbands * tz;
  const int64_t pb = P_all * blockIdx.x / gridDim.x, pe = P_all * (blockIdx.x + 1) / gridDim.x;
  const int lane = (int)threadIdx.x & 31, warp = (int)threadIdx.x >> 5;

  if (warp == 17) {  // ---------------------------------------- producer warp
    uint32_t g = 0;
    for (int64_t pp = pb; pp < pe;) {
      const int64_t col = pp / tz;
      const int z0 = (int)(pp - col * tz);
      const int z1 = (int)(pe - pp < (int64_t)(tz - z0) ? z0 + (pe - pp) : tz);
      const int item_i = (int)(col / p.nbands);
      const int y0 = (int)(col - (int64_t)item_i * p.nbands) * BY;
      const TileItem it = p.items ? p.items[item_i] : p.inline_items[item_i];
      const double* const* gs = p.gsrc + (size_t)it.tile * 6;
      const EdgePtr* es = P.esrc + (size_t)it.tile * 12;
      for (int z = z0 - 2; z <= z1 + 1; ++z, ++g) {
        const int s = (int)(g % S);
        mbar_wait(&empty[s], ((g / S) & 1u) ^ 1u);
        stage_x2<TX, BY, S>(stage_base + (size_t)s * C::STAGE_ELEMS, &full[s], it.in, gs, es, z, ty, tz, y0,
                            lane);
      }
      pp += z1 - z0;
    }
    return;
  }

  // ---------------------------------------------------------- consumers
  const bool ring = warp == 16;
  const int x = 2 * lane;
  const int rb = RW * warp;  // first band row of a row warp
  const double alpha = p.alpha;
  const uint64_t keep = (p.cache_flags & 2) ? policy_evict_last() : policy_evict_normal();
  auto cbar = [] { asm volatile("bar.sync 1, %0;" ::"n"(R::NT) : "memory"); };
  auto wait_g = [&](uint32_t g) { mbar_wait(&full[g % S], (g / S) & 1u); };
  auto release_g = [&](uint32_t g) {
    if (TILES_ARRIVE_PER_THREAD) {
      mbar_arrive(&empty[g % S]);
    } else {
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[g % S]);
    }
  };
  auto row2 = [&](const double* st, int r) {  // band row r (y = y0 + r) of a stage, at x
    return *reinterpret_cast<const double2*>(st + (r + 2) * TX + x);
  };
  auto mid2 = [&](const double* mb, int r) -> double2& {
    return *reinterpret_cast<double2*>(const_cast<double*>(mb) + (r + 1) * C::MPITCH + x + 2);
  };
  uint32_t seq = 0, gm = 0;  // input stage and mid plane counters (across columns)

  for (int64_t pp = pb; pp < pe;) {
    const int64_t col = pp / tz;
    const int z0 = (int)(pp - col * tz);
    const int z1 = (int)(pe - pp < (int64_t)(tz - z0) ? z0 + (pe - pp) : tz);
    const int item_i = (int)(col / p.nbands);
    const int y0 = (int)(col - (int64_t)item_i * p.nbands) * BY;
    const TileItem it = p.items ? p.items[item_i] : p.inline_items[item_i];
    const int64_t tile = it.tile;
    const uint8_t fm = P.fixed_mask[tile];
    const int nq = z1 - z0 + 4;    // input planes z0-2 .. z1+1
    const int nmid = z1 - z0 + 2;  // mid planes z0-1 .. z1
    auto stage = [&](int q) { return stage_base + (size_t)((seq + q) % S) * C::STAGE_ELEMS; };
    auto midb = [&](uint32_t k) { return mid0 + (size_t)(k % 3) * C::MID_ELEMS; };

    double* fxm = p.fexp[XM] + tile * p.face_elems[XM];
    double* fxp = p.fexp[XP] + tile * p.face_elems[XP];
    double* fym = p.fexp[YM] + tile * p.face_elems[YM] + x;
    double* fyp = p.fexp[YP] + tile * p.face_elems[YP] + x;
    double* fzm = p.fexp[ZM] + tile * p.face_elems[ZM] + x;
    double* fzp = p.fexp[ZP] + tile * p.face_elems[ZP] + x;
    double* obase = it.out + (size_t)(y0 + rb) * TX + x;
    const size_t plane_elems = (size_t)ty * TX;

    double2 mp[RW], mc[RW], mn[RW];  // mid(m-2), mid(m-1), mid(m) at own rows
    wait_g(seq);
    wait_g(seq + 1);
    for (int mi = 0; mi < nmid; ++mi) {
      const int m = z0 - 1 + mi;
      wait_g(seq + mi + 2);
      const double* prv = stage(mi);
      const double* cur = stage(mi + 1);
      const double* nxt = stage(mi + 2);
      double* mb = midb(gm + mi);
      const bool zring = m < 0 || m >= tz;
      if (!ring) {
        // ---- u^{s+1} of plane m at the warp's own rows
        const bool zfixed = zring && (fm & bit(m < 0 ? ZM : ZP));
        double2 c[RW];
#pragma unroll
        for (int j = 0; j < RW; ++j) c[j] = row2(cur, rb + j);
        const double2 hm = row2(cur, rb - 1), hp = row2(cur, rb + RW);
#pragma unroll
        for (int j = 0; j < RW; ++j) {
          if (zfixed) {
            mn[j] = c[j];
          } else {
            const int rr = rb + j + 2;  // staged row index
            double xm = __shfl_up_sync(0xffffffffu, c[j].y, 1);
            double xp = __shfl_down_sync(0xffffffffu, c[j].x, 1);
            if (lane == 0) xm = cur[C::XOFF + rr * 2 + 1];
            if (lane == 31) xp = cur[C::XOFF + 2 * C::IROWS + rr * 2];
            const double2 ym = j == 0 ? hm : c[j > 0 ? j - 1 : 0];
            const double2 yp = j == RW - 1 ? hp : c[j < RW - 1 ? j + 1 : 0];
            const double2 zm = row2(prv, rb + j), zp = row2(nxt, rb + j);
            mn[j].x = heat_update(c[j].x, xm, c[j].y, ym.x, yp.x, zm.x, zp.x, alpha);
            mn[j].y = heat_update(c[j].y, c[j].x, xp, ym.y, yp.y, zm.y, zp.y, alpha);
          }
          mid2(mb, rb + j) = mn[j];
        }
      } else if (!zring) {
        // ---- ring warp: mid halo rows y0-1, y0+BY (x-pairs) ...
#pragma unroll
        for (int h = 0; h < 2; ++h) {
          const int r = h ? BY : -1, y = y0 + r;
          const bool yout = y < 0 || y >= ty;
          const double2 c = row2(cur, r);
          double2 v;
          double xm = __shfl_up_sync(0xffffffffu, c.y, 1);
          double xp = __shfl_down_sync(0xffffffffu, c.x, 1);
          if (yout && (fm & bit(y < 0 ? YM : YP))) {
            v = c;  // Dirichlet: the ring keeps its fixed value
          } else {
            const int rr = r + 2;
            if (lane == 0) xm = cur[C::XOFF + rr * 2 + 1];
            if (lane == 31) xp = cur[C::XOFF + 2 * C::IROWS + rr * 2];
            const double2 ym = row2(cur, r - 1), yp = row2(cur, r + 1);
            const double2 zm = row2(prv, r), zp = row2(nxt, r);
            v.x = heat_update(c.x, xm, c.y, ym.x, yp.x, zm.x, zp.x, alpha);
            v.y = heat_update(c.y, c.x, xp, ym.y, yp.y, zm.y, zp.y, alpha);
          }
          mid2(mb, r) = v;
        }
        // ... and the x-ring columns x = -1, TX of the band rows
        for (int e = lane; e < 2 * BY; e += 32) {
          const int side = e / BY;
          const int y = y0 + e % BY;
          const int rr = y - (y0 - 2);
          const double* xb = cur + C::XOFF + side * 2 * C::IROWS + rr * 2;
          const int own = side ? 0 : 1, far = side ? 1 : 0;
          double v;
          if (fm & bit(side ? XP : XM)) {
            v = xb[own];
          } else {
            const double inner = cur[rr * TX + (side ? TX - 1 : 0)];
            const double xm = side ? inner : xb[far], xp = side ? xb[far] : inner;
            v = heat_update(xb[own], xm, xp, xb[own - 2], xb[own + 2],
                            prv[C::XOFF + side * 2 * C::IROWS + rr * 2 + own],
                            nxt[C::XOFF + side * 2 * C::IROWS + rr * 2 + own], alpha);
          }
          mb[(y - y0 + 1) * C::MPITCH + (side ? TX + 2 : 1)] = v;
        }
      }
      cbar();  // mid(m) complete; input plane m-1 no longer read
      release_g(seq + mi);
      if (!ring && mi >= 2) {
        // ---- u^{s+2} of plane o = m-1 at the own rows
        const int o = m - 1;
        const double* cb = midb(gm + mi - 1);  // mid(o): neighbour rows, x ring
        const double2 hm = mid2(cb, rb - 1), hp = mid2(cb, rb + RW);
        double* op = obase + (size_t)o * plane_elems;
        const bool zlo = o < 2, zhi = o >= tz - 2;
#pragma unroll
        for (int j = 0; j < RW; ++j) {
          const double2 c = mc[j];
          double xm = __shfl_up_sync(0xffffffffu, c.y, 1);
          double xp = __shfl_down_sync(0xffffffffu, c.x, 1);
          if (lane == 0) xm = cb[(rb + j + 1) * C::MPITCH + 1];
          if (lane == 31) xp = cb[(rb + j + 1) * C::MPITCH + TX + 2];
          const double2 ym = j == 0 ? hm : mc[j > 0 ? j - 1 : 0];
          const double2 yp = j == RW - 1 ? hp : mc[j < RW - 1 ? j + 1 : 0];
          double2 v;
          v.x = heat_update(c.x, xm, c.y, ym.x, yp.x, mp[j].x, mn[j].x, alpha);
          v.y = heat_update(c.y, c.x, xp, ym.y, yp.y, mp[j].y, mn[j].y, alpha);
          stg2_stream(op + (size_t)j * TX, v);
          const int y = y0 + rb + j;
          if (lane == 0) st2_hint(fxm + ((size_t)o * ty + y) * 2, v, keep);
          if (lane == 31) st2_hint(fxp + ((size_t)o * ty + y) * 2, v, keep);
          if (y < 2) st2_hint(fym + ((size_t)o * 2 + y) * TX, v, keep);
          if (y >= ty - 2) st2_hint(fyp + ((size_t)o * 2 + y - (ty - 2)) * TX, v, keep);
          if (zlo) st2_hint(fzm + ((size_t)o * ty + y) * TX, v, keep);
          if (zhi) st2_hint(fzp + ((size_t)(o - (tz - 2)) * ty + y) * TX, v, keep);
        }
      }
#pragma unroll
      for (int j = 0; j < RW; ++j) {
        mp[j] = mc[j];
        mc[j] = mn[j];
      }
    }
    release_g(seq + nq - 2);
    release_g(seq + nq - 1);
    seq += (uint32_t)nq;
    gm += (uint32_t)nmid;
    pp += z1 - z0;
  }
}

struct X2Entry {
  int tx, by, stages, mb, rows;  // rows = 1: heat7x2r (row-owning layout)
  void (*fn)(Heat2Params);
  int nt;
  size_t smem;
};
#define X2E(TX, BY, S, MB) \
  {TX, BY, S, MB, 0, heat7x2<TX, BY, S, MB>, X2<TX, BY, S, MB>::NT + 32, X2<TX, BY, S, MB>::SMEM}
#define X2RE(BY, S) {64, BY, S, 3, 1, heat7x2r<BY, S>, X2R<BY, S>::NT + 32, X2R<BY, S>::SMEM}
// x2r at band 32 / 6 stages: 0.788 ms per C2 pass vs 0.803 for heat7x2<64,64,4,2>
// (band 64 x2r: 0.997 ms — 18 warps cap it at 96 registers, and it cannot be
// resident under ncu), profiles/r01/x2_profile/
static const X2Entry kX2[] = {X2RE(32, 6),
                              X2E(64, 64, 4, 2), X2E(64, 32, 5, 3), X2E(64, 32, 4, 3),
                              X2E(64, 32, 6, 2), X2E(32, 32, 6, 3), X2E(32, 16, 6, 3),
                              X2E(128, 16, 4, 3), X2E(256, 8, 4, 3)};
#undef X2E
#undef X2RE

static const X2Entry* find_x2(int tx, int by, int st = 0) {
  if (!st)
    if (const char* es = std::getenv("TILES_X2_STAGES")) st = std::atoi(es);  // tuning override
  static const int rows = [] {  // TILES_X2_ROWS=0: the original thread layout only
    const char* e = std::getenv("TILES_X2_ROWS");
    return e ? std::atoi(e) : 1;
  }();
  for (const auto& e : kX2)
    if (e.tx == tx && e.by == by && (!st || e.stages == st) && (rows || !e.rows)) return &e;
  return nullptr;
}

bool heat2_plan(int tx, int ty, int max_smem, int* band, size_t* smem) {
  if (const char* eb = std::getenv("TILES_X2_BAND")) {  // tuning override
    const int by = std::atoi(eb);
    const X2Entry* e = find_x2(tx, by);
    if (e && ty % by == 0 && e->smem <= (size_t)max_smem) {
      *band = by;
      *smem = e->smem;
      return true;
    }
  }
  for (int by : {32, 64, 16, 8}) {  // band 32 first: x2r (see kX2)
    if (ty % by) continue;
    const X2Entry* e = find_x2(tx, by);
    if (e && e->smem <= (size_t)max_smem) {
      *band = by;
      *smem = e->smem;
      return true;
    }
  }
  return false;
}

cudaError_t heat2_configure(int tx, int band, size_t smem, int* ctas_per_sm) {
  const X2Entry* e = find_x2(tx, band);
  if (!e || e->smem != smem) return cudaErrorInvalidValue;
  cudaError_t r = cudaFuncSetAttribute(e->fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (r != cudaSuccess) return r;
  r = cudaOccupancyMaxActiveBlocksPerMultiprocessor(ctas_per_sm, e->fn, e->nt, smem);
  if (r == cudaSuccess && *ctas_per_sm < 1) {
    cudaFuncAttributes fa{};
    cudaFuncGetAttributes(&fa, e->fn);
    std::fprintf(stderr, "libtiles: heat7x2 entry (tx %d, band %d, %d threads): regs %d, static smem %zu, "
                 "max threads %d, max dyn smem %d\n", tx, band, e->nt, fa.numRegs, fa.sharedSizeBytes,
                 fa.maxThreadsPerBlock, fa.maxDynamicSharedSizeBytes);
  }
  return r;
}

cudaError_t launch_heat7x2(const Heat2Params& p, size_t smem, int grid, cudaStream_t s) {
  const X2Entry* e = find_x2(p.h.tx, p.h.band);
  if (!e || e->smem != smem) return cudaErrorInvalidValue;
  void* args[] = {const_cast<Heat2Params*>(&p)};
  return cudaLaunchKernel(reinterpret_cast<const void*>(e->fn), dim3(grid), dim3(e->nt), args, smem, s);
}

}  // namespace tiles
