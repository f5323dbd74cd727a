// kernels_slab.cu — the stream-through (trapezoid) sweep kernel, DESIGN.md §5.
//
// One Jacobi sweep over planes [lo, hi) of a unit's slab (the unit's planes
// plus T halo planes on each side, periodic in x and y within the plane).
// Source and destination are "views" of the same logical slab:
//   - the dense scratch slab [plane][ny][nx] (middle sweeps),
//   - the tile-blocked resident array at local z = zbase + plane, wrapped
//     (first sweep: the gather is fused into it); with z-slab ranks, planes
//     beyond the slab come from the neighbours' planes in the halo layers,
//   - the unit's packed sub-tiles [layer tile][plane - first][ty][tx] (last
//     sweep: the scatter is fused into it),
//   - a ring of three units' packed sub-tiles (units u-1, u, u+1: the
//     out-of-core first sweep).
// Every cell update is the same rounded expression as heat7 (reading R1), so
// results are bit-identical to the untiled oracle.
//
// Register z-march: a thread owns one x-pair (double2) of BY rows and walks a
// chunk of planes keeping planes z-1, z, z+1 in registers;
// the y neighbours are its own rows (plus two halo rows per plane), the x
// neighbours come from the adjacent lanes by shuffle (warp-edge lanes load
// them). Per cell: one 16-B load and one 16-B store of algorithmic traffic.
#include <cuda.h>
#include <cstdlib>
#include <numeric>

#include "kernels.cuh"
#include "ptx.cuh"

namespace tiles {

struct ViewDev {
  double* base;
  int64_t te;
  int tx, ty, tz, ntx, nty, zbase, nz;
  int ring, u, U, un;
  double* ub[3];
  double* hlo;
  double* hhi;
  int nlo;
  // first element of slab plane pl (x = y = 0 of tile column 0, row 0)
  __device__ __forceinline__ double* P(int pl) const {
    int gz = zbase + pl;
    if (hlo && gz < 0) {  // lower rank's top planes / wavefront scratch: nlo tile layers
      const int q = gz + nlo * tz, L = q / tz;
      return hlo + (int64_t)L * nty * ntx * te + (int64_t)(q - L * tz) * ty * tx;
    }
    if (hhi && gz >= nz) return hhi + (int64_t)(gz - nz) * ty * tx;  // upper rank's bottom planes
    if (nz > 0) {
      gz %= nz;
      if (gz < 0) gz += nz;
    }
    if (ring) {
      const int iu = gz / un;
      int k = iu - u + 1;
      if (k < 0) k += U;
      if (k >= U) k -= U;
      double* b = k == 0 ? ub[0] : k == 1 ? ub[1] : ub[2];  // selects, not a local-memory array
      return b + (int64_t)(gz - iu * un) * ty * tx;
    }
    const int iz = gz / tz, lz = gz - iz * tz;
    return base + (int64_t)iz * nty * ntx * te + (int64_t)lz * ty * tx;
  }
  // plane of pl inside its tile layer (the pointer of pl+1 is P(pl) + ty*tx
  // unless this is tz - 1); views without layers (tz = 2^30) never wrap
  __device__ __forceinline__ int LZ(int pl) const {
    int gz = zbase + pl;
    if (hlo && gz < 0) return (gz + nlo * tz) % tz;
    if (hhi && gz >= nz) return gz - nz;
    if (nz > 0) {
      gz %= nz;
      if (gz < 0) gz += nz;
    }
    return gz % tz;
  }
  __device__ __forceinline__ int64_t Y(int y) const {
    const int iy = y / ty;
    return (int64_t)iy * ntx * te + (int64_t)(y - iy * ty) * tx;
  }
  __device__ __forceinline__ int64_t X(int x) const {
    const int ix = x / tx;
    return (int64_t)ix * te + (x - ix * tx);
  }
};

static ViewDev to_dev(const SlabView& v) {
  return ViewDev{v.base, v.te, v.tx, v.ty, v.tz, v.ntx, v.nty, v.zbase, v.nz, v.ring, v.u, v.U, v.un,
                 {v.ubase[0], v.ubase[1], v.ubase[2]}, v.hlo, v.hhi, v.nlo > 0 ? v.nlo : 1};
}

// Work items are (z chunk, column) pairs, column = (x segment of 128 pairs,
// group of BY rows), enumerated chunk-major; a resident grid of (SMs x
// blocks per SM) takes them round-robin, so blocks running at the same time
// work on neighbouring columns of the same z chunk and the halo rows they
// share come from L2.
template <int BY>
__global__ void __launch_bounds__(128, 4) slab_sweep_zm(const ViewDev S, const ViewDev D, const int nx,
                                                        const int ny, const int lo, const int hi,
                                                        const int gx, const int zc, const double alpha) {
  const int npairs = nx >> 1;
  const int lane = threadIdx.x & 31;
  const int cols = gx * (ny / BY);
  const int nch = (hi - lo + zc - 1) / zc;
  const int64_t items = (int64_t)cols * nch;
  const int stx = S.tx, dtx = D.tx;

  for (int64_t it = blockIdx.x; it < items; it += gridDim.x) {
    const int ch = (int)(it / cols), col = (int)(it - (int64_t)ch * cols);
    const int zlo = lo + ch * zc, zhi = min(hi, zlo + zc);
    const int seg = col % gx, y0 = (col / gx) * BY;
    const int px = seg * 128 + (int)threadIdx.x;
    const bool valid = px < npairs;
    const int x = 2 * (valid ? px : npairs - 1);
    const bool ledge = lane == 0, redge = lane == 31 || px + 1 >= npairs;
    const int64_t sx = S.X(x), dx = D.X(x);
    const int64_t exo_m = S.X(x == 0 ? nx - 1 : x - 1) - sx, exo_p = S.X(x + 2 == nx ? 0 : x + 2) - sx;
    // BY divides ty in every view (the launcher picks it so): the BY rows
    // are consecutive rows of one tile row, row j at Y(y0) + j * tx
    const int64_t sy0 = S.Y(y0) + sx, dy0 = D.Y(y0) + dx;
    const int64_t shm = S.Y(y0 == 0 ? ny - 1 : y0 - 1) + sx;
    const int64_t shp = S.Y(y0 + BY == ny ? 0 : y0 + BY) + sx;

    double2 zm[BY], zcur[BY];
    {
      const double* p0 = S.P(zlo - 1);
      const double* p1 = S.P(zlo);
#pragma unroll
      for (int j = 0; j < BY; ++j) {
        zm[j] = *reinterpret_cast<const double2*>(p0 + sy0 + (int64_t)j * stx);
        zcur[j] = *reinterpret_cast<const double2*>(p1 + sy0 + (int64_t)j * stx);
      }
    }
    for (int z = zlo; z < zhi; ++z) {
      const double* pc = S.P(z);
      const double* pn = S.P(z + 1);
      double2 zp[BY];
      double em[BY], ep[BY];
#pragma unroll
      for (int j = 0; j < BY; ++j) {
        const int64_t r = sy0 + (int64_t)j * stx;
        zp[j] = *reinterpret_cast<const double2*>(pn + r);
        em[j] = ledge ? pc[r + exo_m] : 0.0;
        ep[j] = redge ? pc[r + exo_p] : 0.0;
      }
      const double2 hm = *reinterpret_cast<const double2*>(pc + shm);
      const double2 hp = *reinterpret_cast<const double2*>(pc + shp);
      double* pd = D.P(z);
#pragma unroll
      for (int j = 0; j < BY; ++j) {
        const double2 c = zcur[j];
        double xm = __shfl_up_sync(0xffffffffu, c.y, 1);
        double xp = __shfl_down_sync(0xffffffffu, c.x, 1);
        if (ledge) xm = em[j];
        if (redge) xp = ep[j];
        const double2 ym = j == 0 ? hm : zcur[j > 0 ? j - 1 : 0];
        const double2 yp = j == BY - 1 ? hp : zcur[j < BY - 1 ? j + 1 : 0];
        double2 v;
        v.x = heat_update(c.x, xm, c.y, ym.x, yp.x, zm[j].x, zp[j].x, alpha);
        v.y = heat_update(c.y, c.x, xp, ym.y, yp.y, zm[j].y, zp[j].y, alpha);
        if (valid) *reinterpret_cast<double2*>(pd + dy0 + (int64_t)j * dtx) = v;
      }
#pragma unroll
      for (int j = 0; j < BY; ++j) {
        zm[j] = zcur[j];
        zcur[j] = zp[j];
      }
    }
  }
}

// cp.async variant: the same z-march and work order, but every plane a
// thread needs (its BY rows, the two halo rows, the x-edge cells of the warp's
// edge lanes) is fetched S-1 planes ahead with cp.async into a per-thread
// shared-memory ring ([stage][row][thread], conflict-free), one commit group
// per plane. A thread reads only what it fetched itself, so wait_group alone
// orders it (no block barrier); deep memory-level parallelism at a low
// register count.
__device__ __forceinline__ void cp16(void* sdst, const void* gsrc) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"((uint32_t)__cvta_generic_to_shared(sdst)),
               "l"(gsrc)
               : "memory");
}
__device__ __forceinline__ void cp8(void* sdst, const void* gsrc) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8;" ::"r"((uint32_t)__cvta_generic_to_shared(sdst)),
               "l"(gsrc)
               : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

template <int BY, int SG>
struct CaLayout {
  static constexpr int ROWS = BY + 2;                      // own rows, then halo y0-1, y0+BY
  static constexpr int STAGE_V = ROWS * 128;                // double2 per stage (all threads)
  static constexpr int EDGE_D = 4 * 2 * BY;                 // doubles per stage: [warp][side][row]
  static constexpr size_t SMEM = (size_t)SG * (STAGE_V * 16 + EDGE_D * 8);
};

template <int BY, int SG>
__global__ void __launch_bounds__(128, 4) slab_sweep_ca(const ViewDev S, const ViewDev D, const int nx,
                                                        const int ny, const int lo, const int hi,
                                                        const int gx, const int zc, const double alpha) {
  using L = CaLayout<BY, SG>;
  extern __shared__ __align__(16) unsigned char smem_raw[];
  double2* ring = reinterpret_cast<double2*>(smem_raw);
  double* edges = reinterpret_cast<double*>(smem_raw + (size_t)SG * L::STAGE_V * 16);
  const int npairs = nx >> 1;
  const int tid = (int)threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const int cols = gx * (ny / BY);
  const int nch = (hi - lo + zc - 1) / zc;
  const int64_t items = (int64_t)cols * nch;
  const int stx = S.tx, dtx = D.tx;
  auto slot = [&](int st, int row) -> double2& { return ring[(st * L::ROWS + row) * 128 + tid]; };
  auto edge = [&](int st, int side, int row) -> double& {
    return edges[((st * 4 + warp) * 2 + side) * BY + row];
  };

  for (int64_t it = blockIdx.x; it < items; it += gridDim.x) {
    const int ch = (int)(it / cols), col = (int)(it - (int64_t)ch * cols);
    const int zlo = lo + ch * zc, zhi = min(hi, zlo + zc);
    const int seg = col % gx, y0 = (col / gx) * BY;
    const int px = seg * 128 + tid;
    const bool valid = px < npairs;
    const int x = 2 * (valid ? px : npairs - 1);
    // one edge lane per side per warp (the smem edge slots have one writer);
    // invalid (clamped) lanes store nothing and need no edges
    const bool ledge = valid && lane == 0, redge = valid && (lane == 31 || px + 1 == npairs);
    const int64_t sx = S.X(x), dx = D.X(x);
    const int64_t exo_m = S.X(x == 0 ? nx - 1 : x - 1) - sx, exo_p = S.X(x + 2 == nx ? 0 : x + 2) - sx;
    const int64_t sy0 = S.Y(y0) + sx, dy0 = D.Y(y0) + dx;
    const int64_t shm = S.Y(y0 == 0 ? ny - 1 : y0 - 1) + sx;
    const int64_t shp = S.Y(y0 + BY == ny ? 0 : y0 + BY) + sx;
    // planes zlo-1 .. zhi; plane q = zlo - 1 + i goes to stage i % SG
    const int nplanes = zhi - zlo + 2;
    auto fetch = [&](int i) {
      if (i < nplanes) {
        const int z = zlo - 1 + i, st = i % SG;
        const double* pz = S.P(z);
#pragma unroll
        for (int j = 0; j < BY; ++j) {
          const double* g = pz + sy0 + (int64_t)j * stx;
          cp16(&slot(st, j), g);
          if (ledge) cp8(&edge(st, 0, j), g + exo_m);
          if (redge) cp8(&edge(st, 1, j), g + exo_p);
        }
        cp16(&slot(st, BY), pz + shm);
        cp16(&slot(st, BY + 1), pz + shp);
      }
      cp_commit();  // (possibly empty) group per plane keeps the count uniform
    };
#pragma unroll
    for (int i = 0; i < SG; ++i) fetch(i);
    cp_wait<SG - 2>();  // planes zlo-1, zlo landed
    double2 zm[BY], zcur[BY];
#pragma unroll
    for (int j = 0; j < BY; ++j) {
      zm[j] = slot(0, j);
      zcur[j] = slot(1 % SG, j);
    }
    for (int z = zlo; z < zhi; ++z) {
      const int i = z - zlo + 1;  // plane z is index i, z+1 is i+1
      fetch(i + SG - 1);          // into the stage of plane i-1 (its rows are in zm)
      cp_wait<SG - 2>();          // plane i+1 landed
      const int sc = i % SG, sn = (i + 1) % SG;
      const double2 hm = slot(sc, BY), hp = slot(sc, BY + 1);
      double* pd = D.P(z);
#pragma unroll
      for (int j = 0; j < BY; ++j) {
        const double2 c = zcur[j];
        const double2 zp = slot(sn, j);
        double xm = __shfl_up_sync(0xffffffffu, c.y, 1);
        double xp = __shfl_down_sync(0xffffffffu, c.x, 1);
        if (ledge) xm = edge(sc, 0, j);
        if (redge) xp = edge(sc, 1, j);
        const double2 ym = j == 0 ? hm : zcur[j > 0 ? j - 1 : 0];
        const double2 yp = j == BY - 1 ? hp : zcur[j < BY - 1 ? j + 1 : 0];
        double2 v;
        v.x = heat_update(c.x, xm, c.y, ym.x, yp.x, zm[j].x, zp.x, alpha);
        v.y = heat_update(c.y, c.x, xp, ym.y, yp.y, zm[j].y, zp.y, alpha);
        if (valid) *reinterpret_cast<double2*>(pd + dy0 + (int64_t)j * dtx) = v;
      }
#pragma unroll
      for (int j = 0; j < BY; ++j) {  // after the row loop: rows j+-1 read zcur of plane z
        zm[j] = zcur[j];
        zcur[j] = slot(sn, j);
      }
    }
    cp_wait<0>();  // drain the (empty) tail groups before the ring is reused
  }
}

// ---- tile-column TMA variant (the default for tile-blocked views of 64-wide
// tiles): a CTA's column is a band of BY rows of one 64-wide tile column, so
// per plane the producer issues five TMA operations, as heat7_fixed does —
// the band (BY rows, one contiguous range inside a tile), the two y-halo rows
// (periodic, possibly in the neighbour tiles) and, since the x neighbours'
// cells are a strided column, two 2-D tensor copies of a {2 x BY} box of the
// neighbour tile columns (the slot pool / wavefront scratch seen as rows of
// 64 doubles, SweepMaps). Consumers: register z-march, NR rows per thread.
template <int BY, int RPP, int S>
struct TileCfg {
  static constexpr int TX = 64;
  static constexpr int HALF = TX / 2;
  static constexpr int NT = RPP * HALF;
  static constexpr int NR = BY / RPP;
  static constexpr int ROWS = BY + 2;
  static constexpr int XH = ROWS * TX;               // x-halo boxes: [side][BY][2]
  static constexpr int STAGE = XH + 4 * BY;          // doubles (a multiple of 16: 128-B aligned stages)
  static constexpr uint32_t BYTES = (uint32_t)STAGE * 8;
  static constexpr size_t SMEM = (size_t)S * STAGE * 8 + (size_t)2 * S * 8;
  static_assert(BY % RPP == 0 && NT % 32 == 0 && (STAGE % 16) == 0, "bad tile-sweep config");
};

static __device__ __forceinline__ void tma_2d(void* dst, const TensorMapBlob* map, int c0, int c1, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
          smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(smem_u32(bar))
      : "memory");
}

// CS: a consumer thread's NR rows are consecutive (y neighbours of its inner
// rows from its own registers) instead of RPP rows apart
// XS: x neighbours by warp shuffle (a warp holds one 64-wide row) instead
// of shared-memory loads
template <int BY, int RPP, int S, int MB, bool CS = false, bool XS = false>
__global__ void __launch_bounds__(TileCfg<BY, RPP, S>::NT + 32, MB)
    slab_sweep_tile(const ViewDev Sv, const ViewDev Dv, const __grid_constant__ SweepMaps maps, const int ny,
                    const int lo, const int hi, const double alpha, const int st_mode) {
  using C = TileCfg<BY, RPP, S>;
  constexpr int TX = C::TX;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double* stage = reinterpret_cast<double*>(smem_raw);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem_raw + (size_t)S * C::STAGE * 8);
  uint64_t* empty = full + S;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], C::NT);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  // programmatic dependent launch: the next sweep on this stream may be
  // scheduled now (it waits for this grid before touching memory, below)
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const int ntx = Sv.ntx * Sv.tx / TX;  // 64-wide columns per row (views share nx)
  const int np = hi - lo;
  const int64_t ncols = (int64_t)ntx * (ny / BY);
  const int64_t P = ncols * np;
  const int64_t pb = P * blockIdx.x / gridDim.x, pe = P * (blockIdx.x + 1) / gridDim.x;

  if ((int)threadIdx.x >= C::NT) {  // ---------------- producer (one thread)
    if (threadIdx.x != C::NT) return;
    // the previous kernel on the stream complete and its writes visible
    // before the first load (consumers write only after consuming a stage,
    // so this also orders their stores after the previous grid's reads)
    asm volatile("griddepcontrol.wait;" ::: "memory");
    // L2 policy of the staged loads (st_mode >> 4, TILES_SWEEP_LD): 0 none,
    // 1 evict_first (a level's input is dead after the sweep), 2 evict_last
    const int ldm = st_mode >> 4;
    const uint64_t lpol = ldm == 2 ? policy_evict_last() : policy_evict_first();
    uint32_t g = 0;
    for (int64_t pp = pb; pp < pe;) {
      const int64_t col = pp / np;
      const int z0 = lo + (int)(pp - col * np);
      const int64_t left = pe - pp, inrun = lo + np - z0;
      const int n = (int)(left < inrun ? left : inrun);
      pp += n;
      const int cx = (int)(col % ntx), y0 = (int)(col / ntx) * BY;
      const int x0 = cx * TX, xl = (cx == 0 ? ntx - 1 : cx - 1) * TX, xr = (cx == ntx - 1 ? 0 : cx + 1) * TX;
      const int ym = y0 == 0 ? ny - 1 : y0 - 1, yp = y0 + BY == ny ? 0 : y0 + BY;
      const int64_t oband = Sv.Y(y0) + Sv.X(x0), om = Sv.Y(ym) + Sv.X(x0), op = Sv.Y(yp) + Sv.X(x0);
      const int64_t oxl = Sv.Y(y0) + Sv.X(xl), oxr = Sv.Y(y0) + Sv.X(xr);
      for (int q = 0; q < n + 2; ++q, ++g) {
        const int z = z0 - 1 + q;
        const int st = (int)(g % S);
        mbar_wait(&empty[st], ((g / S) & 1u) ^ 1u);
        double* dst = stage + (size_t)st * C::STAGE;
        const double* pz = Sv.P(z);
        fence_proxy_async();
        mbar_expect_tx(&full[st], C::BYTES);
        if (ldm) {
          bulk_g2s_hint(dst + TX, pz + oband, (uint32_t)BY * TX * 8, &full[st], lpol);
          bulk_g2s_hint(dst, pz + om, TX * 8, &full[st], lpol);
          bulk_g2s_hint(dst + (BY + 1) * TX, pz + op, TX * 8, &full[st], lpol);
        } else {
          bulk_g2s(dst + TX, pz + oband, (uint32_t)BY * TX * 8, &full[st]);
          bulk_g2s(dst, pz + om, TX * 8, &full[st]);
          bulk_g2s(dst + (BY + 1) * TX, pz + op, TX * 8, &full[st]);
        }
        const double* a = pz + oxl;
        const double* b = pz + oxr;
        const int ka = (a >= maps.base[1] && a < maps.end[1]) ? 1 : 0;
        const int kb = (b >= maps.base[1] && b < maps.end[1]) ? 1 : 0;
        tma_2d(dst + C::XH, &maps.xmap[ka], TX - 2, (int)((a - maps.base[ka]) / TX), &full[st]);
        tma_2d(dst + C::XH + 2 * BY, &maps.xmap[kb], 0, (int)((b - maps.base[kb]) / TX), &full[st]);
      }
    }
    return;
  }

  // ------------------------------------------------------- consumer warps
  const int c2 = (int)threadIdx.x % C::HALF, r0 = (int)threadIdx.x / C::HALF;
  constexpr int RS = CS ? 1 : RPP;          // row step between a thread's rows
  const int rb = CS ? r0 * C::NR : r0;      // its first row in the band
  const int x = 2 * c2;
  const bool xl_edge = c2 == 0, xr_edge = c2 == C::HALF - 1;
  // output stores: streaming (evict-first; 0) or kept in L2 for the next
  // sweep's reads (1 evict_normal, 2 evict_last)
  const int stm = st_mode & 15;
  const uint64_t spol = stm == 2 ? policy_evict_last() : policy_evict_normal();
  // the x-halo cell of this thread's rows: left box column 1 (x = 63 of the
  // left tile), right box column 0 (x = 0 of the right tile)
  const int hoff = xl_edge ? C::XH + 2 * rb + 1 : C::XH + 2 * BY + 2 * rb;
  uint32_t seq = 0;
  auto wait_g = [&](uint32_t g) { mbar_wait(&full[g % S], (g / S) & 1u); };
  auto release_g = [&](uint32_t g) { mbar_arrive(&empty[g % S]); };
  for (int64_t pp = pb; pp < pe;) {
    const int64_t col = pp / np;
    const int z0 = lo + (int)(pp - col * np);
    const int64_t left = pe - pp, inrun = lo + np - z0;
    const int n = (int)(left < inrun ? left : inrun);
    pp += n;
    const int cx = (int)(col % ntx), y0 = (int)(col / ntx) * BY;
    const int64_t orow = Dv.Y(y0 + rb) + Dv.X(cx * TX + x);
    const int64_t ostep = Dv.Y(y0 + rb + RS) - Dv.Y(y0 + rb);  // rows of a band share a tile
    double2 zm[C::NR], zc[C::NR];
    wait_g(seq);
    wait_g(seq + 1);
    {
      const double* s0 = stage + (size_t)(seq % S) * C::STAGE + (rb + 1) * TX + x;
      const double* s1 = stage + (size_t)((seq + 1) % S) * C::STAGE + (rb + 1) * TX + x;
#pragma unroll
      for (int j = 0; j < C::NR; ++j) {
        zm[j] = *reinterpret_cast<const double2*>(s0 + j * RS * TX);
        zc[j] = *reinterpret_cast<const double2*>(s1 + j * RS * TX);
      }
    }
    release_g(seq);
    double* od = Dv.P(z0) + orow;
    int lz = Dv.LZ(z0);
    const int64_t pstride = (int64_t)Dv.ty * Dv.tx;
    for (int i = 0; i < n; ++i) {
      wait_g(seq + i + 2);
      const double* cur = stage + (size_t)((seq + i + 1) % S) * C::STAGE;
      const double* nxt = stage + (size_t)((seq + i + 2) % S) * C::STAGE + (rb + 1) * TX + x;
      const double* cc = cur + (rb + 1) * TX + x;
      double2 zpn[C::NR];
#pragma unroll
      for (int j = 0; j < C::NR; ++j) {
        const int jo = j * RS * TX;
        const double2 zp = *reinterpret_cast<const double2*>(nxt + jo);
        zpn[j] = zp;
        const double2 ym = CS && j > 0 ? zc[j > 0 ? j - 1 : 0] : *reinterpret_cast<const double2*>(cc + jo - TX);
        const double2 yp =
            CS && j < C::NR - 1 ? zc[j < C::NR - 1 ? j + 1 : 0] : *reinterpret_cast<const double2*>(cc + jo + TX);
        const double2 c = zc[j];
        double xm, xp;
        if (XS) {
          xm = __shfl_up_sync(0xffffffffu, c.y, 1);
          xp = __shfl_down_sync(0xffffffffu, c.x, 1);
        } else {
          xm = cc[jo - 1];
          xp = cc[jo + 2];
        }
        const double hv = cur[hoff + 2 * j * RS];
        if (xl_edge) xm = hv;
        if (xr_edge) xp = hv;
        double2 v;
        v.x = heat_update(c.x, xm, c.y, ym.x, yp.x, zm[j].x, zp.x, alpha);
        v.y = heat_update(c.y, c.x, xp, ym.y, yp.y, zm[j].y, zp.y, alpha);
        if (stm == 0) stg2_stream(od + j * ostep, v);
        else st2_hint(od + j * ostep, v, spol);
      }
#pragma unroll
      for (int j = 0; j < C::NR; ++j) {  // after the row loop: rows j+-1 read zc of this plane
        zm[j] = zc[j];
        zc[j] = zpn[j];
      }
      release_g(seq + i + 1);
      if (++lz == Dv.tz) {  // next tile layer (or the wrap): recompute
        od = Dv.P(z0 + i + 1) + orow;
        lz = 0;
      } else {
        od += pstride;
      }
    }
    release_g(seq + n + 1);
    seq += (uint32_t)(n + 2);
  }
}

template <int BY, int RPP, int S, int MB, bool CS = false, bool XS = false>
static cudaError_t launch_tile_cfg(const ViewDev& Sv, const ViewDev& Dv, const SweepMaps& m, int nx, int ny,
                                   int lo, int hi, double alpha, int sms, cudaStream_t s) {
  using C = TileCfg<BY, RPP, S>;
  static int occ = 0;
  if (!occ) {
    cudaError_t e = cudaFuncSetAttribute(slab_sweep_tile<BY, RPP, S, MB, CS, XS>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)C::SMEM);
    if (e != cudaSuccess) return e;
    int o = 1;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, slab_sweep_tile<BY, RPP, S, MB, CS, XS>, C::NT + 32, C::SMEM);
    occ = o < 1 ? 1 : o;
  }
  const int64_t P = (int64_t)(nx / 64) * (ny / BY) * (hi - lo);
  const int64_t grid = std::max<int64_t>(1, std::min<int64_t>((int64_t)sms * occ, P / 6));
  // stores evict_last by default: the next level's sweep reads them (a
  // 16-plane unit's two slabs nearly fit the 126 MB L2): 0.794 vs 0.761 of
  // HBM per launch, the e2e step the same or faster
  static const int st_mode = [] {
    const char* e = getenv("TILES_SWEEP_ST");
    const char* l = getenv("TILES_SWEEP_LD");
    return (e ? atoi(e) : 2) | ((l ? atoi(l) : 0) << 4);
  }();
  static const int pdl = [] {
    const char* e = getenv("TILES_SWEEP_PDL");
    return e ? atoi(e) : 1;
  }();
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(C::NT + 32);
  cfg.dynamicSmemBytes = C::SMEM;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  return cudaLaunchKernelEx(&cfg, slab_sweep_tile<BY, RPP, S, MB, CS, XS>, Sv, Dv, m, ny, lo, hi, alpha, st_mode);
}

// driver entry point for cuTensorMapEncodeTiled (no -lcuda link dependency)
using EncodeTiledFn = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                   const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                   CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static EncodeTiledFn encode_fn() {
  static EncodeTiledFn f = [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q{};
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess) return
        (EncodeTiledFn) nullptr;
    return reinterpret_cast<EncodeTiledFn>(p);
  }();
  return f;
}

// ---- two levels per pass: slab_sweep2_tile (the wavefront with three level
// buffers). A CTA owns runs of (band column, level-s+1 plane) pairs, as
// slab_sweep_tile does; a run of level-s+1 planes [p0, p1) needs level s on
// [p0-1, p1+1): planes below a (a-2, a-1: the previous chunk's top) are read
// through view mid, the others computed here from level s-1 on the band plus
// one row and one column on each side. Staging (one producer thread, nine
// TMA operations per plane): level s-1 rows y0-2 .. y0+BY+1 of the tile
// column (band; two contiguous row pairs, each inside one tile) and the x
// halos x0-2, x0-1 / x0+64, x0+65 of those rows (tensor-map boxes {2, BY} and
// {2, 2}). Consumers: warp w owns band rows w and w+16 (one pair per lane:
// x neighbours by shuffle) and, warps 0/1, the extended rows y0-1 / y0+BY;
// warps 2..4 compute the 68 extended-column cells (x = -1, 64). Both levels
// march z in registers (level s-1 at z-1, z; level s at z-2, z-1, z), so per
// cell pair and level only the y neighbours and the next plane come from
// shared memory; level s goes through a 3-plane shared ring for the other
// threads' y neighbours and the x edges, one named barrier per plane.
namespace w2 {
constexpr int BY = 32, TX = 64, NT = 512, S = 6;
constexpr int SROWS = BY + 4;                     // staged rows: y0-2 .. y0+BY+1
constexpr int XH = SROWS * TX;                    // x halos: per side boxes at 128-byte boundaries
constexpr int HS = 96;                            // doubles per side: rows 0-1 | 2..BY+1 | BY+2..BY+3
constexpr int STAGE = XH + 2 * HS;                // doubles (multiple of 16)
constexpr uint32_t BYTES = (uint32_t)(SROWS * TX + 4 * SROWS) * 8;
constexpr int MROWS = BY + 2, MW = 68;            // level-s plane: rows y0-1 .. y0+BY, x -2 .. 65
constexpr int MID = MROWS * MW;
constexpr size_t SMEM = (size_t)S * STAGE * 8 + (size_t)3 * MID * 8 + (size_t)2 * S * 8;
static_assert(STAGE % 16 == 0 && MID % 2 == 0 && NT == 16 * 32, "layout");
__device__ __forceinline__ int hoff(int side, int sr) {  // x-halo pair of staged row sr
  const int o = side * HS;
  return sr < 2 ? o + 2 * sr : sr < BY + 2 ? o + 16 + 2 * (sr - 2) : o + 80 + 2 * (sr - BY - 2);
}
}  // namespace w2

static __device__ __forceinline__ void bar_consumers512() { asm volatile("bar.sync 1, 512;" ::: "memory"); }

__global__ void __launch_bounds__(w2::NT + 32, 1)
    slab_sweep2_tile(const ViewDev Sv, const ViewDev Mv, const ViewDev Dv, const __grid_constant__ SweepMaps maps,
                     const int ny, const int a, const int b, const double alpha) {
  using namespace w2;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double* stage = reinterpret_cast<double*>(smem_raw);
  double* mid = stage + (size_t)S * STAGE;
  uint64_t* full = reinterpret_cast<uint64_t*>(mid + (size_t)3 * MID);
  uint64_t* empty = full + S;
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], NT);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const int ntx = Sv.ntx * Sv.tx / TX;
  const int np = b - a;  // level s+1 planes [a-1, b-1)
  const int64_t ncols = (int64_t)ntx * (ny / BY);
  const int64_t P = ncols * np;
  const int64_t pb = P * blockIdx.x / gridDim.x, pe = P * (blockIdx.x + 1) / gridDim.x;
  auto run_at = [&](int64_t pp, int64_t& col, int& p0, int& p1) {
    col = pp / np;
    p0 = a - 1 + (int)(pp - col * np);
    const int64_t left = pe - pp, inrun = (int64_t)(b - 1 - p0);
    p1 = p0 + (int)(left < inrun ? left : inrun);
  };
  auto plan = [&](int p0, int p1, int& zc0, int& nload) {
    zc0 = p0 - 1 > a ? p0 - 1 : a;  // first computed level-s plane
    const int nl = (a < p1 + 1 ? a : p1 + 1) - (p0 - 1);
    nload = nl > 0 ? nl : 0;        // level-s planes read: p0-1 .. p0-2+nload
  };

  if ((int)threadIdx.x >= NT) {  // ---------------- producer (one thread)
    if (threadIdx.x != NT) return;
    asm volatile("griddepcontrol.wait;" ::: "memory");
    uint32_t g = 0;
    for (int64_t pp = pb; pp < pe;) {
      int64_t col;
      int p0, p1, zc0, nload;
      run_at(pp, col, p0, p1);
      pp += p1 - p0;
      plan(p0, p1, zc0, nload);
      const int cx = (int)(col % ntx), y0 = (int)(col / ntx) * BY;
      const int x0 = cx * TX, xl = (cx == 0 ? ntx - 1 : cx - 1) * TX, xr = (cx == ntx - 1 ? 0 : cx + 1) * TX;
      const int ya = y0 < 2 ? y0 - 2 + ny : y0 - 2;
      const int yb = y0 + BY + 2 > ny ? y0 + BY - ny : y0 + BY;
      const int nstg = (p1 + 1) - zc0 + 2;  // level s-1 planes zc0-1 .. p1+1
      // in-plane offsets of the nine copies, per view (0: level s-1, 1: level s), once per run
      int64_t off[2][9];
#pragma unroll
      for (int v = 0; v < 2; ++v) {
        const ViewDev& V = v ? Mv : Sv;
        const int64_t oa = V.Y(ya), o0 = V.Y(y0), ob = V.Y(yb), xc = V.X(x0), xL = V.X(xl), xR = V.X(xr);
        off[v][0] = o0 + xc, off[v][1] = oa + xc, off[v][2] = ob + xc;
        off[v][3] = oa + xL, off[v][4] = o0 + xL, off[v][5] = ob + xL;
        off[v][6] = oa + xR, off[v][7] = o0 + xR, off[v][8] = ob + xR;
      }
      for (int q = 0; q < nload + nstg; ++q, ++g) {
        const bool ld = q < nload;
        const ViewDev& V = ld ? Mv : Sv;
        const int64_t* o = off[ld ? 1 : 0];
        const int z = ld ? p0 - 1 + q : zc0 - 1 + (q - nload);
        const int st = (int)(g % S);
        mbar_wait(&empty[st], ((g / S) & 1u) ^ 1u);
        double* dst = stage + (size_t)st * STAGE;
        const double* pz = V.P(z);
        fence_proxy_async();
        mbar_expect_tx(&full[st], BYTES);
        bulk_g2s(dst + 2 * TX, pz + o[0], (uint32_t)BY * TX * 8, &full[st]);
        bulk_g2s(dst, pz + o[1], 2 * TX * 8, &full[st]);
        bulk_g2s(dst + (BY + 2) * TX, pz + o[2], 2 * TX * 8, &full[st]);
        const int boff[3] = {0, 16, 80};
#pragma unroll
        for (int h = 0; h < 3; ++h) {
          const double* cl = pz + o[3 + h];
          const double* cr = pz + o[6 + h];
          const int kl = (cl >= maps.base[1] && cl < maps.end[1]) ? 1 : 0;
          const int kr = (cr >= maps.base[1] && cr < maps.end[1]) ? 1 : 0;
          tma_2d(dst + XH + boff[h], h == 1 ? &maps.xmap[kl] : &maps.xmap2[kl], TX - 2,
                 (int)((cl - maps.base[kl]) / TX), &full[st]);
          tma_2d(dst + XH + HS + boff[h], h == 1 ? &maps.xmap[kr] : &maps.xmap2[kr], 0,
                 (int)((cr - maps.base[kr]) / TX), &full[st]);
        }
      }
    }
    return;
  }

  // ------------------------------------------------------- consumer warps
  const int t = (int)threadIdx.x, lane = t & 31, warp = t >> 5;
  const int x = 2 * lane;
  // pairs: k = 0, 1 band rows warp, warp + 16 (stage row +2, mid row +1);
  // k = 2 (warps 0, 1): the extended rows y0-1 (mid row 0) / y0+BY (mid row 33)
  const bool ext = warp < 2;
  // stage / ring rows of pair k (band rows: stage r+2, ring r+1)
  auto srow = [&](int k) { return k == 0 ? warp + 2 : k == 1 ? warp + 18 : (warp == 0 ? 1 : BY + 2); };
  auto mrow = [&](int k) { return k == 0 ? warp + 1 : k == 1 ? warp + 17 : (warp == 0 ? 0 : BY + 1); };
  const bool edge = t >= 64 && t < 64 + 2 * MROWS;  // an extended-column cell x = -1 / 64
  const int eside = (t - 64) / MROWS, er = (t - 64) - eside * MROWS, ex = eside ? TX : -1;
  uint32_t seq = 0;
  auto wait_g = [&](uint32_t g) { mbar_wait(&full[g % S], (g / S) & 1u); };
  auto release_g = [&](uint32_t g) { mbar_arrive(&empty[g % S]); };
  auto sv = [&](const double* st, int sr, int xx) -> double {  // staged cell, xx in [-2, 66)
    return xx < 0 ? st[XH + hoff(0, sr) + (xx + 2)] : xx >= TX ? st[XH + hoff(1, sr) + (xx - TX)] : st[sr * TX + xx];
  };
  for (int64_t pp = pb; pp < pe;) {
    int64_t col;
    int p0, p1, zc0, nload;
    run_at(pp, col, p0, p1);
    pp += p1 - p0;
    plan(p0, p1, zc0, nload);
    const int cx = (int)(col % ntx), y0 = (int)(col / ntx) * BY;
    const int base = p0 - 1;  // ring slot of level-s plane z: (z - base) % 3
    // output offsets of the two band pairs (rows warp, warp + 16: one tile row apart by 16)
    const int64_t od0 = Dv.Y(y0 + warp) + Dv.X(cx * TX + x), odd = Dv.Y(y0 + warp + 16) - Dv.Y(y0 + warp);
    const int64_t om0 = Mv.Y(y0 + warp) + Mv.X(cx * TX + x), omd = Mv.Y(y0 + warp + 16) - Mv.Y(y0 + warp);
    // level s of the own band pairs at planes z-2, z-1 (l2, l1): filled by the
    // loaded planes or by the first computed ones
    double2 l1[2], l2[2];
    for (int q = 0; q < nload; ++q) {
      wait_g(seq + q);
      const double* st = stage + (size_t)((seq + q) % S) * STAGE;
      double* m = mid + (size_t)((p0 - 1 + q - base) % 3) * MID;
      for (int i = t; i < MROWS * 66; i += NT) {
        const int r = i / 66, xx = i - r * 66 - 1;
        m[r * MW + xx + 2] = sv(st, r + 1, xx);
      }
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        l2[k] = l1[k];
        l1[k] = *reinterpret_cast<const double2*>(st + srow(k) * TX + x);
      }
      release_g(seq + q);
    }
    const uint32_t s0 = seq + nload;  // stage of level s-1 plane zc0-1
    // level s-1 of the own band pairs at planes z-1, z (register march; the
    // extended rows of warps 0/1 read theirs from the stages)
    double2 cm[2], cc[2];
    wait_g(s0);
    wait_g(s0 + 1);
    {
      const double* a0 = stage + (size_t)(s0 % S) * STAGE;
      const double* a1 = stage + (size_t)((s0 + 1) % S) * STAGE;
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        cm[k] = *reinterpret_cast<const double2*>(a0 + srow(k) * TX + x);
        cc[k] = *reinterpret_cast<const double2*>(a1 + srow(k) * TX + x);
      }
    }
    for (int z = zc0; z <= p1; ++z) {
      const uint32_t gz = s0 + (uint32_t)(z - (zc0 - 1));  // stage of level s-1 plane z
      wait_g(gz + 1);
      const double* s00 = stage + (size_t)(gz % S) * STAGE;
      const double* sp1 = stage + (size_t)((gz + 1) % S) * STAGE;
      double* m = mid + (size_t)((z - base) % 3) * MID;
      const bool top = z >= b - 2;
      double* mo = top ? Mv.P(z) : nullptr;
      double2 lv[2];
      // level s at z, own pairs
      const double* sm1 = stage + (size_t)((gz - 1) % S) * STAGE;
#pragma unroll
      for (int k = 0; k < 3; ++k) {
        if (k == 2 && !ext) break;
        const int sr = srow(k);
        const double2 c = k < 2 ? cc[k] : *reinterpret_cast<const double2*>(s00 + sr * TX + x);
        const double2 zmv = k < 2 ? cm[k] : *reinterpret_cast<const double2*>(sm1 + sr * TX + x);
        const double2 zp = *reinterpret_cast<const double2*>(sp1 + sr * TX + x);
        const double2 ym = *reinterpret_cast<const double2*>(s00 + (sr - 1) * TX + x);
        const double2 yp = *reinterpret_cast<const double2*>(s00 + (sr + 1) * TX + x);
        double xm = __shfl_up_sync(0xffffffffu, c.y, 1);
        double xp = __shfl_down_sync(0xffffffffu, c.x, 1);
        if (lane == 0) xm = s00[XH + hoff(0, sr) + 1];
        if (lane == 31) xp = s00[XH + hoff(1, sr)];
        double2 v;
        v.x = heat_update(c.x, xm, c.y, ym.x, yp.x, zmv.x, zp.x, alpha);
        v.y = heat_update(c.y, c.x, xp, ym.y, yp.y, zmv.y, zp.y, alpha);
        *reinterpret_cast<double2*>(m + mrow(k) * MW + x + 2) = v;
        if (k < 2) {
          lv[k] = v;
          if (top) *reinterpret_cast<double2*>(mo + om0 + k * omd) = v;
          cm[k] = c;
          cc[k] = zp;
        }
      }
      if (edge) {  // the extended columns x = -1 / 64 (stage z-1 still held: released below)
        const int sr = er + 1;
        const double c = sv(s00, sr, ex);
        m[er * MW + ex + 2] = heat_update(c, sv(s00, sr, ex - 1), sv(s00, sr, ex + 1), sv(s00, sr - 1, ex),
                                          sv(s00, sr + 1, ex), sv(sm1, sr, ex), sv(sp1, sr, ex), alpha);
      }
      release_g(gz - 1);  // level s-1 plane z-1: no reader left
      bar_consumers512();  // level s plane z-1 (written last step) complete in the ring
      const int w = z - 1;
      if (w >= p0) {  // level s+1 at w: z-march in registers, y / x neighbours of plane w from the ring
        const double* mw = mid + (size_t)((w - base) % 3) * MID;
        double* dw = Dv.P(w);
#pragma unroll
        for (int k = 0; k < 2; ++k) {
          const double* p = mw + mrow(k) * MW + x + 2;
          const double2 c = l1[k];
          const double2 ym = *reinterpret_cast<const double2*>(p - MW);
          const double2 yp = *reinterpret_cast<const double2*>(p + MW);
          double xm = __shfl_up_sync(0xffffffffu, c.y, 1);
          double xp = __shfl_down_sync(0xffffffffu, c.x, 1);
          if (lane == 0) xm = p[-1];
          if (lane == 31) xp = p[2];
          double2 v;
          v.x = heat_update(c.x, xm, c.y, ym.x, yp.x, l2[k].x, lv[k].x, alpha);
          v.y = heat_update(c.y, c.x, xp, ym.y, yp.y, l2[k].y, lv[k].y, alpha);
          stg2_stream(dw + od0 + k * odd, v);
        }
      }
#pragma unroll
      for (int k = 0; k < 2; ++k) {
        l2[k] = l1[k];
        l1[k] = lv[k];
      }
    }
    // the last two staged planes (p1, p1+1 of level s-1)
    const uint32_t glast = s0 + (uint32_t)(p1 + 1 - (zc0 - 1));
    release_g(glast - 1);
    release_g(glast);
    seq = glast + 1;
    bar_consumers512();  // the ring is reused by the next run
  }
}

cudaError_t launch_slab_sweep2(const SlabView& src, const SlabView& mid, const SlabView& dst, int nx, int ny, int a,
                               int b, double alpha, int sms, cudaStream_t s, const SweepMaps* maps) {
  using namespace w2;
  if (b <= a) return cudaSuccess;
  if (b - a < 2 || !maps || !maps->valid[0] || maps->band != BY || src.ring || mid.ring || src.hhi || mid.hhi ||
      src.tx != TX || mid.tx != TX || dst.tx != TX || src.ty % 64 || mid.ty % 64 || dst.ty % BY || nx % TX ||
      ny % 64 || nx / TX < 2)
    return cudaErrorNotSupported;
  for (const SlabView* v : {&src, &mid})
    if (v->hlo && !(maps->valid[1] && v->hlo >= maps->base[1] && v->hlo < maps->end[1]))
      return cudaErrorNotSupported;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(slab_sweep2_tile, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  const int64_t P = (int64_t)(nx / TX) * (ny / BY) * (b - a);
  const int64_t grid = std::max<int64_t>(1, std::min<int64_t>((int64_t)sms, P / 8));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)grid);
  cfg.blockDim = dim3(NT + 32);
  cfg.dynamicSmemBytes = SMEM;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, slab_sweep2_tile, to_dev(src), to_dev(mid), to_dev(dst), *maps, ny, a, b, alpha);
}

int sweep_tile_band() { return 32; }

bool sweep_map_encode(SweepMaps* m, int k, const double* base, uint64_t bytes, int tx, int band) {
  static_assert(sizeof(CUtensorMap) == sizeof(TensorMapBlob), "CUtensorMap size");
  m->valid[k] = 0;
  EncodeTiledFn f = encode_fn();
  if (!f || !base || (reinterpret_cast<uintptr_t>(base) & 15) || tx != 64) return false;
  const uint64_t rows = bytes / ((uint64_t)tx * 8);
  if (rows < 1 || rows > (1ull << 31)) return false;
  const cuuint64_t dims[2] = {(cuuint64_t)tx, (cuuint64_t)rows};
  const cuuint64_t strides[1] = {(cuuint64_t)tx * 8};
  const cuuint32_t box[2] = {2, (cuuint32_t)band};
  const cuuint32_t estr[2] = {1, 1};
  CUtensorMap* tm = reinterpret_cast<CUtensorMap*>(&m->xmap[k]);
  if (f(tm, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, const_cast<double*>(base), dims, strides, box, estr,
        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
        CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
    return false;
  const cuuint32_t box2[2] = {2, 2};
  if (f(reinterpret_cast<CUtensorMap*>(&m->xmap2[k]), CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 2, const_cast<double*>(base),
        dims, strides, box2, estr, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
        CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) != CUDA_SUCCESS)
    return false;
  m->base[k] = base;
  m->end[k] = base + rows * tx;
  m->valid[k] = 1;
  m->band = band;
  return true;
}


static int sweep_occupancy(int BY) {
  static int occ[3] = {0, 0, 0};
  const int k = BY == 4 ? 2 : BY == 2 ? 1 : 0;
  if (!occ[k]) {
    int o = 1;
    if (BY == 4) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, slab_sweep_zm<4>, 128, 0);
    else if (BY == 2) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, slab_sweep_zm<2>, 128, 0);
    else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&o, slab_sweep_zm<1>, 128, 0);
    occ[k] = o < 1 ? 1 : o;
  }
  return occ[k];
}

cudaError_t launch_slab_sweep(const SlabView& src, const SlabView& dst, int nx, int ny, int lo,
                              int hi, double alpha, int sms, cudaStream_t s, const SweepMaps* maps) {
  if (hi <= lo) return cudaSuccess;
  // TILES_SWEEP_TMA=0: the cp.async kernel everywhere (A/B runs)
  static const int use_tma = [] {
    const char* e = getenv("TILES_SWEEP_TMA");
    return e ? atoi(e) : 1;
  }();
  // tile columns with tensor-map x halos, for 64-wide tiled views whose
  // memory the maps cover (every plane of the source)
  const int tb = sweep_tile_band();
  if (use_tma && maps && maps->valid[0] && maps->band == tb && !src.ring && src.tx == 64 && dst.tx == 64 &&
      src.ty % tb == 0 && dst.ty % tb == 0 && nx % 64 == 0 && ny % tb == 0 && !src.hhi &&
      (!src.hlo || (maps->valid[1] && src.hlo >= maps->base[1] && src.hlo < maps->end[1])))
    // band 32, 4 rows per consumer thread, 5 stages, 2 CTAs per SM (band 16 or 64, 3 CTAs per SM
    // measured slower: profiles/r02/bench_sweep_cfg*.json; 4 / 5 / 6 stages at 2 CTAs per SM:
    // 0.757 / 0.768 / 0.765 of HBM on the C2 e2e step, three alternating runs)
  {
    // consumers: 128 threads, each one x pair of 8 consecutive rows (y
    // neighbours of the inner rows from its registers, x neighbours by warp
    // shuffle): 0.839 of HBM per launch against 0.791-0.795 for 256 threads
    // of 4 rows 8 apart with shared-memory neighbours (TILES_SWEEP_CS=0),
    // three alternating rounds
    static const int cs = [] {
      const char* e = getenv("TILES_SWEEP_CS");
      return e ? atoi(e) : 1;
    }();
    if (cs) return launch_tile_cfg<32, 4, 5, 2, true, true>(to_dev(src), to_dev(dst), *maps, nx, ny, lo, hi, alpha, sms, s);
    return launch_tile_cfg<32, 8, 5, 2>(to_dev(src), to_dev(dst), *maps, nx, ny, lo, hi, alpha, sms, s);
  }
  const int npairs = nx / 2;
  const int gx = (npairs + 127) / 128;
  // rows per thread: must divide every view's ty (the dense slab's is ny,
  // the tiled views' the tile's)
  const int tyg = std::gcd(src.ty, dst.ty);
  static const int by_max = [] {
    const char* e = getenv("TILES_SWEEP_BY");
    return e ? atoi(e) : 4;
  }();
  const int BY = tyg % 4 == 0 && by_max >= 4 ? 4 : tyg % 2 == 0 && by_max >= 2 ? 2 : 1;
  const int64_t cols = (int64_t)gx * (ny / BY);
  const int planes = hi - lo;
  const int64_t G = (int64_t)sms * sweep_occupancy(BY);
  // z chunk: >= 8 planes (a chunk re-reads 2 boundary planes), as many
  // chunks as balance the resident grid best (items / G rounded up)
  int zc = planes, best_nch = 1;
  double best = 1e30;
  for (int nch = 1; nch <= std::max(1, planes / 8); ++nch) {
    const int64_t items = cols * nch;
    const int64_t rounds = (items + G - 1) / G;
    const int c = (planes + nch - 1) / nch;
    const double cost = (double)rounds * (c + 2);  // per-block planes incl. prologue
    if (cost < best) best = cost, best_nch = nch;
  }
  zc = (planes + best_nch - 1) / best_nch;
  const int64_t grid = std::min<int64_t>(G, cols * ((planes + zc - 1) / zc));
  const ViewDev S = to_dev(src), D = to_dev(dst);
  static const int use_ca = [] {
    const char* e = getenv("TILES_SWEEP_CA");
    return e ? atoi(e) : 1;
  }();
  if (use_ca && BY == 4) {  // 4 stages: 4 blocks per SM (5 or 6 stages fit 3: slower, 4.0-4.1 TB/s)
    constexpr size_t sm = CaLayout<4, 4>::SMEM;
    static bool attr = false;
    if (!attr) {
      cudaError_t e = cudaFuncSetAttribute(slab_sweep_ca<4, 4>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
      if (e != cudaSuccess) return e;
      attr = true;
    }
    slab_sweep_ca<4, 4><<<(unsigned)grid, 128, sm, s>>>(S, D, nx, ny, lo, hi, gx, zc, alpha);
    return cudaGetLastError();
  }
  switch (BY) {
    case 4: slab_sweep_zm<4><<<(unsigned)grid, 128, 0, s>>>(S, D, nx, ny, lo, hi, gx, zc, alpha); break;
    case 2: slab_sweep_zm<2><<<(unsigned)grid, 128, 0, s>>>(S, D, nx, ny, lo, hi, gx, zc, alpha); break;
    default: slab_sweep_zm<1><<<(unsigned)grid, 128, 0, s>>>(S, D, nx, ny, lo, hi, gx, zc, alpha); break;
  }
  return cudaGetLastError();
}

}  // namespace tiles
