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
                              int hi, double alpha, int sms, cudaStream_t s) {
  if (hi <= lo) return cudaSuccess;
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
