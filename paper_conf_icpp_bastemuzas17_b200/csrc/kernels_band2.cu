// kernels_band2.cu — two Jacobi steps per pass over a resident periodic grid
// 512 cells wide (heat2_band). Each step is the update of
// P:L35–L37 (reading R1, heat_update), so one pass gives exactly two single
// steps; the point is the traffic: u^s is read and u^{s+2} written once per
// pass, 16 B per cell for two steps instead of 32 B.
//
// A CTA owns one band of BY = 4 rows across the full width (8 tile columns of
// 64, so x is periodic inside the CTA and no column outside it is ever needed)
// and marches z over the whole periodic ring. Per plane thread 0 stages u^s
// rows y0-2 .. y0+5 with three 5-D TMA boxes (2 / 4 / 2 rows x 64 x 8 tile
// columns; the resident array seen as x, y, tile column, z, tile
// row-and-layer). Consumer warp w owns tile column w, lane l the column pair
// x = 2l: u^{s+1} on rows y0-1 .. y0+4 at plane z and u^{s+2} on rows
// y0 .. y0+3 at plane z-1, both marching z in registers (u^s at z-1, z, z+1;
// u^{s+1} at z-2, z-1, z), y neighbours from the thread's own registers, x
// neighbours by shuffle; only the warps' edge columns cross warps — u^s's
// from the stage, u^{s+1}'s through a three-slot edge ring with one named
// barrier per plane. Grid = ny / 4 CTAs, one per SM, all marching z together,
// so a band's y-halo rows were just read by its neighbour band (L2 hits).
#include <cuda.h>

#include <type_traits>

#include "kernels.cuh"
#include "ptx.cuh"

namespace tiles {

namespace b2 {
constexpr int NW = 8, TX = 64, NT = NW * 32, BY = 4, S = 6;
constexpr int OFF_A = 0, OFF_B = NW * 2 * TX, OFF_C = OFF_B + NW * 4 * TX;  // rows y0-2.. | y0.. | y0+4..
constexpr int STAGE = NW * 8 * TX;                                             // doubles
constexpr uint32_t BYTES = (uint32_t)STAGE * 8;
constexpr int ER = 6;                   // u^{s+1} rows y0-1 .. y0+4
constexpr int ESLOT = NW * 2 * ER;      // [tile column][side][row]
constexpr size_t SMEM = (size_t)S * STAGE * 8 + (size_t)3 * ESLOT * 8 + (size_t)S * 8;
// staged row i (y0-2+i) of tile column w, relative to a stage
__device__ __forceinline__ int srow(int i, int w) {
  return i < 2 ? OFF_A + (w * 2 + i) * TX : i < 6 ? OFF_B + (w * 4 + i - 2) * TX : OFF_C + (w * 2 + i - 6) * TX;
}
}  // namespace b2

static __device__ __forceinline__ void tma_5d(void* dst, const TensorMapBlob* map, int c0, int c1, int c2, int c3,
                                              int c4, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.5d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], "
      "[%7];" ::"r"(smem_u32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(c4), "r"(smem_u32(bar))
      : "memory");
}

// v = [addr] in the lanes where pred != 0, unchanged elsewhere (a predicated
// shared load: no branch, no select)
static __device__ __forceinline__ void lds_if(double& v, uint32_t addr, uint32_t pred) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p ld.shared.f64 %0, [%1];\n}" : "+d"(v)
               : "r"(addr), "r"(pred));
}
static __device__ __forceinline__ void sts_if(uint32_t addr, double v, uint32_t pred) {
  asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p st.shared.f64 [%0], %1;\n}" ::"r"(addr), "d"(v),
               "r"(pred)
               : "memory");
}

static __device__ __forceinline__ void bar_consumers_b2() { asm volatile("bar.sync 1, 256;" ::: "memory"); }


__global__ void __launch_bounds__(b2::NT, 1)
    heat2_band(const __grid_constant__ Band2Maps maps, double* __restrict__ dst, const int ty, const int tz,
               const int nty, const int nz, const int64_t te, const double alpha) {
  using namespace b2;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double* stage = reinterpret_cast<double*>(smem_raw);
  double* edge = stage + (size_t)S * STAGE;
  uint64_t* full = reinterpret_cast<uint64_t*>(edge + 3 * ESLOT);
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) mbar_init(&full[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const int ny = nty * ty;
  const int y0 = (int)blockIdx.x * BY;
  const int nq = nz + 4;  // u^s planes -2 .. nz+1
  // the producer is thread 0 (eight warps in all: two per scheduler leave
  // 255 registers per thread, a ninth producer warp would cap them at 168)
  const int ya = (y0 - 2 + ny) % ny, yc = (y0 + 4) % ny;
  const int ta = ya / ty, la = ya % ty, tb = y0 / ty, lb = y0 % ty, tc = yc / ty, lc = yc % ty;
  // thread 0 stages u^s plane q - 2 (wrapped) into slot q % S. A slot is
  // refilled only after the block barrier that follows every thread's last
  // read of it, so no empty-slot mbarrier is needed (the barrier orders those
  // reads before this thread's async-proxy writes, fence.proxy.async below)
  int qz = ((-2 % nz) + nz) % nz, qzl = qz % tz, qzt = qz / tz, qs = 0;  // next plane (z, in-tile z, layer), slot
  auto issue = [&]() {
    double* d = stage + (size_t)qs * STAGE;
    fence_proxy_async();
    mbar_expect_tx(&full[qs], BYTES);
    tma_5d(d + OFF_A, &maps.m2, 0, la, 0, qzl, qzt * nty + ta, &full[qs]);
    tma_5d(d + OFF_B, &maps.m4, 0, lb, 0, qzl, qzt * nty + tb, &full[qs]);
    tma_5d(d + OFF_C, &maps.m2, 0, lc, 0, qzl, qzt * nty + tc, &full[qs]);
    if (++qz == nz) qz = 0, qzl = 0, qzt = 0;
    else if (++qzl == tz) qzl = 0, ++qzt;
    qs = qs + 1 == S ? 0 : qs + 1;
  };
  int issued = 0;  // thread 0: planes staged so far
  if (threadIdx.x == 0) {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    for (; issued < S && issued < nq; ++issued) issue();
  }

  // ------------------------------------------------------- consumer warps
  const int t = (int)threadIdx.x, lane = t & 31, w = t >> 5;
  const int x = 2 * lane;
  // this lane's x-edge source: lane 0 the left tile column's x = 63, lane 31
  // the right one's x = 0 (the other lanes load lane 0's: a broadcast)
  const bool right = lane == 31;
  const int we = right ? (w + 1) % NW : (w + NW - 1) % NW, xe = right ? 0 : TX - 1;
  // u^{s+1} edge ring: [slot][tile column][side 0: x = 0, 1: x = 63][row]
  const int e_mine = right ? (w * 2 + 1) * ER : w * 2 * ER;           // written by lanes 0 / 31
  const int e_nbr = right ? ((w + 1) % NW) * 2 * ER : (((w + NW - 1) % NW) * 2 + 1) * ER;
  const uint32_t is_left = lane == 0, is_right = right;
  const int yl0 = y0 % ty;
  const int64_t obase = (int64_t)((y0 / ty) * NW + w) * te + (int64_t)yl0 * TX + x;  // + layer, plane
  const int64_t oplane = (int64_t)ty * TX;

  auto wait_q = [&](int q) { mbar_wait(&full[q % S], (q / S) & 1); };
  auto ld2 = [&](const double* s, int i) { return *reinterpret_cast<const double2*>(s + srow(i, w) + x); };

  // register rings, period 3 (the loop below is unrolled by three, so no
  // value moves between registers): u^s planes z-1, z, z+1 in a[(k)..(k+2)
  // % 3], u^{s+1} planes z-2, z-1, z in b[(k)..(k+2) % 3] at phase k
  double2 a[3][8], b[3][6];
  wait_q(0);
#pragma unroll
  for (int i = 0; i < 8; ++i) a[0][i] = ld2(stage, i);
  wait_q(1);
#pragma unroll
  for (int i = 0; i < 8; ++i) a[1][i] = ld2(stage + (size_t)STAGE, i);
#pragma unroll
  for (int k = 0; k < 3; ++k)
#pragma unroll
    for (int j = 0; j < 6; ++j) b[k][j] = make_double2(0.0, 0.0);
  int pl = 0, pt = 0;           // level-2 output plane (z - 1): in-tile plane and tile layer
  int sq = 2 % S, sq1 = 1;      // slots of u^s planes z + 1 and z
  int e0 = 0, e1 = 2;           // edge-ring slots of it and it - 1
  auto step = [&](int it, auto kc) {
    constexpr int K = decltype(kc)::value;
    constexpr int P0 = K, P1 = (K + 1) % 3, P2 = (K + 2) % 3;  // z-1, z, z+1 | z-2, z-1, z
    const int q = it + 2;  // u^s plane z + 1
    wait_q(q);
    const double* sz = stage + (size_t)sq1 * STAGE;
    const double* sp = stage + (size_t)sq * STAGE;
#pragma unroll
    for (int i = 0; i < 8; ++i) a[P2][i] = ld2(sp, i);
#pragma unroll
    for (int r = 0; r < 6; ++r) {  // u^{s+1} at z, row y0-1+r
      const double2 c = a[P1][r + 1];
      double xm = __shfl_up_sync(0xffffffffu, c.y, 1);
      double xp = __shfl_down_sync(0xffffffffu, c.x, 1);
      const uint32_t ea = smem_u32(sz + srow(r + 1, we) + xe);
      lds_if(xm, ea, is_left);
      lds_if(xp, ea, is_right);
      b[P2][r].x = heat_update(c.x, xm, c.y, a[P1][r].x, a[P1][r + 2].x, a[P0][r + 1].x, a[P2][r + 1].x, alpha);
      b[P2][r].y = heat_update(c.y, c.x, xp, a[P1][r].y, a[P1][r + 2].y, a[P0][r + 1].y, a[P2][r + 1].y, alpha);
    }
    // u^{s+2} at p = z - 1, rows y0 .. y0+3: own registers and the edges of
    // plane z - 1 (complete since the last barrier), so no barrier between the
    // two levels and the compiler interleaves them
    if (it >= 2) {
      const double* em = edge + (size_t)e1 * ESLOT + e_nbr;
      double* o = dst + obase + (int64_t)((pt * nty) * NW) * te + (int64_t)pl * oplane;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const double2 c = b[P1][j + 1];
        double xm = __shfl_up_sync(0xffffffffu, c.y, 1);
        double xp = __shfl_down_sync(0xffffffffu, c.x, 1);
        lds_if(xm, smem_u32(em + j + 1), is_left);
        lds_if(xp, smem_u32(em + j + 1), is_right);
        double2 v;
        v.x = heat_update(c.x, xm, c.y, b[P1][j].x, b[P1][j + 2].x, b[P0][j + 1].x, b[P2][j + 1].x, alpha);
        v.y = heat_update(c.y, c.x, xp, b[P1][j].y, b[P1][j + 2].y, b[P0][j + 1].y, b[P2][j + 1].y, alpha);
        stg2_stream(o + j * TX, v);
      }
      if (++pl == tz) pl = 0, ++pt;
    }
    {
      const uint32_t ez = smem_u32(edge + (size_t)e0 * ESLOT + e_mine);
#pragma unroll
      for (int r = 0; r < 6; ++r) {
        sts_if(ez + 8 * r, b[P2][r].x, is_left);
        sts_if(ez + 8 * r, b[P2][r].y, is_right);
      }
    }
    bar_consumers_b2();  // u^{s+1} edges of plane z complete (read at it + 1)
    // every thread has released the slots of planes <= z: refill them
    if (t == 0)
      for (; issued < nq && issued <= q - 1 + S; ++issued) issue();
    sq1 = sq;
    sq = sq + 1 == S ? 0 : sq + 1;
    e1 = e0;
    e0 = e0 == 2 ? 0 : e0 + 1;
  };
  const int nit = nz + 2;  // u^{s+1} at z = it - 1 for it in [0, nit)
  for (int it = 0; it < nit; it += 3) {
    step(it, std::integral_constant<int, 0>{});
    if (it + 1 >= nit) break;
    step(it + 1, std::integral_constant<int, 1>{});
    if (it + 2 >= nit) break;
    step(it + 2, std::integral_constant<int, 2>{});
  }
}

// ---- two-level passes over general views on the same band layout
// (heat2_band_slab). MID (the wavefront, slab_sweep2 semantics): level s on
// planes [a, b) from view src (level s-1), only its top two planes b-2, b-1
// written to view mid, whose planes a-2, a-1 it reads; level s+1 on
// [a-1, b-1) into view dst. Staged planes, in order: mid a-2, mid a-1 (rows
// y0-1 .. y0+4 go straight to the level-s registers), then src a-1 .. b.
// SHRINK (two sweeps of the stream-through): level s on [a, b) from src,
// kept on chip; level s+1 on [a+1, b-1) into dst; staged src a-1 .. b.
static __device__ __forceinline__ void b2_coords(const Band2View& v, int z, const TensorMapBlob*& m4,
                                                 const TensorMapBlob*& m2, int& zl, int& zt) {
  z += v.zbase;
  if (z < 0 && v.nlo > 0) {
    const int q = z + v.nlo * v.tz;
    m4 = &v.scr.m4, m2 = &v.scr.m2, zl = q % v.tz, zt = q / v.tz;
  } else {
    if (v.wrap) z = ((z % v.nz) + v.nz) % v.nz;
    m4 = &v.main.m4, m2 = &v.main.m2, zl = z % v.tz, zt = z / v.tz;
  }
}
// first element of view plane z in tile (tile row ty_i, tile column w)
static __device__ __forceinline__ double* b2_plane(const Band2Out& o, int z, int nty, int tyi, int w, int ty) {
  z += o.zbase;
  double* base = o.base;
  if (z < 0) base = o.hlo, z += o.nlo * o.tz;
  return base + ((int64_t)(z / o.tz) * nty * b2::NW + (int64_t)tyi * b2::NW + w) * o.te +
         (int64_t)(z % o.tz) * ty * b2::TX;
}

template <bool MID>
__global__ void __launch_bounds__(b2::NT, 1)
    heat2_band_slab(const __grid_constant__ Band2View src, const __grid_constant__ Band2View mid, const Band2Out mido,
                    const Band2Out dsto, const int ty, const int nty, const int a, const int b, const double alpha) {
  using namespace b2;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double* stage = reinterpret_cast<double*>(smem_raw);
  double* edge = stage + (size_t)S * STAGE;
  uint64_t* full = reinterpret_cast<uint64_t*>(edge + 3 * ESLOT);
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) mbar_init(&full[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const int ny = nty * ty;
  const int y0 = (int)blockIdx.x * BY;
  constexpr int NM = MID ? 2 : 0;  // staged mid planes
  const int nq = NM + b - a + 2;   // staged planes: [mid a-2, a-1,] src a-1 .. b
  const int ya = (y0 - 2 + ny) % ny, yc = (y0 + 4) % ny;
  const int ta = ya / ty, la = ya % ty, tb = y0 / ty, lb = y0 % ty, tc = yc / ty, lc = yc % ty;
  int qn = 0, qs = 0;  // thread 0: next staged index, its slot
  auto issue = [&]() {
    const bool m = qn < NM;
    const int z = m ? a - 2 + qn : a - 1 + (qn - NM);
    const TensorMapBlob *m4, *m2;
    int zl, zt;
    b2_coords(m ? mid : src, z, m4, m2, zl, zt);
    double* d = stage + (size_t)qs * STAGE;
    fence_proxy_async();
    mbar_expect_tx(&full[qs], BYTES);
    tma_5d(d + OFF_A, m2, 0, la, 0, zl, zt * nty + ta, &full[qs]);
    tma_5d(d + OFF_B, m4, 0, lb, 0, zl, zt * nty + tb, &full[qs]);
    tma_5d(d + OFF_C, m2, 0, lc, 0, zl, zt * nty + tc, &full[qs]);
    ++qn;
    qs = qs + 1 == S ? 0 : qs + 1;
  };
  if (threadIdx.x == 0) {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    while (qn < S && qn < nq) issue();
  }

  const int t = (int)threadIdx.x, lane = t & 31, w = t >> 5;
  const int x = 2 * lane;
  const bool right = lane == 31;
  const int we = right ? (w + 1) % NW : (w + NW - 1) % NW, xe = right ? 0 : TX - 1;
  const int e_mine = right ? (w * 2 + 1) * ER : w * 2 * ER;
  const int e_nbr = right ? ((w + 1) % NW) * 2 * ER : (((w + NW - 1) % NW) * 2 + 1) * ER;
  const uint32_t is_left = lane == 0, is_right = right;
  const int oyx = lb * TX + x;  // this lane's first output cell in a tile plane
  auto wait_q = [&](int q) { mbar_wait(&full[q % S], (q / S) & 1); };
  auto ld2 = [&](const double* st, int i) { return *reinterpret_cast<const double2*>(st + srow(i, w) + x); };

  double2 a_[3][8], b_[3][6];
  if (MID) {
    wait_q(0);
#pragma unroll
    for (int r = 0; r < 6; ++r) b_[0][r] = ld2(stage, r + 1);   // level s, plane a-2
    wait_q(1);
#pragma unroll
    for (int r = 0; r < 6; ++r) b_[1][r] = ld2(stage + (size_t)STAGE, r + 1);  // level s, plane a-1
    const uint32_t ez = smem_u32(edge + (size_t)2 * ESLOT + e_mine);  // its edges: slot of it - 1 at it = 0
#pragma unroll
    for (int r = 0; r < 6; ++r) {
      sts_if(ez + 8 * r, b_[1][r].x, is_left);
      sts_if(ez + 8 * r, b_[1][r].y, is_right);
    }
  } else {
#pragma unroll
    for (int k = 0; k < 2; ++k)
#pragma unroll
      for (int r = 0; r < 6; ++r) b_[k][r] = make_double2(0.0, 0.0);
  }
  wait_q(NM);
#pragma unroll
  for (int i = 0; i < 8; ++i) a_[0][i] = ld2(stage + (size_t)(NM % S) * STAGE, i);  // src a-1
  wait_q(NM + 1);
#pragma unroll
  for (int i = 0; i < 8; ++i) a_[1][i] = ld2(stage + (size_t)((NM + 1) % S) * STAGE, i);  // src a
  bar_consumers_b2();  // (MID: plane a-1's edges written); staged 0 .. NM consumed
  if (t == 0)
    while (qn < nq && qn <= NM + S) issue();
  int sq = (NM + 2) % S, sq1 = (NM + 1) % S;  // slots of staged src p+1 and src p
  int e0 = 0, e1 = 2;
  auto step = [&](int it, auto kc) {
    constexpr int K = decltype(kc)::value;
    constexpr int P0 = K, P1 = (K + 1) % 3, P2 = (K + 2) % 3;
    const int p = a + it, q = it + NM + 2;
    wait_q(q);
    const double* sz = stage + (size_t)sq1 * STAGE;
    const double* sp = stage + (size_t)sq * STAGE;
#pragma unroll
    for (int i = 0; i < 8; ++i) a_[P2][i] = ld2(sp, i);
#pragma unroll
    for (int r = 0; r < 6; ++r) {  // level s at p, row y0-1+r
      const double2 c = a_[P1][r + 1];
      double xm = __shfl_up_sync(0xffffffffu, c.y, 1);
      double xp = __shfl_down_sync(0xffffffffu, c.x, 1);
      const uint32_t ea = smem_u32(sz + srow(r + 1, we) + xe);
      lds_if(xm, ea, is_left);
      lds_if(xp, ea, is_right);
      b_[P2][r].x = heat_update(c.x, xm, c.y, a_[P1][r].x, a_[P1][r + 2].x, a_[P0][r + 1].x, a_[P2][r + 1].x, alpha);
      b_[P2][r].y = heat_update(c.y, c.x, xp, a_[P1][r].y, a_[P1][r + 2].y, a_[P0][r + 1].y, a_[P2][r + 1].y, alpha);
    }
    if (MID || it >= 2) {  // level s+1 at p - 1, rows y0 .. y0+3
      const double* em = edge + (size_t)e1 * ESLOT + e_nbr;
      double* o = b2_plane(dsto, p - 1, nty, tb, w, ty) + oyx;
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        const double2 c = b_[P1][j + 1];
        double xm = __shfl_up_sync(0xffffffffu, c.y, 1);
        double xp = __shfl_down_sync(0xffffffffu, c.x, 1);
        lds_if(xm, smem_u32(em + j + 1), is_left);
        lds_if(xp, smem_u32(em + j + 1), is_right);
        double2 v;
        v.x = heat_update(c.x, xm, c.y, b_[P1][j].x, b_[P1][j + 2].x, b_[P0][j + 1].x, b_[P2][j + 1].x, alpha);
        v.y = heat_update(c.y, c.x, xp, b_[P1][j].y, b_[P1][j + 2].y, b_[P0][j + 1].y, b_[P2][j + 1].y, alpha);
        *reinterpret_cast<double2*>(o + j * TX) = v;
      }
    }
    if (MID && p >= b - 2) {  // level s's top two planes, this band's rows, to mid
      double* o = b2_plane(mido, p, nty, tb, w, ty) + oyx;
#pragma unroll
      for (int j = 0; j < 4; ++j) *reinterpret_cast<double2*>(o + j * TX) = b_[P2][j + 1];
    }
    {
      const uint32_t ez = smem_u32(edge + (size_t)e0 * ESLOT + e_mine);
#pragma unroll
      for (int r = 0; r < 6; ++r) {
        sts_if(ez + 8 * r, b_[P2][r].x, is_left);
        sts_if(ez + 8 * r, b_[P2][r].y, is_right);
      }
    }
    bar_consumers_b2();
    if (t == 0)
      while (qn < nq && qn <= q - 1 + S) issue();
    sq1 = sq;
    sq = sq + 1 == S ? 0 : sq + 1;
    e1 = e0;
    e0 = e0 == 2 ? 0 : e0 + 1;
  };
  const int nit = b - a;
  for (int it = 0; it < nit; it += 3) {
    step(it, std::integral_constant<int, 0>{});
    if (it + 1 >= nit) break;
    step(it + 1, std::integral_constant<int, 1>{});
    if (it + 2 >= nit) break;
    step(it + 2, std::integral_constant<int, 2>{});
  }
}

cudaError_t launch_heat2_band_slab(int mid_mode, const Band2View& src, const Band2View& mid, const Band2Out& mido,
                                   const Band2Out& dsto, int ty, int nty, int a, int b, double alpha,
                                   cudaStream_t s) {
  using namespace b2;
  if (b - a < (mid_mode ? 2 : 3)) return cudaErrorNotSupported;
  auto kern = mid_mode ? heat2_band_slab<true> : heat2_band_slab<false>;
  static bool attr[2] = {false, false};
  if (!attr[mid_mode ? 1 : 0]) {
    cudaError_t e = cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM);
    if (e != cudaSuccess) return e;
    attr[mid_mode ? 1 : 0] = true;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(nty * ty / BY));
  cfg.blockDim = dim3(NT);
  cfg.dynamicSmemBytes = SMEM;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, src, mid, mido, dsto, ty, nty, a, b, alpha);
}

// ---- all two-level passes of one wavefront iteration in one launch
// (heat2_band_iter). Pass k (levels s, s+1 with s = s0 + 2k) has the
// heat2_band_slab<MID> semantics over the level views lvl(s-1), lvl(s),
// lvl(s+1). A band runs its passes back to back; between passes it needs
// nothing but its two neighbour bands' progress: the source planes of pass k
// that pass k-1 wrote (rows y0-2 .. y0+5 come from bands b-1, b, b+1) are
// staged only once both neighbours have published that pass k-1 iteration
// (per-band 64-bit flags: epoch << 32 | pass << 16 | iterations done,
// published by thread 0 after the block barrier with a GPU-scope fence, read
// with ld.acquire and followed by a proxy fence before the TMA). Every
// other hazard between consecutive passes is ordered by that wait (DESIGN.md
// §4). The producer's staging runs across pass boundaries, so a pass starts
// with its first planes already on chip. All CTAs must be co-resident (one
// band per SM, grid = ny/4 <= SMs); no programmatic early launch of the next
// kernel (it could take the SMs of CTAs this one waits on).
constexpr int kIterPub = 8;  // progress published every 8 planes (and at each pass's end)
static __device__ __forceinline__ void st_relaxed_gpu_u64(unsigned long long* p, unsigned long long v) {
  asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__global__ void __launch_bounds__(b2::NT, 1) heat2_band_iter(const __grid_constant__ Band2Iter it_) {
  using namespace b2;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  double* stage = reinterpret_cast<double*>(smem_raw);
  double* edge = stage + (size_t)S * STAGE;
  uint64_t* full = reinterpret_cast<uint64_t*>(edge + 3 * ESLOT);
  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) mbar_init(&full[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const int ty = it_.ty, nty = it_.nty, ny = nty * ty;
  const int band = (int)blockIdx.x, nb = (int)gridDim.x;
  const int y0 = band * BY;
  const int ya = (y0 - 2 + ny) % ny, yc = (y0 + 4) % ny;
  const int ta = ya / ty, la = ya % ty, tb = y0 / ty, lb = y0 % ty, tc = yc / ty, lc = yc % ty;
  unsigned long long* const fl_me = it_.flags + band;
  const unsigned long long* const fl_lo = it_.flags + (band + nb - 1) % nb;
  const unsigned long long* const fl_hi = it_.flags + (band + 1) % nb;
  const unsigned long long ep = it_.epoch << 32;
  auto src_of = [&](int k) -> const Band2View& {
    const int s = it_.s0 + 2 * k;
    return s - 1 == 0 ? it_.v[3] : it_.v[(s - 1) % 3];
  };
  // thread 0: staging cursor (pass, staged index within the pass, ring slot)
  int ik = 0, iq = 0, qs = 0;
  unsigned long long seen_lo = 0, seen_hi = 0;  // thread 0: neighbour progress last observed
  const int nqp = 2 + it_.c + 2;  // staged planes per pass: mid a-2, a-1, src a-1 .. b
  auto issue = [&]() {
    const int k = ik, s = it_.s0 + 2 * k, a = it_.ci - s;
    const bool m = iq < 2;
    const int z = m ? a - 2 + iq : a - 1 + (iq - 2);
    if (!m && k > 0) {  // a plane pass k-1 wrote: wait for the neighbour bands
      const int a1 = a + 2;       // pass k-1's a
      if (z >= a1 - 1) {
        // the neighbours are usually a pass ahead: the progress last seen
        // answers most checks without a GPU-scope load
        const unsigned long long need = ep | ((unsigned long long)(k - 1) << 16) | (unsigned)(z - a1 + 2);
        if (seen_lo < need || seen_hi < need) {
          long long spin = 0;
          while ((seen_lo = ld_acquire_gpu(fl_lo)) < need || (seen_hi = ld_acquire_gpu(fl_hi)) < need)
            if (++spin > (1ll << 28)) asm volatile("trap;");
          fence_proxy_async_all();
        }
      }
    }
    const TensorMapBlob *m4, *m2;
    int zl, zt;
    b2_coords(m ? it_.v[s % 3] : src_of(k), z, m4, m2, zl, zt);
    double* d = stage + (size_t)qs * STAGE;
    fence_proxy_async();
    mbar_expect_tx(&full[qs], BYTES);
    tma_5d(d + OFF_A, m2, 0, la, 0, zl, zt * nty + ta, &full[qs]);
    tma_5d(d + OFF_B, m4, 0, lb, 0, zl, zt * nty + tb, &full[qs]);
    tma_5d(d + OFF_C, m2, 0, lc, 0, zl, zt * nty + tc, &full[qs]);
    qs = qs + 1 == S ? 0 : qs + 1;
    if (++iq == nqp) iq = 0, ++ik;
  };
  const int ntot = it_.P * nqp;  // staged planes of the launch
  int issued = 0;                // thread 0: global staged index
  if (threadIdx.x == 0) {
    asm volatile("griddepcontrol.wait;" ::: "memory");
    for (; issued < S && issued < ntot; ++issued) issue();
  }

  const int t = (int)threadIdx.x, lane = t & 31, w = t >> 5;
  const int x = 2 * lane;
  const bool right = lane == 31;
  const int we = right ? (w + 1) % NW : (w + NW - 1) % NW, xe = right ? 0 : TX - 1;
  const int e_mine = right ? (w * 2 + 1) * ER : w * 2 * ER;
  const int e_nbr = right ? ((w + 1) % NW) * 2 * ER : (((w + NW - 1) % NW) * 2 + 1) * ER;
  const uint32_t is_left = lane == 0, is_right = right;
  const int oyx = lb * TX + x;
  auto wait_g = [&](int g) { mbar_wait(&full[g % S], (g / S) & 1); };
  auto ld2 = [&](const double* st, int i) { return *reinterpret_cast<const double2*>(st + srow(i, w) + x); };

  double2 a_[3][8], b_[3][6];
  int g0 = 0;  // global staged index of this pass's first plane
  for (int k = 0; k < it_.P; ++k, g0 += nqp) {
    const int s = it_.s0 + 2 * k, a = it_.ci - s, b = a + it_.c;
    const Band2Out& mido = it_.o[s % 3];
    const Band2Out& dsto = it_.o[(s + 1) % 3];
    wait_g(g0);
#pragma unroll
    for (int r = 0; r < 6; ++r) b_[0][r] = ld2(stage + (size_t)(g0 % S) * STAGE, r + 1);
    wait_g(g0 + 1);
#pragma unroll
    for (int r = 0; r < 6; ++r) b_[1][r] = ld2(stage + (size_t)((g0 + 1) % S) * STAGE, r + 1);
    {
      const uint32_t ez = smem_u32(edge + (size_t)2 * ESLOT + e_mine);
#pragma unroll
      for (int r = 0; r < 6; ++r) {
        sts_if(ez + 8 * r, b_[1][r].x, is_left);
        sts_if(ez + 8 * r, b_[1][r].y, is_right);
      }
    }
    wait_g(g0 + 2);
#pragma unroll
    for (int i = 0; i < 8; ++i) a_[0][i] = ld2(stage + (size_t)((g0 + 2) % S) * STAGE, i);
    wait_g(g0 + 3);
#pragma unroll
    for (int i = 0; i < 8; ++i) a_[1][i] = ld2(stage + (size_t)((g0 + 3) % S) * STAGE, i);
    bar_consumers_b2();
    if (t == 0)
      for (; issued < ntot && issued <= g0 + 2 + S; ++issued) issue();
    int sq = (g0 + 4) % S, sq1 = (g0 + 3) % S;
    int e0 = 0, e1 = 2;
    auto step = [&](int it, auto kc) {
      constexpr int K = decltype(kc)::value;
      constexpr int P0 = K, P1 = (K + 1) % 3, P2 = (K + 2) % 3;
      const int p = a + it, g = g0 + it + 4;
      wait_g(g);
      const double* sz = stage + (size_t)sq1 * STAGE;
      const double* sp = stage + (size_t)sq * STAGE;
#pragma unroll
      for (int i = 0; i < 8; ++i) a_[P2][i] = ld2(sp, i);
#pragma unroll
      for (int r = 0; r < 6; ++r) {
        const double2 c = a_[P1][r + 1];
        double xm = __shfl_up_sync(0xffffffffu, c.y, 1);
        double xp = __shfl_down_sync(0xffffffffu, c.x, 1);
        const uint32_t ea = smem_u32(sz + srow(r + 1, we) + xe);
        lds_if(xm, ea, is_left);
        lds_if(xp, ea, is_right);
        b_[P2][r].x = heat_update(c.x, xm, c.y, a_[P1][r].x, a_[P1][r + 2].x, a_[P0][r + 1].x, a_[P2][r + 1].x, it_.alpha);
        b_[P2][r].y = heat_update(c.y, c.x, xp, a_[P1][r].y, a_[P1][r + 2].y, a_[P0][r + 1].y, a_[P2][r + 1].y, it_.alpha);
      }
      {
        const double* em = edge + (size_t)e1 * ESLOT + e_nbr;
        double* o = b2_plane(dsto, p - 1, nty, tb, w, ty) + oyx;
#pragma unroll
        for (int j = 0; j < 4; ++j) {
          const double2 c = b_[P1][j + 1];
          double xm = __shfl_up_sync(0xffffffffu, c.y, 1);
          double xp = __shfl_down_sync(0xffffffffu, c.x, 1);
          lds_if(xm, smem_u32(em + j + 1), is_left);
          lds_if(xp, smem_u32(em + j + 1), is_right);
          double2 v;
          v.x = heat_update(c.x, xm, c.y, b_[P1][j].x, b_[P1][j + 2].x, b_[P0][j + 1].x, b_[P2][j + 1].x, it_.alpha);
          v.y = heat_update(c.y, c.x, xp, b_[P1][j].y, b_[P1][j + 2].y, b_[P0][j + 1].y, b_[P2][j + 1].y, it_.alpha);
          *reinterpret_cast<double2*>(o + j * TX) = v;
        }
      }
      if (p >= b - 2) {
        double* o = b2_plane(mido, p, nty, tb, w, ty) + oyx;
#pragma unroll
        for (int j = 0; j < 4; ++j) *reinterpret_cast<double2*>(o + j * TX) = b_[P2][j + 1];
      }
      {
        const uint32_t ez = smem_u32(edge + (size_t)e0 * ESLOT + e_mine);
#pragma unroll
        for (int r = 0; r < 6; ++r) {
          sts_if(ez + 8 * r, b_[P2][r].x, is_left);
          sts_if(ez + 8 * r, b_[P2][r].y, is_right);
        }
      }
      bar_consumers_b2();
      if (t == 0) {
        // this band's level s+1 planes up to p - 1 are written: publish every
        // PUB iterations and at the pass's end (a GPU-scope fence costs about
        // a plane's time; the neighbours read a pass's flags a pass later)
        if ((it + 1) % kIterPub == 0 || it + 1 == b - a) {
          fence_acq_rel_gpu();
          st_relaxed_gpu_u64(fl_me, ep | ((unsigned long long)k << 16) | (unsigned)(it + 1));
        }
        for (; issued < ntot && issued <= g - 1 + S; ++issued) issue();
      }
      sq1 = sq;
      sq = sq + 1 == S ? 0 : sq + 1;
      e1 = e0;
      e0 = e0 == 2 ? 0 : e0 + 1;
    };
    const int nit = b - a;
    for (int it = 0; it < nit; it += 3) {
      step(it, std::integral_constant<int, 0>{});
      if (it + 1 >= nit) break;
      step(it + 1, std::integral_constant<int, 1>{});
      if (it + 2 >= nit) break;
      step(it + 2, std::integral_constant<int, 2>{});
    }
  }
}

cudaError_t launch_heat2_band_iter(const Band2Iter& p, cudaStream_t s) {
  using namespace b2;
  if (p.c < 2 || p.P < 1) return cudaErrorNotSupported;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(heat2_band_iter, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  int dev = 0, sms = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const int grid = p.nty * p.ty / BY;
  if (grid > sms) return cudaErrorNotSupported;  // every band co-resident
  // a plain launch: waits for the previous kernel, lets nothing start early
  heat2_band_iter<<<grid, NT, SMEM, s>>>(p);
  return cudaGetLastError();
}

// driver entry point for cuTensorMapEncodeTiled (no -lcuda link dependency)
using EncodeTiledFn5 = CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                    const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                    CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

bool band2_maps_encode(Band2Maps* m, const double* base, int tx, int ty, int tz, int ntx, int nty, int ntz) {
  static EncodeTiledFn5 f = [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q{};
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess)
      return (EncodeTiledFn5) nullptr;
    return reinterpret_cast<EncodeTiledFn5>(p);
  }();
  static_assert(sizeof(CUtensorMap) == sizeof(TensorMapBlob), "CUtensorMap size");
  if (!f || !base || (reinterpret_cast<uintptr_t>(base) & 15) || tx != b2::TX || ntx != b2::NW || ty % b2::BY)
    return false;
  const uint64_t te = (uint64_t)tx * ty * tz;
  // x in the tile, y in the tile, tile column, z in the tile, tile row + layer (iz * nty + iy)
  const cuuint64_t dims[5] = {(cuuint64_t)tx, (cuuint64_t)ty, (cuuint64_t)ntx, (cuuint64_t)tz,
                              (cuuint64_t)nty * ntz};
  const cuuint64_t strides[4] = {(cuuint64_t)tx * 8, te * 8, (cuuint64_t)tx * ty * 8, te * ntx * 8};
  const cuuint32_t estr[5] = {1, 1, 1, 1, 1};
  for (int k = 0; k < 2; ++k) {
    const cuuint32_t box[5] = {(cuuint32_t)tx, k ? 2u : 4u, (cuuint32_t)ntx, 1, 1};
    if (f(reinterpret_cast<CUtensorMap*>(k ? &m->m2 : &m->m4), CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 5,
          const_cast<double*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
          CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) !=
        CUDA_SUCCESS)
      return false;
  }
  return true;
}

bool band2_shape_ok(int64_t nx, int64_t ny, int tx, int ty) {
  return tx == b2::TX && nx == (int64_t)b2::NW * b2::TX && ty % b2::BY == 0 && ny % b2::BY == 0;
}

cudaError_t launch_heat2_band(const Band2Maps& maps, double* dst, int ty, int tz, int nty, int ntz, double alpha,
                              cudaStream_t s) {
  using namespace b2;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(heat2_band, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)SMEM);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  const int ny = nty * ty, nz = ntz * tz;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3((unsigned)(ny / BY));
  cfg.blockDim = dim3(NT);
  cfg.dynamicSmemBytes = SMEM;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, heat2_band, maps, dst, ty, tz, nty, nz, (int64_t)TX * ty * tz, alpha);
}

}  // namespace tiles
