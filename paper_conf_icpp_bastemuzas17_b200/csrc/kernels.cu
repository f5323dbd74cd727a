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

#include <algorithm>

namespace tiles {

// --------------------------------------------------------------- PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
               "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// 1-D bulk copy global -> shared, completion signalled on `bar` (TMA engine).
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes,
                                         uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}

// Reading R1: s = ((xm+xp)+(ym+yp))+(zm+zp); v = c + alpha*(s - 6c).
// Explicit _rn intrinsics are never contracted into FMAs.
__device__ __forceinline__ double heat_update(double c, double xm, double xp, double ym,
                                              double yp, double zm, double zp, double alpha) {
  const double s = __dadd_rn(__dadd_rn(__dadd_rn(xm, xp), __dadd_rn(ym, yp)), __dadd_rn(zm, zp));
  return __dadd_rn(c, __dmul_rn(alpha, __dsub_rn(s, __dmul_rn(6.0, c))));
}

// ---------------------------------------------------------------- heat7_tma
template <int NT>
__global__ void __launch_bounds__(NT) heat7_tma(const __grid_constant__ HeatParams p,
                                                const int stages) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  const int tx = p.tx, ty = p.ty, tz = p.tz, BY = p.band;
  const int rows = BY + 2;
  const int stage_elems = rows * tx + 2 * BY;  // rows + x-ghost columns
  double* stage_base = reinterpret_cast<double*>(smem_raw);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem_raw + (size_t)stages * stage_elems * 8);

  if (threadIdx.x == 0) {
    for (int s = 0; s < stages; ++s) mbar_init(&bars[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  const int64_t ncols = (int64_t)p.nitems * p.nbands;
  const int64_t P = ncols * tz;
  const int64_t pb = P * blockIdx.x / gridDim.x;
  const int64_t pe = P * (blockIdx.x + 1) / gridDim.x;
  const int half = tx >> 1;
  const bool rowmap = (half <= NT) && (NT % half == 0);
  const int rpp = rowmap ? NT / half : 0;
  const int my_c2 = rowmap ? (int)threadIdx.x % half : 0;
  const int my_r0 = rowmap ? (int)threadIdx.x / half : 0;
  const double alpha = p.alpha;
  uint32_t seq = 0;  // planes sequenced through the ring by this CTA

  for (int64_t pp = pb; pp < pe;) {
    const int64_t col = pp / tz;
    const int z0 = (int)(pp - col * tz);
    const int z1 = (int)(pe - pp < (int64_t)(tz - z0) ? z0 + (pe - pp) : tz);
    const int item_i = (int)(col / p.nbands);
    const int y0 = (int)(col - (int64_t)item_i * p.nbands) * BY;
    const TileItem it = p.items ? p.items[item_i] : p.inline_items[item_i];
    const double* const* gs = p.gsrc + (size_t)it.tile * 6;
    const int nq = z1 - z0 + 2;  // planes z0-1 .. z1

    // Producer: stage plane q (z = z0-1+q) of this run.
    auto issue = [&](int q) {
      const uint32_t g = seq + q;
      const int s = (int)(g % stages);
      double* dst = stage_base + (size_t)s * stage_elems;
      uint64_t* bar = &bars[s];
      const int z = z0 - 1 + q;
      fence_proxy_async();
      if (z < 0 || z >= tz) {  // z-ghost plane: band rows of the z- / z+ source face
        const double* src = gs[z < 0 ? ZM : ZP] + (size_t)y0 * tx;
        const uint32_t bytes = (uint32_t)BY * tx * 8;
        mbar_expect_tx(bar, bytes);
        bulk_g2s(dst + tx, src, bytes, bar);
      } else {
        const uint32_t row_b = (uint32_t)tx * 8;
        const uint32_t total = (uint32_t)stage_elems * 8;
        mbar_expect_tx(bar, total);
        const double* plane = it.in + (size_t)z * ty * tx;
        bulk_g2s(dst + tx, plane + (size_t)y0 * tx, row_b * BY, bar);
        const double* lo = y0 > 0 ? plane + (size_t)(y0 - 1) * tx : gs[YM] + (size_t)z * tx;
        const double* hi =
            y0 + BY < ty ? plane + (size_t)(y0 + BY) * tx : gs[YP] + (size_t)z * tx;
        bulk_g2s(dst, lo, row_b, bar);
        bulk_g2s(dst + (size_t)(BY + 1) * tx, hi, row_b, bar);
        bulk_g2s(dst + (size_t)rows * tx, gs[XM] + (size_t)z * ty + y0, (uint32_t)BY * 8, bar);
        bulk_g2s(dst + (size_t)rows * tx + BY, gs[XP] + (size_t)z * ty + y0, (uint32_t)BY * 8,
                 bar);
      }
    };
    auto wait_q = [&](int q) {
      const uint32_t g = seq + q;
      mbar_wait(&bars[g % stages], (g / stages) & 1u);
    };

    if (threadIdx.x == 0) {
      const int first = min(stages, nq);
      for (int q = 0; q < first; ++q) issue(q);
    }
    wait_q(0);
    wait_q(1);

    const int64_t tile = it.tile;
    double* fxm = p.fexp[XM] + tile * p.face_elems[XM];
    double* fxp = p.fexp[XP] + tile * p.face_elems[XP];
    double* fym = p.fexp[YM] + tile * p.face_elems[YM];
    double* fyp = p.fexp[YP] + tile * p.face_elems[YP];
    double* fzm = p.fexp[ZM] + tile * p.face_elems[ZM];
    double* fzp = p.fexp[ZP] + tile * p.face_elems[ZP];

    for (int i = 0; i < z1 - z0; ++i) {
      wait_q(i + 2);
      const int z = z0 + i;
      const double* prv = stage_base + (size_t)((seq + i) % stages) * stage_elems;
      const double* cur = stage_base + (size_t)((seq + i + 1) % stages) * stage_elems;
      const double* nxt = stage_base + (size_t)((seq + i + 2) % stages) * stage_elems;
      const double* xlo = cur + (size_t)rows * tx;
      const double* xhi = xlo + BY;
      double* out_plane = it.out + (size_t)z * ty * tx;

      auto cell_pair = [&](int r, int c2) {
        const int x = c2 << 1;
        const double* crow = cur + (size_t)(r + 1) * tx;
        const double2 c = *reinterpret_cast<const double2*>(crow + x);
        const double2 ym = *reinterpret_cast<const double2*>(cur + (size_t)r * tx + x);
        const double2 yp = *reinterpret_cast<const double2*>(cur + (size_t)(r + 2) * tx + x);
        const double2 zm = *reinterpret_cast<const double2*>(prv + (size_t)(r + 1) * tx + x);
        const double2 zp = *reinterpret_cast<const double2*>(nxt + (size_t)(r + 1) * tx + x);
        const double xm = x == 0 ? xlo[r] : crow[x - 1];
        const double xp = x + 2 == tx ? xhi[r] : crow[x + 2];
        double2 v;
        v.x = heat_update(c.x, xm, c.y, ym.x, yp.x, zm.x, zp.x, alpha);
        v.y = heat_update(c.y, c.x, xp, ym.y, yp.y, zm.y, zp.y, alpha);
        const int y = y0 + r;
        *reinterpret_cast<double2*>(out_plane + (size_t)y * tx + x) = v;
        // Epilogue: export the new boundary layers (ghost sources of the
        // neighbours for the next step).
        if (x == 0) fxm[(size_t)z * ty + y] = v.x;
        if (x + 2 == tx) fxp[(size_t)z * ty + y] = v.y;
        if (y == 0) *reinterpret_cast<double2*>(fym + (size_t)z * tx + x) = v;
        if (y == ty - 1) *reinterpret_cast<double2*>(fyp + (size_t)z * tx + x) = v;
        if (z == 0) *reinterpret_cast<double2*>(fzm + (size_t)y * tx + x) = v;
        if (z == tz - 1) *reinterpret_cast<double2*>(fzp + (size_t)y * tx + x) = v;
      };
      if (rowmap) {
        for (int r = my_r0; r < BY; r += rpp) cell_pair(r, my_c2);
      } else {
        const int npairs = BY * half;
        for (int e = threadIdx.x; e < npairs; e += NT) cell_pair(e / half, e % half);
      }
      __syncthreads();  // stage of plane z-1 is free
      if (threadIdx.x == 0 && i + stages < nq) issue(i + stages);
    }
    seq += (uint32_t)nq;
    pp += z1 - z0;
  }
}

constexpr int kHeatThreads = 256;

bool heat_plan(int tx, int ty, int max_smem, int* band, int* stages, size_t* smem) {
  if (tx < 2 || (tx & 1) || ty < 2 || (ty & 1)) return false;
  // Largest even divisor of ty (<= 64) whose ring fits; prefer 5 stages
  // (3 planes in use + 2 in flight), accept 4 or 3.
  // A band thinner than 16 rows re-reads >12% halo rows; trade a stage for it.
  const int want = std::min(ty, 16);
  int best_by = 0, best_s = 0;
  for (int S : {5, 4, 3}) {
    for (int by = std::min(ty, 64); by >= 2; --by) {
      if ((by & 1) || ty % by) continue;
      size_t bytes = (size_t)S * ((size_t)(by + 2) * tx + 2 * by) * 8 + (size_t)S * 8;
      if (bytes > (size_t)max_smem) continue;
      if (by > best_by) { best_by = by; best_s = S; }
      break;
    }
    if (best_by >= want) break;
  }
  if (!best_by) return false;
  *band = best_by;
  *stages = best_s;
  *smem = (size_t)best_s * ((size_t)(best_by + 2) * tx + 2 * best_by) * 8 + (size_t)best_s * 8;
  return true;
}

cudaError_t heat_configure(int tx, int ty, int band, int stages, size_t smem, int* ctas_per_sm) {
  (void)tx; (void)ty; (void)band; (void)stages;
  cudaError_t e = cudaFuncSetAttribute(heat7_tma<kHeatThreads>,
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(ctas_per_sm, heat7_tma<kHeatThreads>,
                                                       kHeatThreads, smem);
}

cudaError_t launch_heat7(const HeatParams& p, int stages, size_t smem, int grid,
                         cudaStream_t s) {
  heat7_tma<kHeatThreads><<<grid, kHeatThreads, smem, s>>>(p, stages);
  return cudaGetLastError();
}

// -------------------------------------------------------------- sincos_iter
// Listing P:L219-L224: per cell, `iters` times: s=sin(x); c=cos(x);
// x = x + sqrt(s*s + c*c). sincos() shares the argument reduction of sin and
// cos; each thread carries two independent cells (ILP). No FMA contraction.
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
    for (int64_t k = 0; k < p.iters; ++k) {
      double sa, ca, sb, cb;
      sincos(a, &sa, &ca);
      sincos(b, &sb, &cb);
      a = __dadd_rn(a, __dsqrt_rn(__dadd_rn(__dmul_rn(sa, sa), __dmul_rn(ca, ca))));
      b = __dadd_rn(b, __dsqrt_rn(__dadd_rn(__dmul_rn(sb, sb), __dmul_rn(cb, cb))));
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
  const int tx = p.tx, ty = p.ty, tz = p.tz;
  double* dst = p.fexp[f] + (int64_t)it.tile * p.face_elems[f];
  const int64_t n = p.face_elems[f];
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < n;
       e += (int64_t)gridDim.x * blockDim.x) {
    int64_t src;
    if (f <= XP) {  // [z][y]
      const int64_t z = e / ty, y = e % ty;
      src = (z * ty + y) * tx + (f == XM ? 0 : tx - 1);
    } else if (f <= YP) {  // [z][x]
      const int64_t z = e / tx, x = e % tx;
      src = (z * ty + (f == YM ? 0 : ty - 1)) * tx + x;
    } else {  // [y][x]
      src = (int64_t)(f == ZM ? 0 : tz - 1) * ty * tx + e;
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
