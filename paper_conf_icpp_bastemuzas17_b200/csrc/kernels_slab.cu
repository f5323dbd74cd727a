// kernels_slab.cu — "stream-through" (trapezoid) kernels, DESIGN.md §5.
//
// A z-layer of tiles plus T halo planes on each side is gathered into a
// dense slab ([planes][ny][nx], periodic in x and y within the plane), T
// Jacobi sweeps run on the slab with the valid z-range shrinking by one plane
// per sweep at each end, and the layer's tz exact core planes are scattered
// back into tile-blocked order for the D2H. Every cell update is the same
// rounded expression as heat7 (reading R1), so results are bit-identical.
// All three kernels are HBM-streaming (no reuse beyond neighbouring rows and
// planes, which L1/L2 catch): coalesced 128-bit accesses, grids sized in
// multiples of the SM count.
#include "kernels.cuh"
#include "ptx.cuh"

namespace tiles {

// dense slab plane p (global z = zbase + p, wrapped) <- tile-blocked array
__global__ void __launch_bounds__(256) slab_gather(const __grid_constant__ SlabParams p) {
  const int64_t nx = p.nx, ny = p.ny, tx = p.tx, ty = p.ty, tz = p.tz;
  const int64_t pairs_per_plane = nx * ny / 2;
  const int64_t total = pairs_per_plane * p.planes;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t pl = e / pairs_per_plane;
    const int64_t r = e - pl * pairs_per_plane;
    const int64_t y = (2 * r) / nx, x = (2 * r) % nx;
    int64_t gz = (p.zbase + pl) % p.nz;
    if (gz < 0) gz += p.nz;
    const int64_t iz = gz / tz, lz = gz % tz, ix = x / tx, iy = y / ty;
    const int64_t tile = (iz * p.nty + iy) * p.ntx + ix;
    const double* src = p.tiles + tile * p.tile_elems + (lz * ty + (y % ty)) * tx + (x % tx);
    *reinterpret_cast<double2*>(p.slab + (pl * ny + y) * nx + x) =
        *reinterpret_cast<const double2*>(src);
  }
}

// one Jacobi sweep on planes [lo, hi) of the slab (src -> dst), periodic in
// x and y; planes lo-1 and hi must be valid in src
__global__ void __launch_bounds__(256) slab_sweep(const __grid_constant__ SlabParams p,
                                                  const double* __restrict__ src,
                                                  double* __restrict__ dst, int lo, int hi) {
  const int64_t nx = p.nx, ny = p.ny;
  const int64_t pairs_per_plane = nx * ny / 2;
  const int64_t total = pairs_per_plane * (hi - lo);
  const double alpha = p.alpha;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t pl = lo + e / pairs_per_plane;
    const int64_t r = e % pairs_per_plane;
    const int64_t y = (2 * r) / nx, x = (2 * r) % nx;
    const double* row = src + (pl * ny + y) * nx;
    const double2 c = *reinterpret_cast<const double2*>(row + x);
    const double xm = row[x == 0 ? nx - 1 : x - 1];
    const double xp = row[x + 2 == nx ? 0 : x + 2];
    const int64_t ym_ = y == 0 ? ny - 1 : y - 1, yp_ = y + 1 == ny ? 0 : y + 1;
    const double2 ym = *reinterpret_cast<const double2*>(src + (pl * ny + ym_) * nx + x);
    const double2 yp = *reinterpret_cast<const double2*>(src + (pl * ny + yp_) * nx + x);
    const double2 zm = *reinterpret_cast<const double2*>(src + ((pl - 1) * ny + y) * nx + x);
    const double2 zp = *reinterpret_cast<const double2*>(src + ((pl + 1) * ny + y) * nx + x);
    double2 v;
    v.x = heat_update(c.x, xm, c.y, ym.x, yp.x, zm.x, zp.x, alpha);
    v.y = heat_update(c.y, c.x, xp, ym.y, yp.y, zm.y, zp.y, alpha);
    *reinterpret_cast<double2*>(dst + (pl * ny + y) * nx + x) = v;
  }
}

// tile-blocked layer (out) <- slab core planes [first, first+tz)
__global__ void __launch_bounds__(256) slab_scatter(const __grid_constant__ SlabParams p, int first) {
  const int64_t nx = p.nx, ny = p.ny, tx = p.tx, ty = p.ty, tz = p.tz;
  const int64_t pairs_per_plane = nx * ny / 2;
  const int64_t total = pairs_per_plane * tz;
  for (int64_t e = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; e < total;
       e += (int64_t)gridDim.x * blockDim.x) {
    const int64_t lz = e / pairs_per_plane;
    const int64_t r = e - lz * pairs_per_plane;
    const int64_t y = (2 * r) / nx, x = (2 * r) % nx;
    const int64_t tile = (y / ty) * p.ntx + (x / tx);  // within the layer
    double* o = p.out + tile * p.tile_elems + (lz * ty + (y % ty)) * tx + (x % tx);
    stg2_stream(o, *reinterpret_cast<const double2*>(p.slab + ((first + lz) * ny + y) * nx + x));
  }
}

static int slab_grid(int64_t work_pairs, int sms) {
  int64_t g = (work_pairs + 255) / 256;
  const int64_t cap = (int64_t)sms * 16;
  return (int)(g < 1 ? 1 : g > cap ? cap : g);
}

cudaError_t launch_slab_gather(const SlabParams& p, int sms, cudaStream_t s) {
  slab_gather<<<slab_grid(p.nx * p.ny / 2 * p.planes, sms), 256, 0, s>>>(p);
  return cudaGetLastError();
}

cudaError_t launch_slab_sweep(const SlabParams& p, const double* src, double* dst, int lo, int hi,
                              int sms, cudaStream_t s) {
  slab_sweep<<<slab_grid(p.nx * p.ny / 2 * (hi - lo), sms), 256, 0, s>>>(p, src, dst, lo, hi);
  return cudaGetLastError();
}

cudaError_t launch_slab_scatter(const SlabParams& p, int first, int sms, cudaStream_t s) {
  slab_scatter<<<slab_grid(p.nx * p.ny / 2 * p.tz, sms), 256, 0, s>>>(p, first);
  return cudaGetLastError();
}

}  // namespace tiles
