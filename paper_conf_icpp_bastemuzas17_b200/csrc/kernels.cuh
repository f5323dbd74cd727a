// kernels.cuh — internal interface between the runtime (scheduler.cpp) and
// the sm_100a kernels (kernels.cu). Not part of the C ABI.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace tiles {

// Face directions of a tile (regions expanded with ghost cells).
enum Face : int { XM = 0, XP = 1, YM = 2, YP = 3, ZM = 4, ZP = 5 };

// One tile processed by a kernel launch: its interior in (old) and out (new)
// device buffers, both contiguous [tz][ty][tx].
struct TileItem {
  const double* in;
  double* out;
  int32_t tile;  // rank-local tile id (indexes the ghost-source table)
  int32_t pad;
};

constexpr int kMaxInlineItems = 8;

// An edge line of ghost cells: cell i at ptr[i * stride] (ptr may be null
// when the edge is never read).
struct EdgePtr {
  const double* ptr;
  int64_t stride;
};

// Heat7 launch parameters (§VI.A; DESIGN.md §4 "heat7_tma").
struct HeatParams {
  int32_t tx, ty, tz;    // tile extents (cells)
  int32_t band;          // rows of a band (divides ty, even)
  int32_t nbands;        // ty / band
  int32_t nitems;
  double alpha;
  const TileItem* items; // device array, or nullptr -> inline_items
  TileItem inline_items[kMaxInlineItems];
  // Ghost-source planes for the READ parity: gsrc[tile*6 + face] points at the
  // plane holding the cells just outside `face` of `tile` (the neighbour's
  // export of the opposite face, a Dirichlet fixed face or a slab halo).
  const double* const* gsrc;
  // Export faces for the WRITE parity: face f of tile k starts at
  // fexp[f] + k * face_elems[f]. Layouts: x-faces [z][y], y-faces [z][x],
  // z-faces [y][x].
  double* fexp[6];
  int64_t face_elems[6];
  // L2 policy bits: 1 = TMA loads evict_first, 2 = face exports evict_last
  int32_t cache_flags;
  int32_t depth;  // face depth D (1 or 2): layers per face, increasing coordinate
  // Direct ghost sources (resident single-step passes; DESIGN.md §4 "direct
  // ghosts"): when gdir != nullptr the single-step kernels take the y and z
  // ghosts from gdir[tile*6 + f] instead of gsrc, where the pointer is the
  // NEAREST ghost layer itself — a neighbour tile's boundary plane / row inside
  // its resident interior, or the nearest layer of a face (Dirichlet fixed face,
  // slab halo) — and ystr[tile*2 + {0,1}] is the distance between consecutive
  // z of the y- / y+ source row (ty*tx inside a tile, D*tx in a face). x ghosts
  // always come from the exported x faces (gdir entries 0, 1 = face bases).
  const double* const* gdir;
  const int64_t* ystr;
  // Stacked z-march: the items are nstack tile layers of lt items each
  // (item (L, c) = items[L*lt + c], consecutive layers z-adjacent), and a
  // CTA's plane range runs through a column's tiles in z, so the ghost planes
  // between stacked tiles are the neighbour's own planes already in the ring.
  // nstack = 1, lt = nitems: independent tiles.
  int32_t nstack, lt;
  // Work order of the specialised kernels: the first rr_rounds * gridDim.x
  // columns (of lt * nbands) go round-robin, whole (CTA b takes columns b,
  // b + grid, ...: CTAs running side by side march adjacent bands of a tile
  // through the same planes, so the halo rows one reads are the rows its
  // neighbour CTA just staged — L2 hits instead of DRAM re-reads); the rest
  // is split into contiguous plane ranges. rr_rounds = 0: all contiguous.
  int32_t rr_rounds;
  // zchunk > 0: work items are z chunks of zchunk planes of a column (chunk-
  // major), dealt round-robin for rr_rounds rounds, so all CTAs march the same
  // planes of neighbouring columns at the same time; 0: whole columns.
  int32_t zchunk;
  // Exports: x faces always; y faces iff exp_y; the z- face of tile k iff
  // k < exp_zlo_below, the z+ face iff k >= exp_zhi_from (direct runs export
  // only what a face reader still needs: the slab-end layers' z faces for the
  // halo exchange of a multi-rank domain).
  int32_t exp_y;
  int32_t exp_zlo_below, exp_zhi_from;
  // Fused halo push (multi-rank peer transport): when non-null,
  // the z- exports of tiles k < exp_zlo_below are ALSO stored straight into
  // the lower neighbour rank's receive window at zpush_lo + k*face_elems[ZM],
  // and the z+ exports of tiles k >= exp_zhi_from into the upper neighbour's
  // at zpush_hi + (k - exp_zhi_from)*face_elems[ZP] (peer memory over
  // NVLink / NVSwitch); the halo op then only signals.
  double* zpush_lo;
  double* zpush_hi;
  // Persistent multi-step launch (nsteps > 1; DESIGN.md §4 "multi-step"):
  // single rank, whole domain resident, direct ghosts. Step s uses items /
  // gdir / fexp for even s and items_odd / gdir_odd / fexp_odd for odd s (the
  // two buffer arrays and face parities alternate). Between steps each CTA's
  // producer drains its ring, releases the consumers' stores at gpu scope and
  // arrives on the grid counter *prog; step s + 1 is staged once the counter
  // reaches (epoch + s + 1) * gridDim.x (epoch = barrier rounds of earlier
  // launches, so the counter is never reset). Requires all CTAs co-resident
  // (cooperative launch).
  int32_t nsteps;
  // Snake order (persistent launches): odd steps run every CTA's runs in
  // reverse, planes descending, so a step starts on the planes the CTA wrote
  // last in the previous step; the last keep_tail planes of a CTA's step are
  // stored with evict_last instead of streaming, so those reads are L2 hits.
  // (z+1 and z-1 swap roles in the march; their sum is commutative: same bits.)
  int32_t snake, keep_tail;
  int32_t ntx, nty;
  uint32_t epoch;
  unsigned long long* prog;
  const TileItem* items_odd;
  const double* const* gdir_odd;
  double* fexp_odd[6];
};

// Two-step pass (temporal blocking, ghost = 2): u^{s+2} from u^s in one
// launch; ghosts from depth-2 faces and edge lines (runtime.hpp EdgeSrc).
struct Heat2Params {
  HeatParams h;          // shape, items, face sources (read parity), exports
  const EdgePtr* esrc;   // [tile*12 + e] for the read parity
  // per tile: bit f set if face f is a Dirichlet fixed face (ring fixed)
  const uint8_t* fixed_mask;
};

struct SincosParams {
  int64_t tile_elems;
  int32_t nitems;
  int64_t iters;         // kernel_iteration * fused steps
  const TileItem* items;
  TileItem inline_items[kMaxInlineItems];
};

struct ExtractParams {   // export u's boundary layers into faces (parity p)
  int32_t tx, ty, tz;
  int32_t depth;
  int32_t nitems;
  const TileItem* items; // uses .in and .tile
  TileItem inline_items[kMaxInlineItems];
  double* fexp[6];
  int64_t face_elems[6];
};

// Launch helpers (return cudaError_t of the launch).
struct HeatLaunchCfg {
  int stages;
  int threads;
  int grid;
  size_t smem;
};
// Pick the band height and pipeline depth for a tile shape; false if the
// shape cannot be staged (then tile_domain_create rejects it).
bool heat_plan(int tx, int ty, int max_smem, int* band, int* stages, size_t* smem);
cudaError_t heat_configure(int tx, int ty, int band, int stages, size_t smem, int* ctas_per_sm);
cudaError_t launch_heat7(const HeatParams& p, int stages, size_t smem, int grid,
                         cudaStream_t s);
// true if launch_heat7 runs a specialised kernel for this plan (the only
// ones taking direct ghost sources and stacked tiles)
bool heat_is_fixed(int tx, int band, int stages, size_t smem);
cudaError_t launch_sincos(const SincosParams& p, int grid, cudaStream_t s);

// Stream-through (trapezoid) slab kernels (kernels_slab.cu).
// A stream-through slab seen through a (possibly tile-blocked) layout: slab
// plane p, row y, column x live at
//   base + [iz*nty*ntx*te + lz*ty*tx] + [iy*ntx*te + ly*tx] + [ix*te + lx]
// with gz = zbase + p (wrapped mod nz if nz > 0), (iz, lz) = divmod(gz, tz),
// (iy, ly) = divmod(y, ty), (ix, lx) = divmod(x, tx). A dense slab is the view
// with tx = nx, ty = ny, one tile.
// Unit-ring variant (out-of-core stream-through): plane gz lies in unit
// iu = gz / un, held as packed sub-tiles (te = un*ty*tx) in ubase[(iu - u + 1)
// mod U] (units u-1, u, u+1), local plane gz - iu*un; base is unused.
struct SlabView {
  double* base;
  int64_t te;                   // elements per tile (or per packed sub-tile)
  int tx, ty, tz, ntx, nty;
  int zbase, nz;
  int ring;                     // 1: unit-ring view (below)
  int u, U, un;
  double* ubase[3];
  double* hlo;                  // resident view: planes z < 0 from nlo tile-blocked layers here
  double* hhi;                  // (multi-rank halo layer, nlo = 1; wavefront scratch), planes
  int nlo;                      // z >= nz (planes z-nz) from hhi, instead of the periodic wrap
};
// TMA tensor maps over the tile slots for the sweep kernel's x-halo columns
// (2 x band cells per side, a strided column): [k] views memory [base[k],
// end[k]) as rows of tx doubles (k = 0 the slot pool, 1 the wavefront
// scratch); valid[k] = 0 when absent. Opaque 128-byte CUtensorMap blobs.
struct alignas(64) TensorMapBlob {
  unsigned char b[128];
};
struct SweepMaps {
  TensorMapBlob xmap[2];
  TensorMapBlob xmap2[2];  // the same memory, box {2, 2} (the two-level sweep's extra halo rows)
  const double* base[2];
  const double* end[2];
  int valid[2];
  int band;  // box rows the maps were encoded for
};
// encode map k over [base, base + bytes) as rows of tx doubles, box {2, band}
bool sweep_map_encode(SweepMaps* m, int k, const double* base, uint64_t bytes, int tx, int band);
int sweep_tile_band();  // box rows (band) of the tile-column sweep kernel
// Two levels per pass (wavefront with three level buffers):
// level s on planes [a, b) from src (level s-1) stays on chip except its top
// two planes, written to mid (whose planes a-2, a-1 it reads); level s+1 on
// [a-1, b-1) into dst. src and dst must not share memory. Returns
// cudaErrorNotSupported when the shapes do not fit.
cudaError_t launch_slab_sweep2(const SlabView& src, const SlabView& mid, const SlabView& dst, int nx, int ny, int a,
                               int b, double alpha, int sms, cudaStream_t s, const SweepMaps* maps);
// Two steps per pass over a resident periodic grid 512 cells wide
// (heat2_band, kernels_band2.cu): 5-D tensor maps over one resident array
// (boxes of 4 and 2 rows x 64 x 8 tile columns).
struct Band2Maps {
  TensorMapBlob m4, m2;
};
bool band2_shape_ok(int64_t nx, int64_t ny, int tx, int ty);
bool band2_maps_encode(Band2Maps* m, const double* base, int tx, int ty, int tz, int ntx, int nty, int ntz);
// u^{s+2} of the whole grid into dst (the resident array layout) from the
// array the maps were encoded over
cudaError_t launch_heat2_band(const Band2Maps& maps, double* dst, int ty, int tz, int nty, int ntz, double alpha,
                              cudaStream_t s);
// two-level passes on the band layout over general views (heat2_band_slab):
// a view is a tile-blocked region (tiles of tz planes, `layers` tile layers;
// plane z of the view is region plane z + zbase, taken mod nz when wrap)
// plus nlo scratch tile layers for region planes < 0. Inputs go through TMA
// (maps encoded over the region / the scratch), outputs are written directly.
struct Band2View {
  Band2Maps main, scr;
  int nlo, wrap, tz, zbase, nz;
};
struct Band2Out {
  double* base;
  double* hlo;
  int64_t te;  // elements per tile
  int nlo, tz, zbase;
};
// mid = 1 (the wavefront, slab_sweep2 semantics): level s on [a, b) from
// src, its planes b-2, b-1 written to mid (whose planes a-2, a-1 it reads),
// level s+1 on [a-1, b-1) into dst. mid = 0 (stream-through): level s on
// [a, b) from src kept on chip, level s+1 on [a+1, b-1) into dst.
cudaError_t launch_heat2_band_slab(int mid_mode, const Band2View& src, const Band2View& mid, const Band2Out& mido,
                                   const Band2Out& dsto, int ty, int nty, int a, int b, double alpha,
                                   cudaStream_t s);
// all two-level passes of one wavefront iteration (heat2_band_iter): level
// views v[k] = lvl(s) for s % 3 == k (s >= 1), v[3] = lvl(0) (the resident
// array); o[k] the level arrays as outputs; pass k runs levels s0 + 2k and
// s0 + 2k + 1 on planes [ci - s, ci - s + c); bands synchronise through
// per-band progress flags (nbands u64, epoch in the high half)
struct Band2Iter {
  Band2View v[4];
  Band2Out o[3];
  unsigned long long* flags;
  unsigned long long epoch;
  int ty, nty, ci, c, s0, P;
  double alpha;
};
cudaError_t launch_heat2_band_iter(const Band2Iter& p, cudaStream_t s);
// device -> mapped pinned host rows copied by the SMs (pitches, len in doubles;
// len and pitches even)
cudaError_t launch_push_rows(const double* src, int64_t src_pitch, double* dst, int64_t dst_pitch, int64_t rows,
                             int64_t len, int ctas, cudaStream_t st);
cudaError_t launch_slab_sweep(const SlabView& src, const SlabView& dst, int nx, int ny, int lo,
                              int hi, double alpha, int sms, cudaStream_t s, const SweepMaps* maps = nullptr);
// Two-step kernel: returns false from heat2_plan if no specialisation fits.
bool heat2_plan(int tx, int ty, int max_smem, int* band, size_t* smem);
cudaError_t heat2_configure(int tx, int band, size_t smem, int* ctas_per_sm);
cudaError_t launch_heat7x2(const Heat2Params& p, size_t smem, int grid, cudaStream_t s);
cudaError_t launch_extract(const ExtractParams& p, cudaStream_t s);

}  // namespace tiles
