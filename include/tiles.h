/* tiles.h — C ABI of libtiles (B200-native tiled, stream-pipelined fp64 heat
 * stencil and compute-intensive kernel; Bastem et al., "Overlapping Data
 * Transfers with Computation on GPU with Tiles", ICPP 2017).
 *
 * Citations "P:L<n> §<s>" refer to the paper text (PAPER.md line n, section s).
 *
 * Model (§III, §IV.A): the grid is decomposed into regions
 * ("tiles") that are both the transfer unit and the execution unit. Each
 * tile's data lives in pinned host memory; as many tiles as fit are
 * placed on the device and the rest are streamed through a
 * pool of device slots, with transfers queued on CUDA streams so that they
 * overlap computation on other tiles. Ghost cells of a
 * tile are refreshed from its neighbours before each step.
 *
 * Conventions for every function:
 *  - Return TILE_OK (0) on success, otherwise a tile_status code; the
 *    thread-local message is available through tile_last_error().
 *  - TILE_EINVAL never has side effects.
 *  - A CUDA or NCCL failure (TILE_ECUDA / TILE_ENCCL) POISONS the domain:
 *    every later call except tile_free returns TILE_ESTATE.
 *  - Tests force these paths with TILES_FAULT=<kind>:<n> (kind = h2d, d2h,
 *    kernel, sync or host_alloc): the n-th such operation of a domain fails
 *    through the executor's real error path (on a GPU an invalid copy is
 *    queued, so the CUDA runtime reports the error; host_alloc requests an
 *    impossible pinned size). Unset, it costs one integer compare.
 *  - A domain is used from one host thread at a time.
 *  - Grids are fp64, C order [z][y][x] with x fastest. Sizes are int64.
 *  - Ownership: the library owns every pinned host buffer and device buffer
 *    it allocates. Arrays passed to tile_load / tile_store are borrowed for
 *    the duration of the call only. A caller-provided device pool or stream
 *    list (e.g. from PyTorch) is borrowed for the domain's lifetime and never
 *    freed by the library.
 *  - Multi-GPU (nranks > 1): z-slab decomposition; create / run / sync /
 *    free are COLLECTIVE (every rank calls them with identical global dims,
 *    tile_dims, ghost, kernel and steps); load / store move the rank's own
 *    slab. Halo planes travel between z-neighbour ranks via NCCL.
 */
#ifndef TILES_H
#define TILES_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct tile_domain tile_domain; /* opaque, library-owned */

typedef enum {
  TILE_OK = 0,
  TILE_EINVAL = 1,        /* bad argument (no side effects) */
  TILE_ENOMEM_HOST = 2,   /* pinned host allocation failed */
  TILE_ENOMEM_DEVICE = 3, /* device budget below the minimum slot count */
  TILE_ECUDA = 4,         /* CUDA runtime error (domain poisoned) */
  TILE_ENCCL = 5,         /* NCCL error (domain poisoned) */
  TILE_ESTATE = 6,        /* poisoned domain, or call not valid in this state */
  TILE_ENOSYS = 7         /* feature not compiled in (e.g. NCCL) */
} tile_status;

/* Boundary condition of the global grid (the paper is silent, R3). */
typedef enum { TILE_BC_PERIODIC = 0, TILE_BC_DIRICHLET = 1 } tile_bc;

typedef enum {
  /* 7-point Jacobi heat step, "uses its 6 nearest neighbors" (§VI.A):
   * v = u + alpha*(((xm+xp)+(ym+yp))+(zm+zp) - 6u)   (R1) */
  TILE_KERNEL_HEAT7 = 1,
  /* compute-intensive kernel, listing P:L219-L224 §VI.B: per cell,
   * inner_iters times: s=sin(x); c=cos(x); x=x+sqrt(s*s+c*c) */
  TILE_KERNEL_SINCOS = 2,
  TILE_KERNEL_USER = 3,  /* user pointwise function (tile_user_fn_create) */
  TILE_KERNEL_USER_STENCIL = 4 /* user 7-point stencil (tile_user_stencil_create) */
} tile_kernel_kind;

typedef struct tile_user_fn tile_user_fn; /* opaque, a compiled user function */

typedef struct {
  tile_kernel_kind kind;
  double alpha;        /* HEAT7: dt/dx^2, must be in (0, 1/6] (stability) */
  int32_t inner_iters; /* SINCOS: kernel_iteration of P:L220 (>= 0); USER:
                          applications of the function per cell per step */
  const tile_user_fn* user; /* USER: the function (borrowed for the run;
                          ignored for the other kinds) */
  const int64_t* box;   /* USER, optional: 6 values {x0, y0, z0, x1, y1, z1},
                          GLOBAL cell coordinates; the function is applied
                          only to cells with x0 <= x < x1 (etc.) — the
                          paper's ranged compute(tile, lo, hi), P:L126-L147;
                          tiles outside the box launch nothing. NULL = every
                          cell. EINVAL if x0 > x1 (etc.). */
} tile_kernel;

/* Schedules. AUTO picks RESIDENT when every tile fits in the
 * device budget twice (old/new buffers; once for SINCOS), else STREAM. */
typedef enum {
  TILE_SCHED_AUTO = 0,
  TILE_SCHED_RESIDENT = 1, /* all tiles in HBM, z-layer batches, events */
  TILE_SCHED_STREAM = 2,   /* out-of-core: per-tile slots, eviction */
  TILE_SCHED_SYNC = 3      /* synchronous baseline: H2D all, T steps, D2H all,
                              one stream, no overlap (Fig. 5 comparison) */
} tile_sched;

/* Measurement-only knobs (SURVEY.md §8(d) overlap efficiency): results of a
 * run in these modes are NOT valid and must not be checked. */
typedef enum {
  TILE_MEASURE_NORMAL = 0,
  TILE_MEASURE_XFER_ONLY = 1, /* issue every copy/event, launch no kernel */
  TILE_MEASURE_COMP_ONLY = 2  /* skip every host<->device copy */
} tile_measure;

typedef struct {
  int32_t device;               /* CUDA ordinal; -1 = current device */
  tile_bc bc;                   /* default TILE_BC_PERIODIC */
  uint64_t device_budget_bytes; /* 0: cudaMemGetInfo free - reserve;
                                   >0: hard cap, the paper's "limiting GPU
                                   memory" method */
  void* device_pool;            /* optional caller-owned device region ... */
  uint64_t device_pool_bytes;   /* ... and its size; borrowed, never freed */
  void* const* streams;         /* optional caller-owned cudaStream_t list */
  int32_t nstreams_provided;    /* number of entries in `streams` */
  int32_t nranks, rank;         /* z-slab decomposition; 1, 0 = single GPU */
  const void* nccl_unique_id;   /* 128 bytes, identical on all ranks (the
                                   caller broadcasts it, e.g. torch.distributed) */
  tile_sched sched;             /* default TILE_SCHED_AUTO */
  int32_t dry_run;              /* 1: no CUDA calls at all; the scheduler
                                   records its op trace (tests on CPU) */
  int32_t fuse_pointwise_steps; /* SINCOS: 1 (default) = all T steps of a tile
                                   in one residency pass (tile-major); 0 =
                                   step-major, every step re-streams (Fig. 8) */
  void* local_group;            /* optional in-process transport (see
                                   tile_local_group_create); replaces NCCL */
  int32_t pageable_host;        /* 1: host tile store from malloc (pageable),
                                   the paper's "CUDA pageable" baseline (P:L37,
                                   Fig. 1/5); copies are staged by the driver
                                   and do not overlap. 0 (default): pinned. */
  int32_t stream_through;       /* HEAT7 run starting from a fresh upload
                                   (periodic, T <= tile_dims[2], scratch fits;
                                   single rank, or z-slab ranks over the peer
                                   transport, whose windows then also hold two
                                   tile layers that carry the T planes of
                                   initial data beyond each slab end, once per
                                   run — DESIGN.md §6): per unit of planes (a slice
                                   of a z-layer, >= T planes) trapezoid: T
                                   sweeps over the unit + T halo planes, D2H
                                   of the exact core, so H2D, compute and D2H of
                                   different units overlap; each unit's result
                                   is also written back to the device array once
                                   no other unit reads its initial data.
                                   0 (default) = when a cost model (runtime.cpp
                                   streamthrough_ok) rates it faster than the
                                   batched resident schedule; 1 = whenever
                                   feasible; -1 = never. */
  int32_t peer_transport;       /* nranks > 1: 1 = halo exchange by direct
                                   device-to-device stores into the z-neighbour
                                   ranks' memory (CUDA IPC; NVLink / NVSwitch
                                   peer access), synchronised with stream
                                   memory operations on counters in the
                                   neighbours' memory — no NCCL. 2 = the same
                                   windows, but in resident single-step runs the
                                   stencil kernel itself stores each step's
                                   slab-end z layers into the neighbours'
                                   windows as it computes them (fused compute +
                                   exchange); the exchange after a step only
                                   signals. The caller gathers
                                   every rank's tile_peer_handle and passes them
                                   to tile_peer_connect before the first run.
                                   0 (default) = NCCL (or the local_group
                                   transport). */
  int32_t two_step;             /* HEAT7 with ghost >= 2: 0 (default) = two
                                   steps per pass in the streaming schedule
                                   (halves host-link bytes per step), single
                                   steps when resident; 1 = two steps in every
                                   schedule; -1 = never. Any ghost: resident
                                   periodic single-rank domains 512 cells wide
                                   with 64-wide tiles run two steps per kernel
                                   (heat2_band) unless -1, and with 1 their
                                   stream-through runs two sweeps per kernel
                                   (heat2_band_slab) */
  int32_t wavefront;            /* HEAT7 run starting from a fresh upload
                                   (periodic, single rank, resident, 2T planes
                                   of scratch fit): time-skewed march over
                                   chunks of planes — level s of chunk i
                                   covers planes [c*i - s, c*i + c - s), so a
                                   chunk needs only its own upload and the
                                   previous chunk, and its final planes go
                                   back to the host as soon as it ends; no
                                   redundant sweeps besides a T^2 bootstrap at
                                   the periodic seam. -1 =
                                   never, 0 (default) = when the cost model
                                   prefers it to stream-through and the
                                   batched schedule, 1 = whenever feasible.
                                   Grids 512 wide with 64-wide tiles take two
                                   levels per pass (heat2_band_slab, through a
                                   third level buffer when the budget holds
                                   it); 2 = whenever feasible, two levels per
                                   pass at any shape (slab_sweep2_tile off the
                                   band shape: slower than two single-level
                                   passes); 3 = whenever
                                   feasible, one level per pass */
  double sweep_link_ratio;      /* cost model of the fresh-upload schedules
                                   (DESIGN.md §5): time of one stencil sweep
                                   per plane over one plane's duplex host-link
                                   time. 0 (default) = measured on the device
                                   at tile_domain_create (a few ms: up to
                                   64 MiB of H2D and a 32-plane sweep, resident
                                   single-rank domains), else env TILES_ST_R,
                                   else 0.021 */
} tile_options;

typedef struct {
  uint64_t bytes_h2d, bytes_d2h, bytes_halo; /* payload moved */
  uint64_t n_h2d, n_d2h, n_kernels, n_halo;  /* operations issued */
  uint64_t hits, misses, evictions, writebacks;
  uint64_t steps_done;                       /* cell-update steps completed */
  double last_run_ms;                        /* host wall time of last tile_run..sync */
  double kernel_ms;                          /* summed device time of timed kernel launches */
  uint64_t kernel_timed;                     /* number of timed kernel launches */
  double sweep_ms;                           /* the part of kernel_ms spent in stencil
                                                sweeps (heat7, heat7x2, stream-through) */
  uint64_t sweep_cells;                      /* cells those timed sweeps read and wrote
                                                once each (16 B of algorithmic HBM traffic
                                                per cell; a two-step pass counts once) */
  uint64_t sweep_timed;                      /* number of timed sweep launches */
} tile_stats;

typedef struct {
  int64_t dims[3];        /* global grid (nx, ny, nz) */
  int64_t local_dims[3];  /* this rank's slab */
  int64_t tile_dims[3];
  int64_t tiles[3];       /* tiles per axis on this rank */
  int64_t ntiles;
  int64_t z_offset;       /* global z of the slab's first plane */
  int32_t ghost;
  int32_t nslots;         /* device interior buffers */
  int32_t sched;          /* schedule chosen for the last/next run */
  int32_t resident;       /* 1 if every tile currently has a valid device copy */
  uint64_t device_bytes;  /* device memory carved by the domain */
  uint64_t host_bytes;    /* pinned host memory of the tile store */
  int32_t steps_per_pass; /* HEAT7 steps per residency pass: 2 with ghost >= 2
                             (temporal blocking, single rank, supported tile
                             width), else 1 */
  int32_t last_schedule;  /* schedule the last tile_run took:
                             0 none yet, 1 resident batched (layer batches /
                             whole-domain steps), 2 stream-through (fresh
                             upload), 3 out-of-core per-tile stream, 4
                             out-of-core stream-through, 5 synchronous (one
                             stream), 6 wavefront (fresh upload), 7 resident,
                             two steps per kernel (heat2_band: periodic,
                             single rank, 512 cells wide, 64-wide tiles),
                             8 fresh upload at large T: wavefront during the
                             upload, resident two-step passes, wavefront
                             during the download */
  double sweep_link_ratio; /* the cost model's ratio in use (see tile_options) */
} tile_info;

/* One entry of the dry-run trace. */
typedef enum {
  TILE_OP_H2D = 1,      /* host tile a -> slot b */
  TILE_OP_D2H = 2,      /* slot b -> host tile a */
  TILE_OP_KERNEL = 3,   /* tile a: slot b -> slot c, face parity d (reads d, writes d^1) */
  TILE_OP_RECORD = 4,   /* event a recorded on stream */
  TILE_OP_WAIT = 5,     /* stream waits on event a */
  TILE_OP_FACES_H2D = 6,/* upload all host-extracted faces into parity d */
  TILE_OP_EXTRACT = 7,  /* tile a in slot b: export its faces into parity d */
  TILE_OP_HALO = 8,     /* slab halo exchange of parity d */
  TILE_OP_DROP = 9,     /* tile a leaves slot b without a copy (clean) */
  TILE_OP_HIT = 10,     /* tile a found in slot b (P:L90 cache hit) */
  TILE_OP_POINTWISE = 11,/* compute-intensive kernel on tile a in slot b, c iterations */
  TILE_OP_KERNEL2 = 12,  /* like KERNEL, two steps in one pass (ghost width 2) */
  TILE_OP_GATHER = 13,   /* reserved (no longer emitted: fused into SWEEP) */
  TILE_OP_SWEEP = 14,    /* one Jacobi sweep of slab planes [c & 0xffffffff, c >> 32),
                            periodic in x/y. a >= 0: dense slab at slot a; a < 0:
                            the resident array -1-a with slab plane 0 at local
                            z = d (wrapped). b >= 0: dense slab at slot b; b < 0:
                            packed sub-tiles at slot -1-b (sweep plane lo -> 0) */
  TILE_OP_SCATTER = 15,  /* reserved (no longer emitted: fused into SWEEP) */
  TILE_OP_COPY = 16,     /* device copy of c tile slots: slot a -> slot b */
  /* partial (sub-layer) copies of planes [d & 0xffffffff, + d >> 32) of c tiles: */
  TILE_OP_H2D_PART = 17, /* host tiles a.. -> slots b.. */
  TILE_OP_D2H_PART = 18, /* packed sub-tiles at slot b -> host tiles a.. */
  TILE_OP_COPY_PART = 19,/* packed sub-tiles at slot a -> slots b.. */
  TILE_OP_H2D_PACK = 20, /* host tiles a.. (c of them), planes [d & 0xffffffff, +d >> 32)
                            -> packed sub-tiles at slot b */
  TILE_OP_SWEEP_U = 21,  /* like SWEEP, source = units u-1, u, u+1 (packed sub-tiles at
                            slots b & 0x1fffff, b >> 21 & 0x1fffff, b >> 42), slab plane 0
                            at z = u*un - (hi + 1 - un) / 2; a = destination code,
                            c = lo | hi << 32, d = u | un << 32 */
  TILE_OP_KERNELD = 22,  /* like KERNEL (tile a: slot b -> slot c, face parity d), direct
                            ghosts: y/z ghosts read from the neighbours' interiors in the
                            buffer array holding slot b, x ghosts from the parity-d faces;
                            exports the x faces (and, multi-rank, the slab-end layers'
                            z faces) only; d | 0x100: the launch also stores its slab-end
                            z layers into the neighbour ranks' receive buffers (fused
                            halo push, peer_transport = 2) */
  TILE_OP_HALO_SIGNAL = 23,/* halo exchange of parity d whose data the previous kernels
                            pushed (fused): synchronisation only */
  TILE_OP_ST_HALO = 24,  /* multi-rank stream-through (peer transport): a = 0 push the
                            slab-end c planes of initial data (b = 1 top -> upper rank,
                            0 bottom -> lower rank), 1 wait for side b's halo layer,
                            2 release side b's halo layer; d = the run's epoch */
  TILE_OP_SYNC = 25,     /* host waits for every stream (stream -1): every op before it
                            completes before any op after it starts; host-side reads of
                            the pinned store (face extraction) happen here */
  TILE_OP_WSWEEP = 26,   /* wavefront sweep of planes [lo, hi) (c = lo | hi << 32, two
                            signed 32-bit halves), periodic in x/y; a = source view, b =
                            destination view: bit 0 = 1: planes z >= 0 in the tile-blocked
                            array starting at slot (code >> 1) & 0x7fffffff, z < 0 in the d
                            tile layers of scratch starting at slot code >> 32; bit 0 = 0:
                            resident array (bit 1), z wrapped (no scratch) */
  TILE_OP_D2H_PLANES = 27,/* planes [d & 0xffffffff, + d >> 32) of c tile slots b.. ->
                            the same planes of host tiles a.. */
  TILE_OP_COPY_PLANES = 28,/* planes [d & 0xffffffff, + d >> 32) of c tile slots a.. ->
                            the same planes of slots b.. */
  TILE_OP_WSWEEP2 = 29,  /* wavefront, two levels in one kernel (recorded as this op and the
                            next, TILE_OP_WSWEEP2_DST, on the same stream): level s on planes
                            [lo, hi) (c = lo | hi << 32, signed halves) from view a, written to
                            view b only at planes hi-2, hi-1 (its planes lo-2, lo-1 are read
                            from b); d = scratch layers. Views coded as for TILE_OP_WSWEEP */
  TILE_OP_WSWEEP2_DST = 30,/* the same kernel: level s+1 on [lo-1, hi-1) into view a */
  TILE_OP_BAND2 = 31,    /* two steps of the whole resident periodic grid in one kernel
                            (heat2_band): view a (the resident array, coded as for
                            TILE_OP_WSWEEP) -> view b; c = 0 | nz << 32 */
  TILE_OP_SWEEP2S = 32   /* stream-through, two sweeps in one kernel (heat2_band_slab):
                            operands as TILE_OP_SWEEP; level 1 on [lo, hi) stays on
                            chip, level 2 on [lo+1, hi-1) is written to b */
} tile_op_kind;

typedef struct {
  int32_t kind;   /* tile_op_kind */
  int32_t stream;
  int64_t a, b, c, d;
} tile_op;

/* Create a domain: decomposition (tiles = dims / tile_dims per axis), ghost
 * bookkeeping, pinned host tile store, device budget and slots.
 *  dims:      global grid (nx, ny, nz), each >= 1
 *  tile_dims: cells per tile per axis; must divide dims (ragged tiles are
 *             rejected, R6); tile_dims[0] and [1] must be even
 *             (128-bit vector access), and for nranks > 1 tile_dims[2] must
 *             divide nz / nranks.
 *  ghost:     ghost-cell width g, 1 <= g <= min(tile_dims) (HEAT7 reads the
 *             innermost layer; g is the width reported by tile_ghost_map).
 *  opt:       NULL = defaults (periodic, auto budget, 1 rank, own streams).
 * Errors: EINVAL, ENOMEM_HOST, ENOMEM_DEVICE, ECUDA, ENCCL, ENOSYS. */
tile_status tile_domain_create(const int64_t dims[3], const int64_t tile_dims[3],
                               int32_t ghost, const tile_options* opt,
                               tile_domain** out);

/* Copy the rank's dense slab into the pinned tile-blocked store (regions are
 * "physically separated"). PERIODIC: src is [nz_local][ny][nx].
 * DIRICHLET: src is [nz_local+2][ny+2][nx+2] including the fixed 1-deep halo
 * (the stencil radius), whose values are never updated. Invalidates device
 * copies. Implies tile_sync first if a run is in flight. */
tile_status tile_load(tile_domain* dom, const double* src);

/* Pointer to tile `tile_id`'s interior in the pinned host store (contiguous
 * [tz][ty][tx], x fastest), to fill or read it in place without a dense
 * staging array. Valid until tile_free. Writing through it requires a
 * following tile_mark_host_dirty. */
tile_status tile_host_tile(tile_domain* dom, int64_t tile_id, double** ptr);
tile_status tile_mark_host_dirty(tile_domain* dom);

/* GPU-disabled request of one region (§IV.B.4): if the tile's newest
 * data is on the device it is copied back on its stream and waited for
 * (P:L86), then *ptr = the tile's interior in the pinned host store
 * (contiguous [tz][ty][tx]). TILE_HOST_READ keeps the device copy (clean);
 * TILE_HOST_WRITE also drops it because CPU code will change the host data:
 * in the streaming schedule the tile's slot is freed, in the resident one
 * every device-newer tile is written back and the next run re-uploads the
 * domain. Valid until the next tile_run / tile_load / tile_free. */
typedef enum { TILE_HOST_READ = 0, TILE_HOST_WRITE = 1 } tile_host_mode;
tile_status tile_host_region(tile_domain* dom, int64_t tile_id, int32_t mode, double** ptr);

/* Host-side ghost update (§III, §IV.B.6: the ghost cells of a
 * region on the host are updated on the host): fills out (out_len >=
 * (tx+2g)(ty+2g)(tz+2g), layout of tile_ghost_map) with tile `tile_id` and
 * its g-deep shell from the host store — periodic wrap, Dirichlet fixed
 * faces (shell cells outside the domain in two or three axes are NaN: the
 * 7-point stencil never reads them). Device-newer tiles are written back
 * first (implicit tile_sync). z-slab ranks: TILE_EINVAL for tiles whose
 * shell reaches another rank. */
tile_status tile_host_ghosts(tile_domain* dom, int64_t tile_id, double* out, int64_t out_len);

/* GPU-disabled iteration (§IV.B.5: the paper's compute(tile, lambda)
 * with the tile iterator's GPU flag off, "no change in the source code for
 * both CPU and GPU executions"; the regions' newest data comes to the
 * host first, waited for as P:L86 requires; ghost cells of regions on
 * the host are updated on the host). For each tile id in ids[0..n) (ids
 * NULL: every rank-local tile in id order) the library calls, on the calling
 * thread,
 *   fn(ctx, tile_id, tile, shell, tile_dims, origin, ghost)
 * tile      = the tile's interior in the pinned host store ([tz][ty][tx], x
 *             fastest), writable when mode == TILE_HOST_WRITE;
 * shell     = with ghosted != 0, the tile and its g-deep shell as
 *             tile_host_ghosts fills it ((tz+2g)(ty+2g)(tx+2g), library-owned,
 *             valid during the call); with WRITE every listed tile's shell is
 *             gathered before the first call (host memory: one shell per
 *             listed tile), so an update written in place reads only old
 *             values through the shells (Jacobi order); with READ one shell
 *             at a time; NULL otherwise;
 * tile_dims = (tx, ty, tz); origin = the global (x, y, z) of tile[0].
 * The library runs no arithmetic on the cells itself: fn is the caller's CPU
 * code (the paper's lambda); every library cell update stays on the GPU.
 * READ leaves the device copies valid; WRITE hands the host the newest data
 * (device copies are dropped, as tile_mark_host_dirty; the next tile_run
 * re-uploads). fn must not call the library on the same domain (the
 * iteration is in progress). Errors: TILE_EINVAL (null fn, a bad id or mode, n < 0; no
 * side effects), TILE_ENOMEM_HOST (the shells), TILE_EINVAL from the gather
 * of a z-slab rank's end tiles (their shells live on another rank, checked
 * before any call), CUDA errors of the write-back poison the handle. */
typedef void (*tile_host_fn)(void* ctx, int64_t tile_id, double* tile, const double* shell,
                             const int64_t tile_dims[3], const int64_t origin[3], int32_t ghost);
tile_status tile_host_compute(tile_domain* dom, const int64_t* ids, int64_t n, int32_t mode,
                              int32_t ghosted, tile_host_fn fn, void* ctx);

/* Enqueue `steps` steps of kernel k over every tile (no sync
 * after issue). nstreams in [1, 64] streams carry transfers and kernels
 * (P:L81-L84). Returns once all work is enqueued; may block only for
 * residency back-pressure. Host data is not valid until tile_sync. */
tile_status tile_run(tile_domain* dom, const tile_kernel* k, int32_t steps,
                     int32_t nstreams);

/* Write back every dirty device tile (D2H) and wait for all streams; the host
 * store is then current (D2H needs synchronization). */
tile_status tile_sync(tile_domain* dom);

/* tile_sync, then copy the host store into the dense slab dst (same shape as
 * tile_load's src; DIRICHLET: only the interior of dst is written). */
tile_status tile_store(tile_domain* dom, double* dst);

/* Drop every device copy without a transfer (host store must be current,
 * i.e. after tile_sync); the next tile_run re-streams all tiles from host. */
tile_status tile_invalidate(tile_domain* dom);

/* Ghost-source map of one tile over its full expanded box (tz+2g, ty+2g,
 * tx+2g), z-major then y, x fastest: the GLOBAL linear index (z*ny+y)*nx+x
 * of the cell each position holds after periodic wrap, or -1 for a Dirichlet
 * boundary cell; interior cells map to themselves. out_len
 * must be >= (tz+2g)(ty+2g)(tx+2g). tile_id is rank-local. */
tile_status tile_ghost_map(const tile_domain* dom, int64_t tile_id, int64_t* out,
                           int64_t out_len);

/* Face-source descriptors actually used by the kernels: for tile tile_id and
 * each face f in (x-, x+, y-, y+, z-, z+), out[2f] = kind (0 = neighbour tile
 * export on this rank, 1 = Dirichlet fixed face, 2 = slab halo from rank
 * below, 3 = slab halo from rank above) and out[2f+1] = the neighbour's
 * rank-local tile id (kind 0) or the tile's position in its z-layer. */
tile_status tile_face_sources(const tile_domain* dom, int64_t tile_id, int64_t out[12]);

tile_status tile_get_info(const tile_domain* dom, tile_info* out);
tile_status tile_get_stats(const tile_domain* dom, tile_stats* out);
tile_status tile_reset_stats(tile_domain* dom);

/* Measurement mode (tile_measure) for subsequent runs. */
tile_status tile_set_measure(tile_domain* dom, int32_t mode);

/* Device-side timing. tile_timer_start joins every stream of the domain into
 * its first stream and records a timing event there; tile_timer_stop joins
 * again, records a second event, synchronizes and returns the elapsed device
 * milliseconds in *ms. With tile_set_kernel_timing(dom, 1) every kernel
 * launch is bracketed by events on its own stream — a run of consecutive
 * stencil sweeps on one stream by one pair around the run, so programmatic
 * dependent launch still overlaps them — and the summed durations are
 * reported in tile_stats.kernel_ms / kernel_timed (launches) after tile_sync
 * or tile_timer_stop. */
tile_status tile_timer_start(tile_domain* dom);
tile_status tile_timer_stop(tile_domain* dom, double* ms);
tile_status tile_set_kernel_timing(tile_domain* dom, int32_t on);

/* Dry-run trace: number of recorded ops, and copy of up to cap entries. */
tile_status tile_trace(const tile_domain* dom, tile_op* out, int64_t cap, int64_t* n);
tile_status tile_trace_clear(tile_domain* dom);

/* Release everything (implies tile_sync unless poisoned). NULL is a no-op. */
tile_status tile_free(tile_domain* dom);

/* Thread-local description of the last error (never NULL). */
const char* tile_last_error(void);

/* User pointwise kernels (general kernels; the paper's
 * compute(tile) runs user code over a region). `source` is CUDA C
 * defining
 *     __device__ double <name>(double u, long long gidx)
 * (u: the cell's current value; gidx = (z*ny + y)*nx + x, the cell's GLOBAL
 * linear index). NVRTC compiles it for sm_100a with --fmad=false inside a
 * wrapper that applies it inner_iters times per step to every cell, in place;
 * tile_run with {TILE_KERNEL_USER, 0, inner_iters, fn} then schedules tiles
 * like the compute-intensive kernel (resident, streamed out of core, fused
 * or step-major per tile_options.fuse_pointwise_steps; no ghosts).
 * Errors: EINVAL for a null source, a name that is not a C identifier, or a
 * compile error (the NVRTC log is in tile_last_error); ENOSYS if libnvrtc
 * cannot be loaded. The compiled cubin is loaded lazily on each device that
 * runs it. tile_user_fn_free: after the last run using the function has been
 * synchronised (tile_sync / tile_store / tile_free); NULL is a no-op. */
tile_status tile_user_fn_create(const char* source, const char* name, tile_user_fn** out);
tile_status tile_user_fn_free(tile_user_fn* fn);
/* User 7-point stencils (general kernels with ghost exchange): `source` defines
 *     __device__ double <name>(double c, double xm, double xp, double ym,
 *                              double yp, double zm, double zp)
 * (the cell and its six neighbours at the current step, ghosts included).
 * tile_run with {TILE_KERNEL_USER_STENCIL, 0, 0, fn} advances `steps` Jacobi
 * steps of u' = f(...) through the tile machinery: ghosts from the neighbour
 * tiles' exported faces (or Dirichlet fixed faces), each step exporting the new
 * boundary layers, resident or streamed out of core (the heat kernel's
 * specialised paths — direct ghosts, persistent and two-step launches,
 * stream-through — stay HEAT7-only). z-slab ranks exchange the slab-end
 * faces with copies (any transport). ghost = 1 (EINVAL otherwise). Free
 * with tile_user_fn_free like a pointwise function. */
tile_status tile_user_stencil_create(const char* source, const char* name, tile_user_fn** out);

/* Fill out[128] with a fresh ncclUniqueId (call on rank 0, then broadcast).
 * TILE_ENOSYS if built without NCCL. */
tile_status tile_nccl_unique_id(void* out128);

/* Peer transport (tile_options.peer_transport = 1 or 2). tile_peer_handle writes
 * the 64-byte CUDA IPC handle of this rank's halo window (receive buffers,
 * exchange counters and, for periodic slabs whose two tile layers fit 1 GiB,
 * the stream-through halo layers) to out64. tile_peer_connect takes every rank's
 * handle, `nranks` blobs of 64 bytes in rank order (the caller all-gathers
 * them, e.g. with torch.distributed), and maps the z-neighbours' windows;
 * it must precede the first tile_run. ESTATE if the domain has no window
 * (peer_transport off, single rank or dry run); ECUDA if a handle cannot be
 * opened (no peer access between the devices). */
tile_status tile_peer_handle(const tile_domain* dom, void* out64);
tile_status tile_peer_connect(tile_domain* dom, const void* handles, int32_t nranks);

/* In-process multi-rank transport for testing the slab path on ONE device:
 * every rank is a domain driven by its own host thread (ranks may share a
 * GPU); halo exchanges rendezvous on the host and move faces with device
 * copies ordered by cross-rank CUDA events. Pass the group in
 * tile_options.local_group (nranks must match). The group must outlive its
 * domains. */
tile_status tile_local_group_create(int32_t nranks, void** group);
tile_status tile_local_group_free(void* group);

/* Library version string. */
const char* tile_version(void);

#ifdef __cplusplus
}
#endif
#endif /* TILES_H */
