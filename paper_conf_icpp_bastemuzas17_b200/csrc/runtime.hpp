// runtime.hpp — internal state of a tile domain (not part of the C ABI).
#pragma once
#include <cstdint>
#include <deque>
#include <functional>
#include <string>
#include <vector>

#include "../../include/tiles.h"
#include "kernels.cuh"

namespace tiles {

struct Status {
  tile_status code = TILE_OK;
  std::string msg;
  static Status ok() { return {}; }
  bool bad() const { return code != TILE_OK; }
};
Status make_err(tile_status c, const std::string& m);

// ------------------------------------------------------------------ geometry
// Decomposition of a rank's z-slab into tiles (§III, §IV.A).
struct Geometry {
  int64_t g[3];   // global nx, ny, nz
  int64_t l[3];   // local nx, ny, nz (slab)
  int64_t t[3];   // tile dims
  int64_t n[3];   // tiles per axis (local)
  int64_t ntiles;
  int64_t zoff;   // global z of local z = 0
  int ghost;
  int depth;      // face depth D = min(ghost, 2): layers exported per face
  tile_bc bc;
  int nranks, rank;
  int64_t tile_elems;
  int64_t face_elems[6];
  int64_t layer_tiles;  // tiles per z-layer = n[0]*n[1]

  void tile_coords(int64_t id, int64_t* ix, int64_t* iy, int64_t* iz) const {
    *ix = id % n[0];
    *iy = (id / n[0]) % n[1];
    *iz = id / (n[0] * n[1]);
  }
  int64_t tile_id(int64_t ix, int64_t iy, int64_t iz) const {
    return (iz * n[1] + iy) * n[0] + ix;
  }
};

Status make_geometry(const int64_t dims[3], const int64_t tdims[3], int ghost, tile_bc bc,
                     int nranks, int rank, Geometry* out);

// Face source of tile `id`, face f: kind 0 = export of a
// neighbour tile on this rank (val = its id), 1 = Dirichlet fixed face
// (val = id), 2 = halo from the rank below (val = position in layer),
// 3 = halo from the rank above (val = position in layer).
struct FaceSrc {
  int kind;
  int64_t val;
};
FaceSrc face_source(const Geometry& G, int64_t id, int f);

// Edge ghost cells for a two-step pass (D = 2): the 12 lines of cells just
// outside two faces at once (x,y,z = -1 or t in two axes). Edge e: 0..3 = xy
// (cells along z), 4..7 = xz (along y), 8..11 = yz (along x); within a group
// (e & 3) = 2*g_a + g_b with g = 0 for the minus side, 1 for the plus side of
// the group's first and second axis. Cell i of the line is ptr[i * stride].
// The value lives in a depth-2 face array: a diagonal neighbour's export, or
// a Dirichlet fixed face of the tile that borders the out-of-domain axis.
// kind: 0 export (parity-dependent), 1 Dirichlet face, -1 not needed (both
// axes leave a Dirichlet domain), -2 unsupported (crosses a slab seam).
struct EdgeSrc {
  int kind;
  int64_t tile;   // owner of the face array
  int face;       // which face array of that tile
  int64_t offset; // element offset of cell 0 within that tile's face
  int64_t stride; // element stride along the line
};
EdgeSrc edge_source(const Geometry& G, int64_t id, int e);
void ghost_map(const Geometry& G, int64_t id, int64_t* out);  // (t+2g)^3 box

// ----------------------------------------------------------------- executor
// All device work goes through an executor: CudaExec issues CUDA/NCCL calls,
// DryExec only records the op trace (tests on a CPU-only box).
struct Domain;
// Where a stream-through slab lives (runtime.cpp run_streamthrough):
//   DENSE    - dense [plane][ny][nx] scratch at tile slot `slot`;
//   RESIDENT - the tile-blocked resident array `slot` (0/1), slab plane 0 at
//              local z = zbase (wrapped);
//   SUB      - the unit's packed sub-tiles at slot `slot`; slab plane lo of
//              the sweep is sub-tile plane 0.
//   UNITS    - (source only) units u-1, u, u+1 of `un` planes each as packed
//              sub-tiles at slots ring[0..2]; slab plane 0 at local z = zbase
//              (wrapped), z in unit z / un.
//   WAVE     - wavefront (runtime.cpp run_wavefront): the tile-blocked
//              array starting at slot `slot` for planes z >= 0 (no wrap) and,
//              for z < 0, ring[0] = first slot of un tile layers of scratch
//              holding planes [-un*tz, 0).
struct SlabRef {
  enum Kind { DENSE = 0, RESIDENT = 1, SUB = 2, UNITS = 3, WAVE = 4 };
  int kind;
  int slot;
  int64_t zbase;
  int ring[3];
  int64_t u, un;
};

struct Exec {
  virtual ~Exec() = default;
  virtual Status h2d(Domain& d, int64_t tile0, int64_t ntile, int slot0, int stream) = 0;
  virtual Status d2h(Domain& d, int64_t tile0, int64_t ntile, int slot0, int stream) = 0;
  virtual Status record(Domain& d, int ev, int stream) = 0;
  virtual Status wait(Domain& d, int ev, int stream) = 0;
  // heat over tiles [tile0, tile0+ntile) of one z-layer batch (resident) or
  // one tile (stream); in/out given by slots
  // direct_bit >= 0: resident pass reading y/z ghosts straight from the
  // neighbours' interiors in buffer array direct_bit (HeatParams::gdir);
  // nstack: the items are nstack consecutive tile layers (stacked z-march)
  virtual Status heat(Domain& d, const int64_t* tiles, const int* in_slots, const int* out_slots,
                      int nitems, int read_parity, const TileItem* dev_items, int stream,
                      int direct_bit = -1, int nstack = 1, int nsteps = 1) = 0;
  virtual Status sincos(Domain& d, int64_t tile, int slot, int64_t iters, int stream) = 0;
  // stream-through: one Jacobi sweep of slab planes [lo, hi) (periodic in
  // x and y) from src to dst; see SlabRef
  virtual Status slab_sweep(Domain& d, const SlabRef& src, const SlabRef& dst, int lo, int hi,
                            int stream) = 0;
  virtual Status copy_slots(Domain& d, int src_slot, int dst_slot, int64_t n, int stream) = 0;
  // wavefront, two levels per pass (three level buffers): level s on planes
  // [a, b) from src, only its top two planes written to mid (whose planes a-2,
  // a-1 are read), level s+1 on [a-1, b-1) into dst
  virtual Status slab_sweep2(Domain& d, const SlabRef& src, const SlabRef& mid, const SlabRef& dst, int a, int b,
                             int stream) = 0;
  // the wavefront: passes k = 0..P-1 of iteration ci/c (levels s0+2k,
  // s0+2k+1 on [ci - s, ci - s + c)) in one launch (heat2_band_iter); lv[k]
  // the view of the levels s with s % 3 == k, lv[3] level 0; the trace
  // records the passes as separate TILE_OP_WSWEEP2 ops
  virtual bool wave_iter_ok(Domain& d) = 0;
  virtual Status wave_iteration(Domain& d, const SlabRef* lv, int64_t ci, int c, int s0, int P, int stream) = 0;
  // stream-through, two sweeps in one kernel (heat2_band_slab, shrink mode):
  // level 1 on [lo, hi) from src kept on chip, level 2 on [lo+1, hi-1) into
  // dst; sweep2s_ok: the executor runs it for this domain's shape
  virtual bool sweep2s_ok(Domain& d) = 0;
  virtual Status slab_sweep2s(Domain& d, const SlabRef& src, const SlabRef& dst, int lo, int hi, int stream) = 0;
  // two steps of the whole resident periodic grid in one kernel (heat2_band):
  // resident array src_bit -> dst_bit; band2_ok: the executor can run it for
  // this domain (the caller has checked the shape, band2_shape_ok)
  virtual bool band2_ok(Domain& d) = 0;
  virtual Status band2(Domain& d, int src_bit, int dst_bit, int stream) = 0;
  // planes [p0, p0+np) of n tile slots: slots s0.. -> host tiles t0.. (the
  // same planes), and slots -> slots (wavefront)
  virtual Status d2h_planes(Domain& d, int64_t t0, int64_t n, int s0, int64_t p0, int64_t np, int stream) = 0;
  virtual Status copy_planes(Domain& d, int src0, int dst0, int64_t n, int64_t p0, int64_t np, int stream) = 0;
  // planes [p0, p0+np) of n tiles; "packed" = n sub-tiles of np*ty*tx
  // elements back to back starting at a slot
  virtual Status h2d_part(Domain& d, int64_t tile0, int64_t n, int slot0, int64_t p0, int64_t np,
                          int stream) = 0;
  virtual Status d2h_part(Domain& d, int64_t tile0, int64_t n, int packed_slot, int64_t p0,
                          int64_t np, int stream) = 0;
  virtual Status copy_part(Domain& d, int packed_slot, int slot0, int64_t n, int64_t p0, int64_t np,
                           int stream) = 0;
  // host tiles' planes [p0, p0+np) -> packed sub-tiles at a slot
  virtual Status h2d_pack(Domain& d, int64_t tile0, int64_t n, int packed_slot, int64_t p0, int64_t np,
                          int stream) = 0;
  // two-step pass (temporal blocking): same arguments as heat
  virtual Status heat2(Domain& d, const int64_t* tiles, const int* in_slots, const int* out_slots,
                       int nitems, int read_parity, const TileItem* dev_items, int stream) = 0;
  virtual Status extract(Domain& d, int64_t tile0, int64_t ntile, int slot0, int parity,
                         const TileItem* dev_items, int stream) = 0;
  virtual Status faces_h2d(Domain& d, int parity, int stream) = 0;
  // mode (peer transport): 0 = push the faces with copies;
  // 1 = copies, and arm the next exchange, whose data the kernels push
  // (fused); 2 = signal only: the previous step's kernels pushed the data
  virtual Status halo(Domain& d, int parity, int stream, int mode = 0) = 0;
  // multi-rank stream-through (comm_peer.cu): op 0 = push my slab-end T
  // planes of initial data (side 1: top -> upper, 0: bottom -> lower) once the
  // receiver has released the previous run's; 1 = wait until side's halo
  // layer has arrived; 2 = release side's halo layer (read by the first sweep)
  virtual Status st_halo(Domain& d, int op, int side, int T, int stream) = 0;
  virtual Status note(Domain& d, int kind, int64_t a, int64_t b, int stream) = 0;  // trace-only ops
  virtual Status sync_all(Domain& d) = 0;
  // cost-model calibration: *r = one sweep's time per plane / one plane's
  // duplex host-link time, measured on this device (0: not measured)
  virtual Status calibrate(Domain& d, double* r) = 0;
  // resources
  virtual Status mem_info(Domain& d, uint64_t* free_b, uint64_t* total_b) = 0;
  virtual Status alloc_host(Domain& d, uint64_t bytes, void** p) = 0;
  virtual void free_host(Domain& d, void* p) = 0;
  virtual Status alloc_device(Domain& d, uint64_t bytes, void** p) = 0;
  virtual void free_device(Domain& d, void* p) = 0;
  virtual Status setup(Domain& d) = 0;       // streams, events, device tables
  virtual Status upload_dir(Domain& d) = 0;  // Dirichlet fixed faces (sync)
  virtual void destroy(Domain& d) = 0;
  virtual Status timer_start(Domain& d) = 0;
  virtual Status timer_stop(Domain& d, double* ms) = 0;
};

// -------------------------------------------------------------------- domain
enum Mode : int { MODE_RESIDENT = 1, MODE_STREAM = 2 };
constexpr int kMaxProgCtas = 2048;  // progress counters of a persistent multi-step launch

// Fault injection for tests of the error contract (tiles.h conventions):
// TILES_FAULT=<kind>:<n> makes the n-th operation of that kind (counted
// from tile_domain_create) fail through the executor's real error path.
enum FaultKind { FAULT_NONE = 0, FAULT_H2D, FAULT_D2H, FAULT_KERNEL, FAULT_SYNC, FAULT_HOST_ALLOC };
struct Fault {
  int kind = FAULT_NONE;
  int64_t left = 0;  // operations of `kind` still to pass before the failing one
};
Fault parse_fault_env();
bool fault_fires(Domain& d, int kind);  // true once, at the n-th call of `kind`

struct Domain {
  Geometry G;
  tile_options opt;
  Fault fault;
  bool poisoned = false;
  int last_schedule = 0;  // tile_info.last_schedule
  double r_sweep = 0.021;  // cost model: sweep / duplex link time per plane (calibrated at setup)
  // wavefront scratch (allocated at its first use, within the budget):
  // slots [nslots, nslots + wave_slots), whole tile layers
  int wave_slots = 0;
  double* wave_base = nullptr;
  bool own_wave = false;
  uint64_t budget_left = 0;  // device budget not carved by domain_setup
  int device = 0;
  int mode = MODE_RESIDENT;
  int measure = TILE_MEASURE_NORMAL;

  // host (pinned unless dry-run)
  double* host = nullptr;                  // ntiles * tile_elems, tile-blocked
  double* host_faces[6] = {};              // initial faces for STREAM mode
  double* host_dir[6] = {};                // Dirichlet fixed faces
  bool host_faces_valid = false;
  bool dir_uploaded = false;
  uint64_t host_bytes = 0;

  // device (carved from one pool)
  char* pool = nullptr;
  uint64_t pool_bytes = 0;
  bool own_pool = false;
  double* faces[6][2] = {};                // export faces [face][parity]
  double* dir_faces[6] = {};               // Dirichlet fixed faces
  double* halo[2][2] = {};                 // [0 = from below (z-), 1 = from above (z+)][parity]
  const double** gsrc_dev[2] = {};         // [parity] -> ntiles*6 pointers
  // direct ghost sources (resident mode, HeatParams::gdir): [bit][parity]
  // -> ntiles*6 nearest-layer pointers, and ntiles*2 y source z-strides
  const double** gdir_dev[2][2] = {};
  int64_t* ystr_dev = nullptr;
  std::vector<const double*> gdir_host[2][2];
  std::vector<int64_t> ystr_host;
  bool direct_ok = false;                  // single-step resident passes read neighbours directly
  // persistent multi-step launches (HeatParams::nsteps): per-CTA progress
  // counters and the step epoch their values are relative to
  bool persist_ok = false;
  unsigned long long* prog_dev = nullptr;  // [0]: grid barrier arrival counter
  uint32_t prog_epoch = 0;                  // barrier rounds completed by earlier launches
  int64_t prog_grid = 0;                    // grid of the persistent launches (fixed per domain)
  EdgePtr* esrc_dev[2] = {};               // [parity] -> ntiles*12 (D = 2 only)
  std::vector<EdgePtr> esrc_host[2];
  uint8_t* fixed_mask_dev = nullptr;       // per tile: Dirichlet faces (bit f)
  std::vector<uint8_t> fixed_mask_host;
  int64_t st_unit = 0;                     // stream-through unit (planes) of the current run
  int64_t slab_depth = 0;                  // planes per stream-through scratch slab (tile-blocked)
  bool x2_ok = false;                      // two-step passes available
  int band2 = 0, heat2_grid = 0;
  size_t heat2_smem = 0;
  TileItem* items_dev[2] = {};             // resident mode: [bit] -> ntiles items
  double* slot_base = nullptr;
  int nslots = 0;
  uint64_t device_bytes = 0;

  // residency
  std::vector<int> slot_owner;             // tile id or -1
  std::vector<int> tile_slot;              // slot or -1
  std::vector<char> tile_dirty;
  std::vector<int64_t> tile_last_use;
  std::deque<int> free_slots;
  int res_bit = 0;                         // resident mode: 0 -> A current, 1 -> B
  bool resident_valid = false;             // resident mode: all tiles on device
  bool faces_valid = false;                // device faces hold the current state
  bool xfaces_valid = false;               // x faces (and, multi-rank, the slab-end z faces) do:
                                           // what a direct single-step pass reads and leaves
  int face_parity = 0;                     // parity of the current state's faces
  int64_t use_clock = 0;

  // streams / events (ids; CudaExec maps them to CUDA objects)
  int nstreams_max = 64;
  int halo_stream = 64;                    // index of the dedicated halo stream
  int ev_layer_base = 0;                   // 2 per layer
  int ev_tile_base = 0;                    // 2 per tile (face events)
  int ev_slot_base = 0;                    // 1 per slot
  int ev_in_base = 0;                      // 1 per tile / batch (H2D done)
  int ev_host_base = 0;                    // 1 per tile (host copy written)
  int ev_misc_base = 0;                    // faces init, halo[2], done
  int nevents = 0;

  // NCCL
  void* nccl_comm = nullptr;
  // peer transport (comm_peer.cu): own window (halo buffers + counters),
  // the neighbours' windows [0 = lower, 1 = upper], exchange counter
  void* peer_window = nullptr;
  void* peer_flags = nullptr;
  uint64_t peer_halo_bytes = 0;
  void* peer_base[2] = {nullptr, nullptr};
  void* peer_opened[2] = {nullptr, nullptr};
  unsigned int peer_wait_flags = 0;
  uint32_t peer_k = 0;
  bool peer_connected = false;
  bool peer_fused = false;                 // resident direct passes push z halos from the kernel
  // multi-rank stream-through: two tile layers in the window
  // ([0] lo: the lower neighbour's top T planes of initial data, [1] hi: the
  // upper neighbour's bottom T planes), tile-blocked like the resident array
  double* st_halo[2] = {nullptr, nullptr};
  uint64_t st_halo_bytes = 0;              // one layer (0: no multi-rank stream-through)
  uint32_t st_epoch = 0;                   // multi-rank stream-through runs so far
  struct UserFn* user_fn = nullptr;        // TILE_KERNEL_USER run in progress (borrowed)
  int64_t user_box[6] = {0, 0, 0, 0, 0, 0}; // its global cell box [x0,y0,z0; x1,y1,z1)

  // kernel plan
  int band = 0, stages = 0, heat_grid = 0, sm_count = 148;
  size_t heat_smem = 0;
  int heat_cache_flags = 2;               // L2 policy bits (kernels.cuh): exports evict_last

  // run bookkeeping
  struct BatchRec { int64_t L0, L1; int stream, out, ev; };  // ev: last kernel's event
  std::vector<BatchRec> last_batches;      // resident: where each layer's last kernel ran
  double kernel_alpha = 0.125;
  int streams_used = 1;                    // streams touched so far (joined at run start)
  int last_S = 1;
  bool last_serial = false;
  std::vector<const double*> gsrc_host[2]; // [parity] -> ntiles*6
  std::vector<TileItem> items_host[2];

  tile_stats stats{};
  std::vector<tile_op> trace;
  Exec* exec = nullptr;
  bool in_flight = false;
  bool host_pending = false;               // async D2H into the host store in flight (ooc stream-through)
  double run_t0 = 0;
  bool kernel_timing = false;

  double* slot_ptr(int s) const {
    return s < nslots ? slot_base + (int64_t)s * G.tile_elems : wave_base + (int64_t)(s - nslots) * G.tile_elems;
  }
  double* host_tile(int64_t k) const { return host + k * G.tile_elems; }
  const double* face_src_ptr(int64_t id, int f, int parity) const;
  const double* direct_src_ptr(int64_t id, int f, int bit, int parity) const;
  int64_t direct_ystride(int64_t id, int f) const;
  EdgePtr edge_src_ptr(int64_t id, int e, int parity) const;
};

// runtime.cpp
Status domain_create(const int64_t dims[3], const int64_t tdims[3], int ghost,
                     const tile_options* opt, Domain** out);
Status domain_load(Domain& d, const double* src);
Status domain_run(Domain& d, const tile_kernel& k, int steps, int nstreams);
Status domain_sync(Domain& d);
Status domain_store(Domain& d, double* dst);
Status domain_invalidate(Domain& d);
Status domain_host_region(Domain& d, int64_t tile, int mode, double** ptr);
Status domain_host_ghosts(Domain& d, int64_t tile, double* out);
Status domain_host_compute(Domain& d, const int64_t* ids, int64_t n, int mode, int ghosted, tile_host_fn fn,
                           void* ctx);
Status domain_free(Domain* d);
Status domain_setup(Domain& d);
void host_extract_faces(const Geometry& G, const double* host, double* const faces[6]);
void host_parallel_for(int64_t n, const std::function<void(int64_t, int64_t)>& fn);

// executors (exec_cuda.cu / exec_dry.cpp)
Exec* make_cuda_exec(Domain& d, Status* st);
Exec* make_dry_exec();

// comm_nccl.cpp
Status nccl_unique_id(void* out128);
Status nccl_init(Domain& d);
Status nccl_halo(Domain& d, int parity, void* stream);
void nccl_destroy(Domain& d);

// comm_local.cu (in-process transport, tests)
Status local_group_create(int n, void** out);
void local_group_free(void* g);
Status local_halo(Domain& d, int parity, void* stream, void* ready_event);
struct UserFn;  // userfn.cpp
Status userfn_create(const char* source, const char* name, UserFn** out);
void userfn_free(UserFn* f);
Status userfn_create_stencil(const char* source, const char* name, UserFn** out);
bool userfn_is_stencil(const UserFn* f);
Status userfn_launch_stencil(UserFn* f, const void* dev_items, int nitems, const double* in, double* out,
                             int tile, const double* const* gsrc, double* const fexp[6],
                             const int64_t face_elems[6], const int64_t t[3], int depth, void* stream);
Status userfn_launch(UserFn* f, double* data, int64_t n, const int64_t tdims[2], const int64_t org[3],
                     const int64_t gdims[2], int64_t iters, const int64_t box[6], void* stream);
Status peer_setup(Domain& d, uint64_t halo_bytes, uint64_t st_bytes);
Status peer_st_halo(Domain& d, int op, int side, int T, void* stream);
Status peer_handle(const Domain& d, void* out64);
Status peer_connect(Domain& d, const void* handles, int n);
Status peer_halo(Domain& d, int parity, void* stream, int mode);
void peer_destroy(Domain& d);

}  // namespace tiles
