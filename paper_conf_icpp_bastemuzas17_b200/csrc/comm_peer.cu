// comm_peer.cu — z-slab halo exchange by direct stores into the neighbour
// ranks' device memory (CUDA IPC; over NVLink 5 / NVSwitch between the GPUs
// of a node), without NCCL. Not in the paper (single GPU).
//
// Each rank owns a "window" (one cudaMalloc, exported with cudaIpcGetMemHandle):
// its receive buffers halo[2][2] and four 32-bit counters. Exchange k (the
// k-th halo op, identical on every rank: the op is collective) of parity p,
// on the rank's halo stream, which is already ordered after the boundary
// kernels that wrote the exported faces and after the previous readers of
// halo[.][p]:
//   1. ready:   write k into the upper neighbour's R_DN and the lower one's
//               R_UP (my halo[.][p] may now be overwritten);
//   2. wait:    my R_UP >= k and my R_DN >= k (my receivers are ready);
//   3. push:    my top z-faces -> upper.halo[0][p], bottom -> lower.halo[1][p]
//               (peer-to-peer copies);
//   4. arrived: write k into upper.A_DN and lower.A_UP (after the copies:
//               cuStreamWriteValue32 fences prior work of the stream);
//   5. wait:    my A_DN >= k and my A_UP >= k, then the caller records the
//               halo event its boundary kernels wait for.
// This is the rendezvous an NCCL send/recv pair provides, without a proxy
// thread or a staging copy.
// Fused mode (tile_options.peer_transport = 2, resident direct passes): the
// stencil kernel itself stores its slab-end z layers into the neighbours'
// windows (HeatParams::zpush_*), so the exchange after step s only signals:
//   mode 2 (op k): A := k at the neighbours (this step's kernels, which the
//   halo stream follows, have pushed), R := k+1 (my step-s kernels no longer
//   read the buffers the neighbours' next kernels will push into); wait my
//   A >= k and R >= k+1. The first exchange of a run (mode 1) is the copy
//   exchange above plus the R := k+1 arming for the first fused push.
// Multi-rank stream-through (peer_st_halo): the trapezoid of T
// steps over a rank's z-slab needs the T planes of INITIAL data beyond each
// slab end, once per run, and no exchange after that. Run e (d.st_epoch, the
// same on every rank: runs are collective), on the rank's halo stream once
// the H2D of its slab-end unit has landed: wait until the receiver released
// run e-1's layer (CR_UP / CR_DN >= e-1), copy the T planes of every tile of
// the slab-end layer into the receiver's halo layer (top -> upper.st_lo,
// bottom -> lower.st_hi), then S_LO / S_HI := e at the receiver. The receiver's
// compute stream waits S >= e before the first sweep of its unit 0 / U-1,
// which reads the halo layer in place of the periodic wrap, and writes
// CR := e at the sender after that sweep.
// Counters are stream memory operations (cuStreamWriteValue32 /
// cuStreamWaitValue32, fetched with cudaGetDriverEntryPoint), so no kernel
// spins and no SM is held.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstdio>
#include <cstring>

#include "runtime.hpp"

namespace tiles {
namespace {

enum { R_DN = 0, R_UP = 1, A_DN = 2, A_UP = 3, S_LO = 4, S_HI = 5, CR_UP = 6, CR_DN = 7, NFLAGS = 8 };
constexpr uint64_t kFlagBytes = 256;

using WriteFn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
using WaitFn = CUresult (*)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
WriteFn g_write = nullptr;
WaitFn g_wait = nullptr;

Status load_memops() {
  if (g_write && g_wait) return Status::ok();
  void* w = nullptr;
  void* v = nullptr;
  cudaDriverEntryPointQueryResult q1{}, q2{};
  if (cudaGetDriverEntryPoint("cuStreamWriteValue32", &w, cudaEnableDefault, &q1) != cudaSuccess ||
      cudaGetDriverEntryPoint("cuStreamWaitValue32", &v, cudaEnableDefault, &q2) != cudaSuccess || !w || !v)
    return make_err(TILE_ENOSYS, "cuStreamWriteValue32/cuStreamWaitValue32 not available");
  g_write = reinterpret_cast<WriteFn>(w);
  g_wait = reinterpret_cast<WaitFn>(v);
  return Status::ok();
}

#define PK(call)                                                                         \
  do {                                                                                   \
    cudaError_t e_ = (call);                                                             \
    if (e_ != cudaSuccess) return make_err(TILE_ECUDA, std::string(#call ": ") + cudaGetErrorString(e_)); \
  } while (0)
#define DK(call)                                                            \
  do {                                                                      \
    CUresult e_ = (call);                                                   \
    if (e_ != CUDA_SUCCESS) return make_err(TILE_ECUDA, std::string(#call " failed")); \
  } while (0)

CUdeviceptr flag(void* window_flags, int i) {
  return reinterpret_cast<CUdeviceptr>(static_cast<uint32_t*>(window_flags) + i);
}

}  // namespace

// Window: [halo 0/1][parity 0/1] receive buffers, the counters, then the two
// stream-through halo layers (st_bytes each; 0 = none).
Status peer_setup(Domain& d, uint64_t halo_bytes, uint64_t st_bytes) {
  Status s = load_memops();
  if (s.bad()) return s;
  const uint64_t bytes = 4 * halo_bytes + kFlagBytes + 2 * st_bytes;
  void* w = nullptr;
  PK(cudaMalloc(&w, bytes));
  PK(cudaMemset(w, 0, bytes));
  PK(cudaDeviceSynchronize());
  d.peer_window = w;
  char* c = static_cast<char*>(w);
  for (int a = 0; a < 2; ++a)
    for (int p = 0; p < 2; ++p) d.halo[a][p] = reinterpret_cast<double*>(c + (2 * a + p) * halo_bytes);
  d.peer_flags = c + 4 * halo_bytes;
  d.peer_halo_bytes = halo_bytes;
  d.st_halo_bytes = st_bytes;
  for (int a = 0; a < 2; ++a)
    d.st_halo[a] = st_bytes ? reinterpret_cast<double*>(c + 4 * halo_bytes + kFlagBytes + a * st_bytes) : nullptr;
  int flush = 0, dev = 0;
  PK(cudaGetDevice(&dev));
  // CU_DEVICE_ATTRIBUTE_CAN_FLUSH_REMOTE_WRITES: needed to make the peers'
  // copies visible to work after a satisfied wait
  PK(cudaDeviceGetAttribute(&flush, cudaDevAttrCanFlushRemoteWrites, dev));
  d.peer_wait_flags = CU_STREAM_WAIT_VALUE_GEQ | (flush ? CU_STREAM_WAIT_VALUE_FLUSH : 0);
  return Status::ok();
}

Status peer_handle(const Domain& d, void* out64) {
  if (!d.peer_window) return make_err(TILE_ESTATE, "no peer window (peer_transport off or dry run)");
  cudaIpcMemHandle_t h;
  PK(cudaIpcGetMemHandle(&h, d.peer_window));
  static_assert(sizeof h == 64, "cudaIpcMemHandle_t is 64 bytes");
  std::memcpy(out64, &h, sizeof h);
  return Status::ok();
}

Status peer_connect(Domain& d, const void* handles, int n) {
  const Geometry& G = d.G;
  if (n != G.nranks) return make_err(TILE_EINVAL, "peer_connect: handle count != nranks");
  if (!d.peer_window) return make_err(TILE_ESTATE, "no peer window (peer_transport off or dry run)");
  const int r = G.rank, R = G.nranks;
  const bool per = G.bc == TILE_BC_PERIODIC;
  const int nb[2] = {(r - 1 + R) % R, (r + 1) % R};  // lower, upper
  const bool has[2] = {per || r > 0, per || r < R - 1};
  for (int s = 0; s < 2; ++s) {
    d.peer_base[s] = nullptr;
    if (!has[s]) continue;
    const int q = nb[s];
    if (q == r) return make_err(TILE_EINVAL, "peer_connect: a rank cannot be its own neighbour");
    if (s == 1 && nb[1] == nb[0] && d.peer_base[0]) {  // G == 2: one peer for both sides
      d.peer_base[1] = d.peer_base[0];
      continue;
    }
    cudaIpcMemHandle_t h;
    std::memcpy(&h, static_cast<const char*>(handles) + (size_t)q * 64, 64);
    void* p = nullptr;
    PK(cudaIpcOpenMemHandle(&p, h, cudaIpcMemLazyEnablePeerAccess));
    d.peer_base[s] = p;
    d.peer_opened[s] = p;
  }
  d.peer_connected = true;
  return Status::ok();
}

void peer_destroy(Domain& d) {
  for (int s = 0; s < 2; ++s) {
    if (d.peer_opened[s]) cudaIpcCloseMemHandle(d.peer_opened[s]);
    d.peer_opened[s] = nullptr;
    d.peer_base[s] = nullptr;
  }
  if (d.peer_window) cudaFree(d.peer_window);
  d.peer_window = nullptr;
}

Status peer_halo(Domain& d, int par, void* stream_v, int mode) {
  if (!d.peer_connected) return make_err(TILE_ESTATE, "peer transport: call tile_peer_connect first");
  const Geometry& G = d.G;
  CUstream st = static_cast<CUstream>(stream_v);
  const uint32_t k = ++d.peer_k;
  const uint64_t hb = d.peer_halo_bytes;
  const size_t cnt = (size_t)G.layer_tiles * G.face_elems[ZM];
  char* lo = static_cast<char*>(d.peer_base[0]);  // lower neighbour's window
  char* up = static_cast<char*>(d.peer_base[1]);  // upper neighbour's window
  void* lo_flags = lo ? lo + 4 * hb : nullptr;
  void* up_flags = up ? up + 4 * hb : nullptr;
  if (mode == 2) {  // signal only: the kernels of this step pushed the data
    if (up) DK(g_write(st, flag(up_flags, A_DN), k, 0));
    if (lo) DK(g_write(st, flag(lo_flags, A_UP), k, 0));
    if (up) DK(g_write(st, flag(up_flags, R_DN), k + 1, 0));
    if (lo) DK(g_write(st, flag(lo_flags, R_UP), k + 1, 0));
    if (lo) DK(g_wait(st, flag(d.peer_flags, A_DN), k, d.peer_wait_flags));
    if (up) DK(g_wait(st, flag(d.peer_flags, A_UP), k, d.peer_wait_flags));
    if (up) DK(g_wait(st, flag(d.peer_flags, R_UP), k + 1, d.peer_wait_flags));
    if (lo) DK(g_wait(st, flag(d.peer_flags, R_DN), k + 1, d.peer_wait_flags));
    const size_t cnt = (size_t)d.G.layer_tiles * d.G.face_elems[ZM];
    if (d.measure != TILE_MEASURE_COMP_ONLY)
      d.stats.bytes_halo += (uint64_t)((up ? 1 : 0) + (lo ? 1 : 0)) * cnt * 8;
    return Status::ok();
  }
  // 1. ready to receive exchange k
  if (up) DK(g_write(st, flag(up_flags, R_DN), k, 0));
  if (lo) DK(g_write(st, flag(lo_flags, R_UP), k, 0));
  // 2. receivers ready
  if (up) DK(g_wait(st, flag(d.peer_flags, R_UP), k, d.peer_wait_flags));
  if (lo) DK(g_wait(st, flag(d.peer_flags, R_DN), k, d.peer_wait_flags));
  // 3. push the boundary faces of parity par, 4. signal arrival
  if (d.measure != TILE_MEASURE_COMP_ONLY) {
    const double* top = d.faces[ZP][par] + (G.n[2] - 1) * G.layer_tiles * G.face_elems[ZP];
    const double* bot = d.faces[ZM][par];
    if (up) PK(cudaMemcpyAsync(up + (0 * 2 + par) * hb, top, cnt * 8, cudaMemcpyDeviceToDevice, (cudaStream_t)st));
    if (lo) PK(cudaMemcpyAsync(lo + (1 * 2 + par) * hb, bot, cnt * 8, cudaMemcpyDeviceToDevice, (cudaStream_t)st));
    d.stats.bytes_halo += (uint64_t)((up ? 1 : 0) + (lo ? 1 : 0)) * cnt * 8;
  }
  if (up) DK(g_write(st, flag(up_flags, A_DN), k, 0));
  if (lo) DK(g_write(st, flag(lo_flags, A_UP), k, 0));
  if (mode == 1) {  // arm the first fused push: nothing reads the other parity yet
    if (up) DK(g_write(st, flag(up_flags, R_DN), k + 1, 0));
    if (lo) DK(g_write(st, flag(lo_flags, R_UP), k + 1, 0));
  }
  // 5. my ghosts have arrived
  if (lo) DK(g_wait(st, flag(d.peer_flags, A_DN), k, d.peer_wait_flags));
  if (up) DK(g_wait(st, flag(d.peer_flags, A_UP), k, d.peer_wait_flags));
  if (mode == 1) {
    if (up) DK(g_wait(st, flag(d.peer_flags, R_UP), k + 1, d.peer_wait_flags));
    if (lo) DK(g_wait(st, flag(d.peer_flags, R_DN), k + 1, d.peer_wait_flags));
  }
  return Status::ok();
}

Status peer_st_halo(Domain& d, int op, int side, int T, void* stream_v) {
  if (!d.peer_connected) return make_err(TILE_ESTATE, "peer transport: call tile_peer_connect first");
  if (!d.st_halo_bytes) return make_err(TILE_ESTATE, "no stream-through halo layers in the window");
  const Geometry& G = d.G;
  CUstream st = static_cast<CUstream>(stream_v);
  const uint32_t e = d.st_epoch;
  const uint64_t hb = d.peer_halo_bytes;
  char* nb = static_cast<char*>(d.peer_base[side]);  // side 0: lower, 1: upper neighbour
  if (!nb) return make_err(TILE_EINVAL, "stream-through halo: no neighbour on that side");
  void* nb_flags = nb + 4 * hb;
  if (op == 0) {  // push my slab-end planes to the neighbour on `side`
    DK(g_wait(st, flag(d.peer_flags, side ? CR_UP : CR_DN), e - 1, d.peer_wait_flags));
    if (d.measure != TILE_MEASURE_COMP_ONLY) {
      const size_t plane = (size_t)G.t[0] * G.t[1], te = (size_t)G.tile_elems;
      const int64_t layer = side ? G.n[2] - 1 : 0;
      const size_t p0 = side ? (size_t)(G.t[2] - T) : 0;  // first plane within the tiles
      const double* src = d.slot_ptr(d.res_bit ? (int)G.ntiles : 0) + (size_t)layer * G.layer_tiles * te + p0 * plane;
      char* dst = nb + 4 * hb + kFlagBytes + (side ? 0 : 1) * d.st_halo_bytes + p0 * plane * 8;
      PK(cudaMemcpy2DAsync(dst, te * 8, src, te * 8, (size_t)T * plane * 8, (size_t)G.layer_tiles,
                           cudaMemcpyDeviceToDevice, (cudaStream_t)st));
      d.stats.bytes_halo += (uint64_t)G.layer_tiles * T * plane * 8;
    }
    DK(g_write(st, flag(nb_flags, side ? S_LO : S_HI), e, 0));
    return Status::ok();
  }
  if (op == 1) {  // my halo layer on `side` has arrived
    DK(g_wait(st, flag(d.peer_flags, side ? S_HI : S_LO), e, d.peer_wait_flags));
    return Status::ok();
  }
  // op 2: my halo layer on `side` has been read: its sender may overwrite it
  DK(g_write(st, flag(nb_flags, side ? CR_DN : CR_UP), e, 0));
  return Status::ok();
}

}  // namespace tiles
