// comm_local.cu — in-process transport for the slab halo exchange (testing
// the multi-rank path on a single GPU). Each rank is a domain driven by its
// own host thread. A halo op is a collective: all ranks rendezvous on the
// host, exchange the addresses of their exported boundary faces and two CUDA
// events, then each rank pulls its ghost planes with device copies on its
// halo stream:
//   ready[r]   recorded after rank r's boundary kernels (RAW on its exports)
//   done[r]    recorded after rank r's pulls of the PREVIOUS generation; a
//              rank's next exchange waits for every peer's done, so a peer's
//              pull completes before the exports it read can be overwritten
//              (exports of parity p are rewritten two steps later, after the
//              next exchange on the writer's own stream order).
#include <condition_variable>
#include <cstdio>
#include <mutex>
#include <vector>

#include "runtime.hpp"

namespace tiles {

struct LocalGroup {
  int n;
  std::mutex m;
  std::condition_variable cv;
  uint64_t gen = 0;      // completed rendezvous generations
  int arrived = 0;
  int departed = 0;
  struct Entry {
    const double* top = nullptr;  // exports of the rank's top layer (z+ faces)
    const double* bot = nullptr;  // exports of the rank's bottom layer (z- faces)
    cudaEvent_t ready = nullptr;
    cudaEvent_t done_prev = nullptr;
  };
  std::vector<Entry> e;
  std::vector<cudaEvent_t> done;  // per rank, recorded after its pulls
  explicit LocalGroup(int nr) : n(nr), e(nr), done(nr, nullptr) {}
};

Status local_group_create(int n, void** out) {
  if (n < 1) return make_err(TILE_EINVAL, "nranks must be >= 1");
  *out = new LocalGroup(n);
  return Status::ok();
}

void local_group_free(void* g) {
  auto* G = static_cast<LocalGroup*>(g);
  if (!G) return;
  for (auto ev : G->done)
    if (ev) cudaEventDestroy(ev);
  delete G;
}

#define LK(call)                                                                        \
  do {                                                                                  \
    cudaError_t e_ = (call);                                                            \
    if (e_ != cudaSuccess) return make_err(TILE_ECUDA, std::string(#call ": ") + cudaGetErrorString(e_)); \
  } while (0)

Status local_halo(Domain& d, int par, void* stream_v, void* ready_ev_v) {
  auto* G = static_cast<LocalGroup*>(d.opt.local_group);
  cudaStream_t st = static_cast<cudaStream_t>(stream_v);
  cudaEvent_t ready = static_cast<cudaEvent_t>(ready_ev_v);
  const Geometry& Gm = d.G;
  const int R = Gm.nranks, r = Gm.rank;
  if (G->n != R) return make_err(TILE_EINVAL, "local group size != nranks");
  const size_t cnt = (size_t)Gm.layer_tiles * Gm.face_elems[ZM];
  std::vector<LocalGroup::Entry> peers;
  {
    std::unique_lock<std::mutex> lk(G->m);
    // wait until the previous generation has fully departed (every peer has
    // issued its waits on this rank's previous `ready` record)
    G->cv.wait(lk, [&] { return G->departed == 0 || G->departed == G->n; });
    if (G->departed == G->n) G->departed = 0;
    if (cudaEventRecord(ready, st) != cudaSuccess) return make_err(TILE_ECUDA, "cudaEventRecord (ready)");
    if (!G->done[r]) {
      cudaError_t e = cudaEventCreateWithFlags(&G->done[r], cudaEventDisableTiming);
      if (e != cudaSuccess) return make_err(TILE_ECUDA, "cudaEventCreate (local group)");
      e = cudaEventRecord(G->done[r], st);
      if (e != cudaSuccess) return make_err(TILE_ECUDA, "cudaEventRecord (local group)");
    }
    G->e[r].top = d.faces[ZP][par] + (Gm.n[2] - 1) * Gm.layer_tiles * Gm.face_elems[ZP];
    G->e[r].bot = d.faces[ZM][par];
    G->e[r].ready = ready;
    G->e[r].done_prev = G->done[r];
    const uint64_t my_gen = G->gen;
    if (++G->arrived == G->n) {
      G->arrived = 0;
      ++G->gen;
      G->cv.notify_all();
    } else {
      G->cv.wait(lk, [&] { return G->gen != my_gen; });
    }
    peers = G->e;  // snapshot of this generation's deposits
    // bind the waits to this generation's records before departing
    for (int q = 0; q < R; ++q) {
      if (q == r) continue;
      if (cudaStreamWaitEvent(st, peers[q].ready, 0) != cudaSuccess ||
          cudaStreamWaitEvent(st, peers[q].done_prev, 0) != cudaSuccess)
        return make_err(TILE_ECUDA, "cudaStreamWaitEvent (local group)");
    }
    ++G->departed;
    G->cv.notify_all();
  }
  const bool per = Gm.bc == TILE_BC_PERIODIC;
  const bool has_up = per || r < R - 1, has_dn = per || r > 0;
  const int up = (r + 1) % R, dn = (r - 1 + R) % R;
  if (d.measure != TILE_MEASURE_COMP_ONLY) {
    if (has_dn)
      LK(cudaMemcpyAsync(d.halo[0][par], peers[dn].top, cnt * 8, cudaMemcpyDeviceToDevice, st));
    if (has_up)
      LK(cudaMemcpyAsync(d.halo[1][par], peers[up].bot, cnt * 8, cudaMemcpyDeviceToDevice, st));
    d.stats.bytes_halo += (uint64_t)((has_up ? 1 : 0) + (has_dn ? 1 : 0)) * cnt * 8;
  }
  LK(cudaEventRecord(G->done[r], st));
  return Status::ok();
}

}  // namespace tiles
