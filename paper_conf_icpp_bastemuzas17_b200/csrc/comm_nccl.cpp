// comm_nccl.cpp — z-slab halo exchange between GPUs through NCCL p2p
// (NVLink 5 / NVSwitch on a B200 node). Not in the paper (single GPU); the
// north star adds it: each rank owns a z-slab, and per step the boundary
// z-faces travel to the z-neighbour ranks.
//
// NCCL is loaded with dlopen (the copy PyTorch ships, or the system one), so
// the library itself has no link-time NCCL dependency and single-GPU use
// never touches it.
#include <dlfcn.h>

#include <cstdio>
#include <cstring>

#include <cuda_runtime.h>
#include <nccl.h>

#include "runtime.hpp"

namespace tiles {
namespace {

struct NcclApi {
  void* h = nullptr;
  ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
  ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
  ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
  ncclResult_t (*Send)(const void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*Recv)(void*, size_t, ncclDataType_t, int, ncclComm_t, cudaStream_t) = nullptr;
  ncclResult_t (*GroupStart)() = nullptr;
  ncclResult_t (*GroupEnd)() = nullptr;
  const char* (*GetErrorString)(ncclResult_t) = nullptr;
};

NcclApi g_api;

Status load_nccl() {
  if (g_api.h) return Status::ok();
  const char* names[] = {"libnccl.so.2", "libnccl.so", nullptr};
  void* h = nullptr;
  // prefer an already-loaded copy (e.g. torch's) over loading a second one
  for (int i = 0; names[i] && !h; ++i) h = dlopen(names[i], RTLD_NOW | RTLD_GLOBAL | RTLD_NOLOAD);
  if (const char* p = std::getenv("TILES_NCCL_PATH")) {
    if (!h) h = dlopen(p, RTLD_NOW | RTLD_GLOBAL);
  }
  for (int i = 0; names[i] && !h; ++i) h = dlopen(names[i], RTLD_NOW | RTLD_GLOBAL);
  if (!h) return make_err(TILE_ENOSYS, "libnccl.so.2 not found (import torch first or set TILES_NCCL_PATH)");
  NcclApi a;
  a.h = h;
#define SYM(field, name)                                              \
  a.field = reinterpret_cast<decltype(a.field)>(dlsym(h, name));      \
  if (!a.field) return make_err(TILE_ENOSYS, "NCCL symbol missing: " name);
  SYM(GetUniqueId, "ncclGetUniqueId");
  SYM(CommInitRank, "ncclCommInitRank");
  SYM(CommDestroy, "ncclCommDestroy");
  SYM(Send, "ncclSend");
  SYM(Recv, "ncclRecv");
  SYM(GroupStart, "ncclGroupStart");
  SYM(GroupEnd, "ncclGroupEnd");
  SYM(GetErrorString, "ncclGetErrorString");
#undef SYM
  g_api = a;
  return Status::ok();
}

Status nccl_err(ncclResult_t r, const char* what) {
  char buf[256];
  std::snprintf(buf, sizeof buf, "%s: %s", what, g_api.GetErrorString ? g_api.GetErrorString(r) : "?");
  return make_err(TILE_ENCCL, buf);
}
#define NK(call)                                      \
  do {                                                \
    ncclResult_t r_ = (call);                         \
    if (r_ != ncclSuccess) return nccl_err(r_, #call); \
  } while (0)

}  // namespace

Status nccl_unique_id(void* out128) {
  Status s = load_nccl();
  if (s.bad()) return s;
  ncclUniqueId id;
  NK(g_api.GetUniqueId(&id));
  std::memcpy(out128, &id, sizeof id);
  return Status::ok();
}

Status nccl_init(Domain& d) {
  Status s = load_nccl();
  if (s.bad()) return s;
  ncclUniqueId id;
  std::memcpy(&id, d.opt.nccl_unique_id, sizeof id);
  ncclComm_t comm = nullptr;
  NK(g_api.CommInitRank(&comm, d.G.nranks, id, d.G.rank));
  d.nccl_comm = comm;
  return Status::ok();
}

// Exchange the boundary z-faces of parity `par`:
//   my top layer's z+ exports  -> rank above's halo[0] (its z- ghosts)
//   my bottom layer's z- exports -> rank below's halo[1] (its z+ ghosts)
// Periodic: ring. Dirichlet: rank 0 has no lower and rank G-1 no upper
// neighbour. Sends are issued before receives so that with G == 2 (the two
// neighbours are the same rank) messages pair up in order: top -> halo[0],
// bottom -> halo[1].
Status nccl_halo(Domain& d, int par, void* stream_v) {
  const Geometry& G = d.G;
  cudaStream_t st = static_cast<cudaStream_t>(stream_v);
  ncclComm_t comm = static_cast<ncclComm_t>(d.nccl_comm);
  const int R = G.nranks, r = G.rank;
  const bool per = G.bc == TILE_BC_PERIODIC;
  const bool has_up = per || r < R - 1;
  const bool has_dn = per || r > 0;
  const int up = (r + 1) % R, dn = (r - 1 + R) % R;
  const size_t cnt = (size_t)G.layer_tiles * G.face_elems[ZM];
  const double* top = d.faces[ZP][par] + (G.n[2] - 1) * G.layer_tiles * G.face_elems[ZP];
  const double* bot = d.faces[ZM][par];
  if (d.measure == TILE_MEASURE_COMP_ONLY) return Status::ok();
  NK(g_api.GroupStart());
  if (has_up) NK(g_api.Send(top, cnt, ncclFloat64, up, comm, st));
  if (has_dn) NK(g_api.Send(bot, cnt, ncclFloat64, dn, comm, st));
  if (has_dn) NK(g_api.Recv(d.halo[0][par], cnt, ncclFloat64, dn, comm, st));
  if (has_up) NK(g_api.Recv(d.halo[1][par], cnt, ncclFloat64, up, comm, st));
  NK(g_api.GroupEnd());
  d.stats.bytes_halo += (uint64_t)((has_up ? 1 : 0) + (has_dn ? 1 : 0)) * cnt * 8;
  return Status::ok();
}

void nccl_destroy(Domain& d) {
  if (d.nccl_comm && g_api.CommDestroy) g_api.CommDestroy(static_cast<ncclComm_t>(d.nccl_comm));
  d.nccl_comm = nullptr;
}

}  // namespace tiles
