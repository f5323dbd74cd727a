// capi.cpp — the extern "C" boundary declared in include/tiles.h: argument
// validation, error codes, poisoning and the thread-local error message.
#include <chrono>
#include <cstring>
#include <string>

#include "runtime.hpp"

using tiles::Domain;
using tiles::Status;

struct tile_domain {
  Domain* d;
};
struct tile_user_fn {
  tiles::UserFn* f;
};

namespace {
thread_local std::string g_err = "no error";

tile_status finish(tile_domain* h, const Status& s) {
  if (s.bad()) {
    g_err = s.msg;
    if (h && h->d && (s.code == TILE_ECUDA || s.code == TILE_ENCCL)) h->d->poisoned = true;
  }
  return s.code;
}
tile_status fail(tile_status c, const char* m) {
  g_err = m;
  return c;
}
#define CHECK_DOM(h)                                                      \
  do {                                                                    \
    if (!(h) || !(h)->d) return fail(TILE_EINVAL, "null domain");         \
    if ((h)->d->poisoned) return fail(TILE_ESTATE, "domain poisoned by an earlier CUDA/NCCL error"); \
  } while (0)
}  // namespace

extern "C" {

const char* tile_last_error(void) { return g_err.c_str(); }
const char* tile_version(void) { return "tiles-b200 0.1 (sm_100a)"; }

tile_status tile_domain_create(const int64_t dims[3], const int64_t tile_dims[3], int32_t ghost,
                               const tile_options* opt, tile_domain** out) {
  if (!dims || !tile_dims || !out) return fail(TILE_EINVAL, "null argument");
  *out = nullptr;
  Domain* d = nullptr;
  Status s = tiles::domain_create(dims, tile_dims, ghost, opt, &d);
  if (s.bad()) return finish(nullptr, s);
  *out = new tile_domain{d};
  return TILE_OK;
}

tile_status tile_load(tile_domain* h, const double* src) {
  CHECK_DOM(h);
  if (!src) return fail(TILE_EINVAL, "null src");
  return finish(h, tiles::domain_load(*h->d, src));
}

tile_status tile_host_tile(tile_domain* h, int64_t tile_id, double** ptr) {
  CHECK_DOM(h);
  if (!ptr || tile_id < 0 || tile_id >= h->d->G.ntiles) return fail(TILE_EINVAL, "bad tile id");
  *ptr = h->d->host_tile(tile_id);
  return TILE_OK;
}

tile_status tile_host_region(tile_domain* h, int64_t tile_id, int32_t mode, double** ptr) {
  CHECK_DOM(h);
  if (!ptr || tile_id < 0 || tile_id >= h->d->G.ntiles) return fail(TILE_EINVAL, "bad tile id");
  if (mode != TILE_HOST_READ && mode != TILE_HOST_WRITE) return fail(TILE_EINVAL, "bad host mode");
  return finish(h, tiles::domain_host_region(*h->d, tile_id, mode, ptr));
}

tile_status tile_host_ghosts(tile_domain* h, int64_t tile_id, double* out, int64_t out_len) {
  CHECK_DOM(h);
  const tiles::Geometry& G = h->d->G;
  if (!out || tile_id < 0 || tile_id >= G.ntiles) return fail(TILE_EINVAL, "bad tile id or out");
  const int64_t need = (G.t[0] + 2 * G.ghost) * (G.t[1] + 2 * G.ghost) * (G.t[2] + 2 * G.ghost);
  if (out_len < need) return fail(TILE_EINVAL, "out_len too small");
  return finish(h, tiles::domain_host_ghosts(*h->d, tile_id, out));
}

tile_status tile_host_compute(tile_domain* h, const int64_t* ids, int64_t n, int32_t mode, int32_t ghosted,
                              tile_host_fn fn, void* ctx) {
  CHECK_DOM(h);
  const tiles::Geometry& G = h->d->G;
  if (!fn || n < 0 || (n > 0 && !ids)) return fail(TILE_EINVAL, "null fn, n < 0 or null ids");
  if (mode != TILE_HOST_READ && mode != TILE_HOST_WRITE) return fail(TILE_EINVAL, "bad host mode");
  for (int64_t i = 0; ids && i < n; ++i)
    if (ids[i] < 0 || ids[i] >= G.ntiles) return fail(TILE_EINVAL, "bad tile id");
  if (ghosted && G.nranks > 1)
    for (int64_t i = 0; i < (ids ? n : G.ntiles); ++i) {
      int64_t c[3];
      G.tile_coords(ids ? ids[i] : i, &c[0], &c[1], &c[2]);
      const bool lo = c[2] == 0 && (G.bc == TILE_BC_PERIODIC || G.rank > 0);
      const bool hi = c[2] == G.n[2] - 1 && (G.bc == TILE_BC_PERIODIC || G.rank < G.nranks - 1);
      if (lo || hi) return fail(TILE_EINVAL, "ghost cells of a listed tile live on another rank");
    }
  return finish(h, tiles::domain_host_compute(*h->d, ids, ids ? n : G.ntiles, mode, ghosted, fn, ctx));
}

tile_status tile_mark_host_dirty(tile_domain* h) {
  CHECK_DOM(h);
  Domain& d = *h->d;
  if (d.in_flight) {
    Status s = tiles::domain_sync(d);
    if (s.bad()) return finish(h, s);
  }
  d.host_faces_valid = false;
  for (auto& x : d.tile_dirty) x = 0;
  return finish(h, tiles::domain_invalidate(d));
}

tile_status tile_run(tile_domain* h, const tile_kernel* k, int32_t steps, int32_t nstreams) {
  CHECK_DOM(h);
  if (!k) return fail(TILE_EINVAL, "null kernel");
  auto t0 = std::chrono::steady_clock::now();
  // USER kernels: the function is read while this call enqueues the launches
  h->d->user_fn = (k->kind == TILE_KERNEL_USER || k->kind == TILE_KERNEL_USER_STENCIL) && k->user
                      ? k->user->f : nullptr;
  if (h->d->user_fn && tiles::userfn_is_stencil(h->d->user_fn) != (k->kind == TILE_KERNEL_USER_STENCIL)) {
    h->d->user_fn = nullptr;
    return fail(TILE_EINVAL, "user function kind does not match the kernel kind (pointwise vs stencil)");
  }
  if (h->d->user_fn && k->kind == TILE_KERNEL_USER) {
    const tiles::Geometry& G = h->d->G;
    const int64_t all[6] = {0, 0, 0, G.g[0], G.g[1], G.g[2]};
    const int64_t* b = k->box ? k->box : all;
    for (int a = 0; a < 3; ++a)
      if (b[a] > b[3 + a]) {
        h->d->user_fn = nullptr;
        return fail(TILE_EINVAL, "kernel box: lo > hi");
      }
    for (int i = 0; i < 6; ++i) h->d->user_box[i] = b[i];
  }
  Status s = tiles::domain_run(*h->d, *k, steps, nstreams);
  h->d->user_fn = nullptr;
  h->d->run_t0 = std::chrono::duration<double, std::milli>(t0.time_since_epoch()).count();
  return finish(h, s);
}

tile_status tile_sync(tile_domain* h) {
  CHECK_DOM(h);
  Status s = tiles::domain_sync(*h->d);
  if (!s.bad() && h->d->run_t0 > 0) {
    double now = std::chrono::duration<double, std::milli>(
                     std::chrono::steady_clock::now().time_since_epoch())
                     .count();
    h->d->stats.last_run_ms = now - h->d->run_t0;
    h->d->run_t0 = 0;
  }
  return finish(h, s);
}

tile_status tile_store(tile_domain* h, double* dst) {
  CHECK_DOM(h);
  if (!dst) return fail(TILE_EINVAL, "null dst");
  return finish(h, tiles::domain_store(*h->d, dst));
}

tile_status tile_invalidate(tile_domain* h) {
  CHECK_DOM(h);
  return finish(h, tiles::domain_invalidate(*h->d));
}

tile_status tile_ghost_map(const tile_domain* h, int64_t tile_id, int64_t* out, int64_t out_len) {
  CHECK_DOM(h);
  const tiles::Geometry& G = h->d->G;
  if (!out || tile_id < 0 || tile_id >= G.ntiles) return fail(TILE_EINVAL, "bad tile id or out");
  const int64_t need = (G.t[0] + 2 * G.ghost) * (G.t[1] + 2 * G.ghost) * (G.t[2] + 2 * G.ghost);
  if (out_len < need) return fail(TILE_EINVAL, "out_len too small");
  tiles::ghost_map(G, tile_id, out);
  return TILE_OK;
}

tile_status tile_face_sources(const tile_domain* h, int64_t tile_id, int64_t out[12]) {
  CHECK_DOM(h);
  if (!out || tile_id < 0 || tile_id >= h->d->G.ntiles) return fail(TILE_EINVAL, "bad tile id");
  for (int f = 0; f < 6; ++f) {
    tiles::FaceSrc s = tiles::face_source(h->d->G, tile_id, f);
    out[2 * f] = s.kind;
    out[2 * f + 1] = s.val;
  }
  return TILE_OK;
}

tile_status tile_get_info(const tile_domain* h, tile_info* o) {
  CHECK_DOM(h);
  if (!o) return fail(TILE_EINVAL, "null argument");
  const Domain& d = *h->d;
  std::memset(o, 0, sizeof *o);
  for (int a = 0; a < 3; ++a) {
    o->dims[a] = d.G.g[a];
    o->local_dims[a] = d.G.l[a];
    o->tile_dims[a] = d.G.t[a];
    o->tiles[a] = d.G.n[a];
  }
  o->ntiles = d.G.ntiles;
  o->z_offset = d.G.zoff;
  o->ghost = d.G.ghost;
  o->nslots = d.nslots;
  o->sched = d.opt.sched == TILE_SCHED_SYNC ? TILE_SCHED_SYNC
             : d.mode == tiles::MODE_RESIDENT ? TILE_SCHED_RESIDENT
                                               : TILE_SCHED_STREAM;
  o->resident = d.resident_valid ? 1 : 0;
  o->device_bytes = d.device_bytes;
  o->host_bytes = d.host_bytes;
  o->steps_per_pass = d.x2_ok && (d.opt.two_step > 0 || d.mode == tiles::MODE_STREAM) ? 2 : 1;
  o->last_schedule = d.last_schedule;
  o->sweep_link_ratio = d.r_sweep;
  return TILE_OK;
}

tile_status tile_get_stats(const tile_domain* h, tile_stats* o) {
  CHECK_DOM(h);
  if (!o) return fail(TILE_EINVAL, "null argument");
  *o = h->d->stats;
  return TILE_OK;
}

tile_status tile_reset_stats(tile_domain* h) {
  CHECK_DOM(h);
  h->d->stats = tile_stats{};
  return TILE_OK;
}

tile_status tile_set_measure(tile_domain* h, int32_t mode) {
  CHECK_DOM(h);
  if (mode < TILE_MEASURE_NORMAL || mode > TILE_MEASURE_COMP_ONLY)
    return fail(TILE_EINVAL, "bad measure mode");
  h->d->measure = mode;
  return TILE_OK;
}

tile_status tile_timer_start(tile_domain* h) {
  CHECK_DOM(h);
  return finish(h, h->d->exec->timer_start(*h->d));
}

tile_status tile_timer_stop(tile_domain* h, double* ms) {
  CHECK_DOM(h);
  if (!ms) return fail(TILE_EINVAL, "null ms");
  Status s = h->d->exec->timer_stop(*h->d, ms);
  if (!s.bad()) h->d->in_flight = false;
  return finish(h, s);
}

tile_status tile_set_kernel_timing(tile_domain* h, int32_t on) {
  CHECK_DOM(h);
  h->d->kernel_timing = on != 0;
  return TILE_OK;
}

tile_status tile_trace(const tile_domain* h, tile_op* out, int64_t cap, int64_t* n) {
  CHECK_DOM(h);
  if (!n) return fail(TILE_EINVAL, "null argument");
  const auto& t = h->d->trace;
  *n = (int64_t)t.size();
  if (out && cap > 0) std::memcpy(out, t.data(), sizeof(tile_op) * (size_t)std::min<int64_t>(cap, *n));
  return TILE_OK;
}

tile_status tile_trace_clear(tile_domain* h) {
  CHECK_DOM(h);
  h->d->trace.clear();
  return TILE_OK;
}

tile_status tile_free(tile_domain* h) {
  if (!h) return TILE_OK;
  Status s = tiles::domain_free(h->d);
  delete h;
  if (s.bad()) g_err = s.msg;
  return s.code;
}

tile_status tile_local_group_create(int32_t nranks, void** group) {
  if (!group) return fail(TILE_EINVAL, "null group");
  return finish(nullptr, tiles::local_group_create(nranks, group));
}

tile_status tile_local_group_free(void* group) {
  tiles::local_group_free(group);
  return TILE_OK;
}

tile_status tile_user_fn_create(const char* source, const char* name, tile_user_fn** out) {
  if (!out) return fail(TILE_EINVAL, "null out");
  *out = nullptr;
  tiles::UserFn* f = nullptr;
  Status s = tiles::userfn_create(source, name, &f);
  if (s.bad()) return finish(nullptr, s);
  *out = new tile_user_fn{f};
  return TILE_OK;
}

tile_status tile_user_stencil_create(const char* source, const char* name, tile_user_fn** out) {
  if (!out) return fail(TILE_EINVAL, "null out");
  *out = nullptr;
  tiles::UserFn* f = nullptr;
  Status s = tiles::userfn_create_stencil(source, name, &f);
  if (s.bad()) return finish(nullptr, s);
  *out = new tile_user_fn{f};
  return TILE_OK;
}

tile_status tile_user_fn_free(tile_user_fn* fn) {
  if (!fn) return TILE_OK;
  tiles::userfn_free(fn->f);
  delete fn;
  return TILE_OK;
}

tile_status tile_nccl_unique_id(void* out128) {
  if (!out128) return fail(TILE_EINVAL, "null out");
  return finish(nullptr, tiles::nccl_unique_id(out128));
}

tile_status tile_peer_handle(const tile_domain* h, void* out64) {
  CHECK_DOM(h);
  if (!out64) return fail(TILE_EINVAL, "null argument");
  return finish(nullptr, tiles::peer_handle(*h->d, out64));
}

tile_status tile_peer_connect(tile_domain* h, const void* handles, int32_t nranks) {
  CHECK_DOM(h);
  if (!handles) return fail(TILE_EINVAL, "null handles");
  return finish(h, tiles::peer_connect(*h->d, handles, nranks));
}

}  // extern "C"
