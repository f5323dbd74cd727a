// runtime.cpp — domain lifecycle and the tile scheduler (host C++).
//
// Paper mechanisms and where they live here:
//   allocation policy, "as many regions as fit" -> domain_create
//   pinned host regions                                 -> host store
//   one stream per device buffer, async H2D, no sync -> run_*
//   cache list with -1 = free, D2H(owner) before reuse -> acquire()
//   ghost update on the device                           -> fused into
//     heat7 (faces), ordered by per-tile / per-layer events instead of the
//     paper's global `acc wait` (difference D3)
//   D2H + synchronize before host access          -> domain_sync
#include <algorithm>
#include <cmath>
#include <cstdlib>
#include <cstring>
#include <set>

#include "runtime.hpp"

namespace tiles {

namespace {

constexpr uint64_t kReserveBytes = 1ull << 30;  // head-room left to the driver/others
constexpr uint64_t kStHaloMax = 1ull << 30;     // multi-rank stream-through halo layers, both
constexpr uint64_t kAlign = 256;

uint64_t align_up(uint64_t v) { return (v + kAlign - 1) / kAlign * kAlign; }

int ev_layer(const Domain& d, int64_t L, int par) { return d.ev_layer_base + (int)(2 * L + par); }
int ev_tile(const Domain& d, int64_t k, int par) { return d.ev_tile_base + (int)(2 * k + par); }
int ev_slot(const Domain& d, int s) { return d.ev_slot_base + s; }
int ev_faces_init(const Domain& d) { return d.ev_misc_base + 0; }
int ev_halo(const Domain& d, int par) { return d.ev_misc_base + 1 + par; }
int ev_phase(const Domain& d) { return d.ev_misc_base + 3; }
int ev_in(const Domain& d, int64_t i) { return d.ev_in_base + (int)i; }
int ev_host(const Domain& d, int64_t k) { return d.ev_host_base + (int)k; }
int ev_stream_tail(const Domain& d, int s) { return d.ev_misc_base + 4 + s; }

bool z_wraps_locally(const Geometry& G) { return G.nranks == 1 && G.bc == TILE_BC_PERIODIC; }

// Stream roles of pipeline i: kernels on comp(i), copies in
// on in(i), copies out on out(i) — separate streams when 3S <= 64, so a
// queued copy never holds back an unrelated kernel or copy. Serial (the
// synchronous baseline) puts everything on stream 0.
struct Pipes {
  int S;
  bool split;
  Pipes(int s, bool serial) : S(serial ? 1 : s), split(!serial && 3 * s <= 64) {}
  int comp(int64_t i) const { return (int)(i % S); }
  int in(int64_t i) const { return split ? S + (int)(i % S) : comp(i); }
  int out(int64_t i) const { return split ? 2 * S + (int)(i % S) : comp(i); }
  int used() const { return split ? 3 * S : S; }
};

}  // namespace

// ------------------------------------------------------------------ create
Status domain_create(const int64_t dims[3], const int64_t tdims[3], int ghost,
                     const tile_options* opt_in, Domain** out) {
  tile_options opt{};
  opt.device = -1;
  opt.bc = TILE_BC_PERIODIC;
  opt.nranks = 1;
  opt.rank = 0;
  opt.sched = TILE_SCHED_AUTO;
  opt.fuse_pointwise_steps = 1;
  if (opt_in) opt = *opt_in;
  if (opt.nranks == 0) opt.nranks = 1;
  if (opt.sched < TILE_SCHED_AUTO || opt.sched > TILE_SCHED_SYNC)
    return make_err(TILE_EINVAL, "bad sched");
  if (opt.nstreams_provided < 0 || opt.nstreams_provided > 64)
    return make_err(TILE_EINVAL, "nstreams_provided must be in [0, 64]");
  if (opt.peer_transport < 0 || opt.peer_transport > 2)
    return make_err(TILE_EINVAL, "peer_transport must be 0, 1 or 2");
  Geometry G;
  Status st = make_geometry(dims, tdims, ghost, opt.bc, opt.nranks, opt.rank, &G);
  if (st.bad()) return st;
  if (G.nranks > 1 && !opt.nccl_unique_id && !opt.dry_run && !opt.local_group && !opt.peer_transport)
    return make_err(TILE_EINVAL, "nranks > 1 needs nccl_unique_id, peer_transport or local_group");

  int band = 0, stages = 0;
  size_t smem = 0;
  if (!heat_plan((int)G.t[0], (int)G.t[1], 227 * 1024, &band, &stages, &smem))
    return make_err(TILE_EINVAL, "tile x extent too large to stage a 2-row band in shared memory");

  Domain* d = new Domain();
  d->G = G;
  if (G.depth == 2 && G.nranks == 1 && opt.two_step >= 0) {
    int b2 = 0;
    size_t s2 = 0;
    if (heat2_plan((int)G.t[0], (int)G.t[1], 227 * 1024, &b2, &s2)) {
      d->x2_ok = true;
      d->band2 = b2;
      d->heat2_smem = s2;
    }
  }
  d->opt = opt;
  d->band = band;
  d->stages = stages;
  d->heat_smem = smem;
  if (const char* cf = std::getenv("TILES_HEAT_CACHE")) d->heat_cache_flags = std::atoi(cf);
  d->fault = parse_fault_env();
  if (opt.dry_run) {
    d->exec = make_dry_exec();
  } else {
    d->exec = make_cuda_exec(*d, &st);
    if (st.bad()) {
      delete d;
      return st;
    }
  }
  st = domain_setup(*d);
  if (st.bad()) {
    domain_free(d);
    return st;
  }
  *out = d;
  return Status::ok();
}

Fault parse_fault_env() {
  Fault f;
  const char* e = std::getenv("TILES_FAULT");
  if (!e || !*e) return f;
  static const struct { const char* name; int kind; } kinds[] = {
      {"h2d", FAULT_H2D}, {"d2h", FAULT_D2H}, {"kernel", FAULT_KERNEL}, {"sync", FAULT_SYNC},
      {"host_alloc", FAULT_HOST_ALLOC}};
  const char* colon = std::strchr(e, ':');
  const size_t len = colon ? (size_t)(colon - e) : std::strlen(e);
  for (auto& k : kinds)
    if (std::strlen(k.name) == len && std::strncmp(e, k.name, len) == 0) {
      f.kind = k.kind;
      f.left = colon ? std::max<int64_t>(1, std::atoll(colon + 1)) - 1 : 0;
    }
  return f;
}

bool fault_fires(Domain& d, int kind) {
  if (d.fault.kind != kind) return false;
  if (d.fault.left-- > 0) return false;
  d.fault.kind = FAULT_NONE;  // fires once
  return true;
}

// Memory plan ("calculates how many regions can fit into device
// memory by checking available memory with cudaMemGetInfo"): persistent
// face/halo/table storage first, then as many tile slots as the budget holds.
Status domain_setup(Domain& d) {
  const Geometry& G = d.G;
  Exec& X = *d.exec;
  const uint64_t tile_bytes = (uint64_t)G.tile_elems * 8;
  const bool dir = G.bc == TILE_BC_DIRICHLET;
  const bool multi = G.nranks > 1;

  // host: tile store (+ initial faces for streaming, + Dirichlet faces)
  uint64_t face_bytes_all = 0;
  for (int f = 0; f < 6; ++f) face_bytes_all += align_up((uint64_t)G.ntiles * G.face_elems[f] * 8);
  const uint64_t host_store = align_up((uint64_t)G.ntiles * tile_bytes);
  const uint64_t host_total = host_store + face_bytes_all * (dir ? 2 : 1);
  void* hp = nullptr;
  Status st = X.alloc_host(d, host_total, &hp);
  if (st.bad()) return st;
  d.host_bytes = host_total;
  char* hc = static_cast<char*>(hp);
  d.host = reinterpret_cast<double*>(hc);
  uint64_t off = host_store;
  for (int f = 0; f < 6; ++f) {
    d.host_faces[f] = reinterpret_cast<double*>(hc + off);
    off += align_up((uint64_t)G.ntiles * G.face_elems[f] * 8);
  }
  if (dir)
    for (int f = 0; f < 6; ++f) {
      d.host_dir[f] = reinterpret_cast<double*>(hc + off);
      std::memset(d.host_dir[f], 0, (size_t)G.ntiles * G.face_elems[f] * 8);
      off += align_up((uint64_t)G.ntiles * G.face_elems[f] * 8);
    }

  // device: persistent part
  uint64_t persist = 2 * face_bytes_all;  // export faces, 2 parities
  if (dir) persist += face_bytes_all;
  const uint64_t halo_bytes = align_up((uint64_t)G.layer_tiles * G.face_elems[ZM] * 8);
  const bool peer = multi && d.opt.peer_transport && !d.opt.dry_run;  // halos live in the IPC window
  if (multi && !peer) persist += 4 * halo_bytes;
  // multi-rank stream-through: two tile layers of halo planes in the peer
  // window (periodic slabs; skipped when they would exceed kStHaloMax)
  uint64_t st_bytes = 0;
  if (peer && G.bc == TILE_BC_PERIODIC && d.opt.stream_through >= 0) {
    const uint64_t layer = align_up((uint64_t)G.layer_tiles * G.tile_elems * 8);
    if (2 * layer <= kStHaloMax) st_bytes = layer;
  }
  // dry runs (trace replay on CPU) of a peer-transport domain take the same
  // multi-rank stream-through decisions, with no window behind them
  if (multi && d.opt.peer_transport && d.opt.dry_run && G.bc == TILE_BC_PERIODIC && d.opt.stream_through >= 0)
    d.st_halo_bytes = (uint64_t)G.layer_tiles * G.tile_elems * 8;
  const uint64_t gsrc_bytes = align_up((uint64_t)G.ntiles * 6 * sizeof(double*));
  const uint64_t items_bytes = align_up((uint64_t)G.ntiles * sizeof(TileItem));
  persist += 2 * gsrc_bytes + 2 * items_bytes;
  const uint64_t ystr_bytes = align_up((uint64_t)G.ntiles * 2 * sizeof(int64_t));
  persist += 4 * gsrc_bytes + ystr_bytes;  // direct ghost-source tables (resident mode)
  const uint64_t prog_bytes = align_up(kMaxProgCtas * sizeof(unsigned long long));
  persist += prog_bytes;                    // multi-step progress counters
  const uint64_t esrc_bytes = d.x2_ok ? align_up((uint64_t)G.ntiles * 12 * sizeof(EdgePtr)) : 0;
  const uint64_t mask_bytes = d.x2_ok ? align_up((uint64_t)G.ntiles) : 0;
  persist += 2 * esrc_bytes + mask_bytes;

  uint64_t budget;
  if (d.opt.device_pool) {
    budget = d.opt.device_pool_bytes;
  } else {
    uint64_t fr = 0, tot = 0;
    st = X.mem_info(d, &fr, &tot);
    if (st.bad()) return st;
    budget = fr > kReserveBytes ? fr - kReserveBytes : 0;
    const uint64_t window = peer ? 4 * halo_bytes + 256 + 2 * st_bytes : 0;  // own cudaMalloc
    budget = budget > window ? budget - window : 0;
  }
  if (d.opt.device_budget_bytes) budget = std::min<uint64_t>(budget, d.opt.device_budget_bytes);
  if (budget < persist + 2 * tile_bytes)
    return make_err(TILE_ENOMEM_DEVICE, "device budget below faces + 2 tile slots");
  const uint64_t fit = (budget - persist) / tile_bytes;
  const uint64_t want_res = 2 * (uint64_t)G.ntiles;
  switch (d.opt.sched) {
    case TILE_SCHED_RESIDENT:
    case TILE_SCHED_SYNC:
      if (fit < want_res) return make_err(TILE_ENOMEM_DEVICE, "resident schedule does not fit");
      d.mode = MODE_RESIDENT;
      d.nslots = (int)want_res;
      break;
    case TILE_SCHED_STREAM:
      d.mode = MODE_STREAM;
      d.nslots = (int)std::min<uint64_t>(fit, want_res);
      break;
    default:
      d.mode = fit >= want_res ? MODE_RESIDENT : MODE_STREAM;
      d.nslots = (int)std::min<uint64_t>(fit, want_res);
  }
  const uint64_t dev_total = persist + (uint64_t)d.nslots * tile_bytes;
  void* dp = nullptr;
  if (d.opt.device_pool) {
    dp = d.opt.device_pool;
    d.own_pool = false;
  } else {
    st = X.alloc_device(d, dev_total, &dp);
    if (st.bad()) return st;
    d.own_pool = true;
  }
  d.pool = static_cast<char*>(dp);
  d.pool_bytes = dev_total;
  d.device_bytes = dev_total;
  d.budget_left = budget > dev_total ? budget - dev_total : 0;
  off = 0;
  auto carve = [&](uint64_t bytes) {
    char* p = d.pool + off;
    off += align_up(bytes);
    return p;
  };
  for (int p = 0; p < 2; ++p)
    for (int f = 0; f < 6; ++f)
      d.faces[f][p] = reinterpret_cast<double*>(carve((uint64_t)G.ntiles * G.face_elems[f] * 8));
  if (dir)
    for (int f = 0; f < 6; ++f)
      d.dir_faces[f] = reinterpret_cast<double*>(carve((uint64_t)G.ntiles * G.face_elems[f] * 8));
  if (multi && !peer)
    for (int a = 0; a < 2; ++a)
      for (int p = 0; p < 2; ++p) d.halo[a][p] = reinterpret_cast<double*>(carve(halo_bytes));
  if (peer) {  // before the ghost-source tables, which point into the halos
    st = peer_setup(d, halo_bytes, st_bytes);
    if (st.bad()) return st;
  }
  for (int p = 0; p < 2; ++p) d.gsrc_dev[p] = reinterpret_cast<const double**>(carve(gsrc_bytes));
  for (int p = 0; p < 2; ++p) d.items_dev[p] = reinterpret_cast<TileItem*>(carve(items_bytes));
  for (int b = 0; b < 2; ++b)
    for (int p = 0; p < 2; ++p) d.gdir_dev[b][p] = reinterpret_cast<const double**>(carve(gsrc_bytes));
  d.ystr_dev = reinterpret_cast<int64_t*>(carve(ystr_bytes));
  d.prog_dev = reinterpret_cast<unsigned long long*>(carve(prog_bytes));
  if (d.x2_ok) {
    for (int p = 0; p < 2; ++p) d.esrc_dev[p] = reinterpret_cast<EdgePtr*>(carve(esrc_bytes));
    d.fixed_mask_dev = reinterpret_cast<uint8_t*>(carve(mask_bytes));
  }
  d.slot_base = reinterpret_cast<double*>(d.pool + off);

  // ghost-source tables (both parities) and resident item lists
  for (int p = 0; p < 2; ++p) {
    d.gsrc_host[p].resize((size_t)G.ntiles * 6);
    for (int64_t k = 0; k < G.ntiles; ++k)
      for (int f = 0; f < 6; ++f) d.gsrc_host[p][(size_t)k * 6 + f] = d.face_src_ptr(k, f, p);
  }
  if (d.x2_ok) {
    for (int p = 0; p < 2; ++p) {
      d.esrc_host[p].resize((size_t)G.ntiles * 12);
      for (int64_t k = 0; k < G.ntiles; ++k)
        for (int e = 0; e < 12; ++e) d.esrc_host[p][(size_t)k * 12 + e] = d.edge_src_ptr(k, e, p);
    }
    d.fixed_mask_host.assign((size_t)G.ntiles, 0);
    for (int64_t k = 0; k < G.ntiles; ++k)
      for (int f = 0; f < 6; ++f)
        if (face_source(G, k, f).kind == 1) d.fixed_mask_host[(size_t)k] |= (uint8_t)(1u << f);
  }
  // direct ghost sources: resident mode with a specialised single-step kernel
  // (TILES_DIRECT=0 keeps every ghost read on the exported faces)
  {
    const char* e = std::getenv("TILES_DIRECT");
    d.direct_ok = d.mode == MODE_RESIDENT && heat_is_fixed((int)G.t[0], d.band, d.stages, d.heat_smem) &&
                  !(e && std::atoi(e) == 0);
  }
  // fused halo push: peer transport mode 2 with direct passes (multi-rank resident)
  d.peer_fused = multi && d.opt.peer_transport == 2 && d.direct_ok;
  // persistent multi-step launches: single rank, direct passes (TILES_PERSIST=0: off)
  {
    const char* e = std::getenv("TILES_PERSIST");
    d.persist_ok = !multi && d.direct_ok && !(e && std::atoi(e) == 0);
  }
  if (d.direct_ok) {
    for (int b = 0; b < 2; ++b)
      for (int p = 0; p < 2; ++p) {
        d.gdir_host[b][p].resize((size_t)G.ntiles * 6);
        for (int64_t k = 0; k < G.ntiles; ++k)
          for (int f = 0; f < 6; ++f) d.gdir_host[b][p][(size_t)k * 6 + f] = d.direct_src_ptr(k, f, b, p);
      }
    d.ystr_host.resize((size_t)G.ntiles * 2);
    for (int64_t k = 0; k < G.ntiles; ++k) {
      d.ystr_host[(size_t)k * 2] = d.direct_ystride(k, YM);
      d.ystr_host[(size_t)k * 2 + 1] = d.direct_ystride(k, YP);
    }
  }
  if (d.mode == MODE_RESIDENT) {
    for (int b = 0; b < 2; ++b) {
      d.items_host[b].resize((size_t)G.ntiles);
      for (int64_t k = 0; k < G.ntiles; ++k) {
        const int cur = b == 0 ? (int)k : (int)(G.ntiles + k);
        const int nxt = b == 0 ? (int)(G.ntiles + k) : (int)k;
        d.items_host[b][(size_t)k] = {d.slot_ptr(cur), d.slot_ptr(nxt), (int32_t)k, 0};
      }
    }
  } else {
    d.items_dev[0] = d.items_dev[1] = nullptr;
  }

  // residency: cache list all -1
  d.slot_owner.assign((size_t)d.nslots, -1);
  d.tile_slot.assign((size_t)G.ntiles, -1);
  d.tile_dirty.assign((size_t)G.ntiles, 0);
  d.tile_last_use.assign((size_t)G.ntiles, 0);
  d.free_slots.clear();
  for (int s = 0; s < d.nslots; ++s) d.free_slots.push_back(s);

  // events
  d.ev_layer_base = 0;
  d.ev_tile_base = d.ev_layer_base + (int)(2 * G.n[2]);
  d.ev_slot_base = d.ev_tile_base + (int)(2 * G.ntiles);
  d.ev_in_base = d.ev_slot_base + d.nslots;
  d.ev_host_base = d.ev_in_base + (int)G.ntiles;
  d.ev_misc_base = d.ev_host_base + (int)G.ntiles;
  d.nevents = d.ev_misc_base + 4 + d.halo_stream + 1 + 3;  // + 2 stream-through ring events, 1 halo push
  st = X.setup(d);
  if (st.bad()) return st;
  // cost-model calibration: r = sweep time / duplex link time
  // per plane. Explicit (tile_options.sweep_link_ratio, env TILES_ST_R), else
  // measured here on the box when a fresh-upload schedule can use it, else
  // the B200 + PCIe 5 fit (0.021)
  d.r_sweep = 0.021;
  if (d.opt.sweep_link_ratio > 0) {
    d.r_sweep = d.opt.sweep_link_ratio;
  } else if (const char* e = getenv("TILES_ST_R")) {
    d.r_sweep = atof(e);
  } else if (d.mode == MODE_RESIDENT && !multi && G.t[0] % 2 == 0 && G.l[2] >= 32) {
    double r = 0;
    st = X.calibrate(d, &r);
    if (st.bad()) return st;
    if (r > 0) d.r_sweep = r;
  }
  if (multi && !d.opt.dry_run && !d.opt.local_group && !d.opt.peer_transport) {
    st = nccl_init(d);
    if (st.bad()) return st;
  }
  return Status::ok();
}

Status domain_free(Domain* d) {
  if (!d) return Status::ok();
  Status r;
  if (d->exec) {
    if (!d->poisoned && d->in_flight) r = d->exec->sync_all(*d);
    if (d->nccl_comm) nccl_destroy(*d);
    if (d->peer_window) peer_destroy(*d);
    d->exec->destroy(*d);
    if (d->own_pool && d->pool) d->exec->free_device(*d, d->pool);
    if (d->own_wave && d->wave_base) d->exec->free_device(*d, d->wave_base);
    if (d->host) d->exec->free_host(*d, d->host);
    delete d->exec;
  }
  delete d;
  return r;
}

// --------------------------------------------------------------- residency
namespace {

// Every operation on a device slot waits for the slot's event and records
// it again afterwards, so the operations on one slot are totally ordered in
// issue order whatever stream they run on (WAR/WAW/RAW on the slot).
struct Sched {
  Domain& d;
  Exec& X;
  Pipes P;
  std::set<std::pair<int64_t, int>> lru;  // (last_use, tile) of resident tiles

  explicit Sched(Domain& dd, const Pipes& p) : d(dd), X(*dd.exec), P(p) {
    for (int64_t k = 0; k < d.G.ntiles; ++k)
      if (d.tile_slot[k] >= 0) lru.insert({d.tile_last_use[k], (int)k});
  }

  void touch(int64_t k) {
    lru.erase({d.tile_last_use[k], (int)k});
    d.tile_last_use[k] = ++d.use_clock;
    lru.insert({d.tile_last_use[k], (int)k});
  }

  // D2H of tile k from its slot into the pinned host store.
  Status writeback(int64_t k) {
    const int s = d.tile_slot[k];
    const int st = P.out(k);
    Status r = X.wait(d, ev_slot(d, s), st);
    if (r.bad()) return r;
    r = X.d2h(d, k, 1, s, st);
    if (r.bad()) return r;
    d.tile_dirty[k] = 0;
    d.stats.writebacks++;
    r = X.record(d, ev_slot(d, s), st);
    if (r.bad()) return r;
    return X.record(d, ev_host(d, k), st);  // host copy of k written (RAW for its next H2D)
  }

  // A free device slot for tile k: a free pointer, else the least
  // recently used resident tile is evicted — copied back first if dirty
  // ("queues memory transfers of the region that is currently using
  // the assigned device memory pointer from device to host"), dropped if
  // clean. `protect` is never evicted.
  Status acquire(int64_t k, int stream, int protect, int* out) {
    int s;
    if (!d.free_slots.empty()) {
      s = d.free_slots.front();
      d.free_slots.pop_front();
    } else {
      int victim = -1;
      for (auto& e : lru) {
        const int t = e.second;
        if (t != k && d.tile_slot[t] != protect) {
          victim = t;
          break;
        }
      }
      if (victim < 0) return make_err(TILE_ENOMEM_DEVICE, "no evictable slot");
      s = d.tile_slot[victim];
      if (d.tile_dirty[victim]) {
        Status r = writeback(victim);
        if (r.bad()) return r;
      } else {
        Status r = X.note(d, TILE_OP_DROP, victim, s, P.comp(victim));
        if (r.bad()) return r;
      }
      d.stats.evictions++;
      lru.erase({d.tile_last_use[victim], victim});
      d.tile_slot[victim] = -1;
      d.slot_owner[s] = -1;
    }
    Status r = X.wait(d, ev_slot(d, s), stream);
    if (r.bad()) return r;
    d.slot_owner[s] = (int)k;
    *out = s;
    return Status::ok();
  }

  void release(int s) {
    d.slot_owner[s] = -1;
    d.free_slots.push_back(s);
  }
};

// Make every stream of this run wait for everything issued before it
// (previous runs may have used other streams, faces are shared state).
Status join_streams(Domain& d, int S) {  // S = number of low-index streams in use
  Exec& X = *d.exec;
  const int nst = d.halo_stream + 1;
  for (int s = 0; s < nst; ++s) {
    if (s >= S && s != d.halo_stream) continue;
    Status r = X.record(d, ev_stream_tail(d, s), s);
    if (r.bad()) return r;
  }
  for (int s = 0; s < nst; ++s) {
    if (s >= S && s != d.halo_stream) continue;
    for (int t = 0; t < nst; ++t) {
      if (t == s || (t >= S && t != d.halo_stream)) continue;
      Status r = X.wait(d, ev_stream_tail(d, t), s);
      if (r.bad()) return r;
    }
  }
  return Status::ok();
}

}  // namespace

// ----------------------------------------------------- resident heat runs
// Batches are contiguous z-layer ranges; batch i runs on stream i % S. A
// batch's step s waits for its neighbour batches' step s-1 (their faces are
// its ghost sources, and it overwrites the face parity they read).
namespace {

struct Batch {
  int64_t L0, L1;  // layers [L0, L1)
  int stream;      // compute stream
  int in, out;     // copy-in / copy-out streams
};

struct ResidentRun {
  Domain& d;
  Exec& X;
  const Geometry& G;
  std::vector<Batch> B;
  std::vector<std::vector<int>> nbr;  // neighbour batches (excluding self)
  bool need_load, need_extract, multi;
  bool entry_wait = false;  // first op of every batch waits ev_phase (phase join)
  int bit0, fp0, T;         // T = number of passes (a pass advances 1 or 2 steps)
  std::vector<int> kpass;   // steps per pass
  double alpha;

  ResidentRun(Domain& dd) : d(dd), X(*dd.exec), G(dd.G) {}

  int64_t tile0(const Batch& b) const { return b.L0 * G.layer_tiles; }
  int64_t ntl(const Batch& b) const { return (b.L1 - b.L0) * G.layer_tiles; }
  int cur_slot(int64_t k, int bit) const { return bit == 0 ? (int)k : (int)(G.ntiles + k); }

  void build(int S, bool serial, bool layered) {
    const int64_t nL = G.n[2];
    B.clear();
    const Pipes P(S, serial);
    if (serial || (!layered && !multi)) {
      B.push_back({0, nL, 0, P.in(0), P.out(0)});
    } else if (!layered && multi && nL > 2) {
      B.push_back({0, 1, 0, 0, 0});
      B.push_back({nL - 1, nL, 0, 0, 0});
      B.push_back({1, nL - 1, 0, 0, 0});
    } else {
      for (int64_t L = 0; L < nL; ++L) B.push_back({L, L + 1, 0, 0, 0});
      // wrap-aware order: 0, nL-1, 1, nL-2, ... so a periodic layer's
      // neighbours arrive early
      std::vector<Batch> o;
      int64_t lo = 0, hi = nL - 1;
      bool front = true;
      while (lo <= hi) {
        o.push_back(B[front ? lo++ : hi--]);
        front = !front;
      }
      if (!z_wraps_locally(G)) std::sort(o.begin(), o.end(), [](auto& a, auto& b) { return a.L0 < b.L0; });
      B = o;
    }
    if (B.size() > 1)
      for (size_t i = 0; i < B.size(); ++i) {
        B[i].stream = P.comp((int64_t)i);
        B[i].in = P.in((int64_t)i);
        B[i].out = P.out((int64_t)i);
      }
    // neighbour batches
    auto batch_of = [&](int64_t L) {
      for (size_t i = 0; i < B.size(); ++i)
        if (L >= B[i].L0 && L < B[i].L1) return (int)i;
      return -1;
    };
    nbr.assign(B.size(), {});
    for (size_t i = 0; i < B.size(); ++i) {
      std::vector<int64_t> ls = {B[i].L0 - 1, B[i].L1};
      for (int64_t L : ls) {
        if (L < 0 || L >= nL) {
          if (!z_wraps_locally(G)) continue;
          L = (L + nL) % nL;
        }
        int j = batch_of(L);
        if (j >= 0 && j != (int)i &&
            std::find(nbr[i].begin(), nbr[i].end(), j) == nbr[i].end())
          nbr[i].push_back(j);
      }
    }
  }
  bool boundary(const Batch& b) const { return b.L0 == 0 || b.L1 == G.n[2]; }

  Status issue_load(size_t i) {
    const Batch& b = B[i];
    Status r;
    if (entry_wait) {
      r = X.wait(d, ev_phase(d), b.stream);
      if (r.bad()) return r;
    }
    if (need_load) {
      r = X.h2d(d, tile0(b), ntl(b), cur_slot(tile0(b), bit0), b.in);
      if (r.bad()) return r;
      if (b.in != b.stream) {
        r = X.record(d, ev_in(d, (int64_t)i), b.in);
        if (r.bad()) return r;
        r = X.wait(d, ev_in(d, (int64_t)i), b.stream);
        if (r.bad()) return r;
      }
    }
    if (need_extract) {
      r = X.extract(d, tile0(b), ntl(b), cur_slot(tile0(b), bit0), fp0,
                    d.items_dev[bit0] ? d.items_dev[bit0] + tile0(b) : nullptr, b.stream);
      if (r.bad()) return r;
    }
    return X.record(d, ev_layer(d, (int64_t)i, 1), b.stream);
  }

  Status issue_kernel(size_t i, int s) {
    const Batch& b = B[i];
    Status r;
    for (int j : nbr[i]) {
      r = X.wait(d, ev_layer(d, j, (s - 1) & 1), b.stream);
      if (r.bad()) return r;
    }
    if (multi && boundary(b)) {
      r = X.wait(d, ev_halo(d, (s - 1) & 1), b.stream);
      if (r.bad()) return r;
    }
    const int bit = bit0 ^ (s & 1);
    const int rp = fp0 ^ (s & 1);
    const TileItem* items = d.items_dev[bit] ? d.items_dev[bit] + tile0(b) : nullptr;
    if (kpass[(size_t)s] == 2)
      r = X.heat2(d, nullptr, nullptr, nullptr, (int)ntl(b), rp, items, b.stream);
    else if (d.direct_ok && items)  // y/z ghosts from the neighbours' interiors, stacked z-march
      r = X.heat(d, nullptr, nullptr, nullptr, (int)ntl(b), rp, items, b.stream, bit, (int)(b.L1 - b.L0));
    else
      r = X.heat(d, nullptr, nullptr, nullptr, (int)ntl(b), rp, items, b.stream);
    if (r.bad()) return r;
    (void)alpha;
    return X.record(d, ev_layer(d, (int64_t)i, s & 1), b.stream);
  }

  // every pass of this phase as ONE persistent launch (HeatParams::nsteps):
  // one whole-domain batch, single rank, direct single steps
  bool persistent() const {
    if (!d.persist_ok || multi || B.size() != 1 || T < 2 || !d.items_dev[0]) return false;
    for (int s = 0; s < T; ++s)
      if (kpass[(size_t)s] != 1) return false;
    return true;
  }
  Status issue_kernels_persistent() {
    const Batch& b = B[0];
    const TileItem* items = d.items_dev[bit0] + tile0(b);
    Status r = X.heat(d, nullptr, nullptr, nullptr, (int)ntl(b), fp0, items, b.stream, bit0,
                      (int)(b.L1 - b.L0), T);
    if (r.bad()) return r;
    return X.record(d, ev_layer(d, 0, (T - 1) & 1), b.stream);
  }

  Status issue_halo(int s) {  // exchange the faces written at step s (s = -1: current)
    const int hs = d.halo_stream;
    Status r;
    for (size_t i = 0; i < B.size(); ++i) {
      if (!boundary(B[i])) continue;
      r = X.wait(d, ev_layer(d, (int64_t)i, s & 1), hs);
      if (r.bad()) return r;
    }
    // fused peer transport: after a step, the kernels have pushed the data
    const int mode = !d.peer_fused ? 0 : s < 0 ? 1 : 2;
    r = X.halo(d, fp0 ^ ((s + 1) & 1), hs, mode);
    if (r.bad()) return r;
    return X.record(d, ev_halo(d, s & 1), hs);
  }

  // Greedy list issue of the (load, kernel, halo) DAG in dependency order.
  Status run() {
    const size_t nb = B.size();
    std::vector<int> done(nb, -2);  // last issued: -2 nothing, -1 load, s kernel step s
    int halo_done = -2;              // last halo step issued (-1 = initial)
    size_t loads = 0;
    std::vector<size_t> load_order(nb);
    for (size_t i = 0; i < nb; ++i) load_order[i] = i;
    auto kernel_ready = [&](size_t i) {
      const int s = done[i] + 1;
      if (s >= T || done[i] < -1) return false;
      for (int j : nbr[i])
        if (done[j] < s - 1) return false;
      if (multi && boundary(B[i]) && halo_done < s - 1) return false;
      return true;
    };
    auto halo_ready = [&]() {
      if (!multi) return false;
      const int s = halo_done + 1;  // next halo step to issue
      if (s > T - 2) return false;  // nobody consumes the last step's halo
      for (size_t i = 0; i < nb; ++i)
        if (boundary(B[i]) && done[i] < s) return false;
      // WAR: the step-s halo overwrites buffers read by step s-1 kernels,
      // which precede the step-s boundary kernels in stream order.
      return true;
    };
    if (persistent()) {
      Status r = issue_load(0);
      if (r.bad()) return r;
      return issue_kernels_persistent();
    }
    for (;;) {
      bool progress = false;
      // drain everything ready, in (step, batch) order
      for (bool again = true; again;) {
        again = false;
        if (halo_ready()) {
          Status r = issue_halo(halo_done + 1);
          if (r.bad()) return r;
          ++halo_done;
          again = progress = true;
        }
        int best_s = 1 << 30;
        for (size_t i = 0; i < nb; ++i)
          if (kernel_ready(i)) best_s = std::min(best_s, done[i] + 1);
        for (size_t i = 0; i < nb; ++i) {
          if (kernel_ready(i) && done[i] + 1 == best_s) {
            Status r = issue_kernel(i, done[i] + 1);
            if (r.bad()) return r;
            ++done[i];
            again = progress = true;
          }
        }
      }
      if (loads < nb) {
        Status r = issue_load(load_order[loads]);
        if (r.bad()) return r;
        done[load_order[loads]] = -1;
        ++loads;
        if (loads == nb && multi && halo_done == -2) {
          r = issue_halo(-1);
          if (r.bad()) return r;
          halo_done = -1;
        }
        continue;
      }
      if (!progress) break;
    }
    for (size_t i = 0; i < nb; ++i)
      if (done[i] != T - 1) return make_err(TILE_ESTATE, "internal: resident schedule incomplete");
    return Status::ok();
  }
};

}  // namespace

static Status upload_dirichlet_if_needed(Domain& d);

// Phases: with a fresh upload, layer batches for the steps
// the load wavefront can overlap (k1 = nL/2 + 1), whole-domain batches for
// the middle steps (one launch per step, or bottom/top/interior with slab
// halos), and layer batches again for the final step so each layer's D2H can
// start as soon as its last kernel ends. Phases are joined through ev_phase.
// Steps -> passes: with ghost 2 (and a two-step kernel for the tile shape)
// a pass advances two steps; an odd remainder is one single-step pass.
static std::vector<int> plan_passes(const Domain& d, int steps) {
  std::vector<int> k;
  if (d.x2_ok && (d.opt.two_step > 0 || d.mode == MODE_STREAM)) {
    for (int i = 0; i < steps / 2; ++i) k.push_back(2);
    if (steps & 1) k.push_back(1);
  } else {
    k.assign((size_t)steps, 1);
  }
  return k;
}

// Stream-through: with a fresh upload, a cell after T steps
// depends only on cells within T planes, so with T <= tz a unit of >= T
// planes needs only its own and its two neighbour units' initial data. Per
// unit (in z order): T sweeps over the unit and T halo planes with the valid
// range shrinking by one plane per end (the first reads the resident array,
// the last writes the exact core into packed sub-tiles), then its D2H. H2D of
// later units, compute and D2H of earlier units overlap (duplex host link).
// Scratch = the resident mode's second buffer array (not needed otherwise in
// this run). Each unit's result is also copied back into the resident array
// once its initial data has no reader left (after the next unit's first
// sweep; unit 0, read by the last unit through the periodic wrap, at the
// end), so the domain stays resident. Periodic, single rank.
struct UnitDef {
  int64_t layer, p0, np;  // planes [p0, p0+np) of tile layer `layer`
};
struct StreamPlan {
  int64_t unit;        // nominal planes per unit (divides tz, >= T)
  int64_t units;       // number of units
  std::vector<UnitDef> u;
  int64_t slab_tiles;  // one dense slab of max unit + 2T planes, in tile slots
  int64_t sub_tiles;   // one packed unit result (layer_tiles sub-tiles), in tile slots
};

// Units in z order: each tile layer cut into tz / un pieces of un planes
// (un >= T: a unit's halo lies in its two neighbour units). The H2D order
// is U-1, 0, 1, ..., U-2: the first D2H waits for the uploads of U-1, 0
// and 1 (the fill), and the last upload (unit U-2) gates the computes and
// D2Hs of units U-3, U-2 and U-1, which all follow it (the drain). The last
// layer's tail is therefore cut into `thin` units of T planes (the smallest
// a unit may be) and the first layer's head into thin - 1 (<= 2) of them
// (TILES_ST_THIN, default 3; 0 = uniform units).
static int st_thin_default() {
  static const int thin = [] {
    const char* e = getenv("TILES_ST_THIN");
    return e ? std::max(0, atoi(e)) : 3;
  }();
  return thin;
}

// Units per H2D copy in the stream-through steady state (TILES_ST_H2D_MERGE,
// default 2; 1 = one copy per unit).
static int st_h2d_merge() {
  static const int m = [] {
    const char* e = getenv("TILES_ST_H2D_MERGE");
    return e ? std::max(1, atoi(e)) : 2;
  }();
  return m;
}

static std::vector<UnitDef> make_units(const Geometry& G, int64_t un, int T, int thin) {
  std::vector<UnitDef> v;
  const int64_t tz = G.t[2];
  const bool cut = thin > 0 && un > T && G.n[2] * (tz / un) >= 4 && G.n[2] >= 2;
  for (int64_t L = 0; L < G.n[2]; ++L) {
    const bool last = L == G.n[2] - 1;
    int64_t tail = 0, head = 0;  // planes of the layer cut into thin units
    if (cut && last) {
      tail = (int64_t)thin * T;
      while (tail > 0 && tz - tail < T) tail -= T;  // the rest stays a unit of >= T planes
    }
    if (cut && L == 0) {  // the fill: units 0 and 1 (with U-1) gate the first D2H
      head = std::min<int64_t>(2, thin - 1) * T;
      while (head > 0 && tz - head < T) head -= T;
    }
    int64_t p = 0;
    for (; p < head; p += T) v.push_back({L, p, (int64_t)T});
    for (; p + un <= tz - tail; p += un) v.push_back({L, p, un});
    if (p < tz - tail) {  // remainder: its own unit if >= T planes, else extends the previous one
      if (tz - tail - p < T && !v.empty() && v.back().layer == L) v.back().np += tz - tail - p;
      else v.push_back({L, p, tz - tail - p});
      p = tz - tail;
    }
    for (; p < tz; p += T) v.push_back({L, p, (int64_t)T});
  }
  return v;
}

static bool streamthrough_ok(const Domain& d, int T, StreamPlan* sp, double* est_out) {
  const Geometry& G = d.G;
  if (d.opt.stream_through < 0 || G.bc != TILE_BC_PERIODIC) return false;
  // z-slab ranks: the peer transport's halo layers carry the T planes beyond
  // each slab end (comm_peer.cu peer_st_halo)
  if (G.nranks != 1 && !(d.st_halo_bytes && (d.peer_connected || d.opt.dry_run))) return false;
  if (T < 1 || (int64_t)T > G.t[2]) return false;
  if (G.t[0] % 2 || G.l[2] > (1 << 30)) return false;  // x-pairs (double2); int plane index
  const int64_t plane = G.l[0] * G.l[1];
  // unit = a divisor of tz, >= T (after T steps a unit then depends on its
  // two neighbour units only) and >= min_unit (per-unit overheads). Thin
  // units shorten the pipeline's fill and drain (~3 units of one-way copies);
  // thick ones cut the redundant halo sweeps (a unit sweeps T*unit + T^2 - T
  // planes). Pick the divisor minimising, in per-plane link-copy times,
  //   max(nz, r * nz * (T + (T^2 - T) / unit)) + 3 * unit,
  // r = sweep time / duplex link time per plane, 0.021 measured on B200 +
  // PCIe 5 (slab_sweep_ca ~0.8 us per 512^2 plane, ~48 GB/s per direction;
  // profiles/r01/ncu_slab_sweep.txt, bench_fig5_st_*.json).
  static const int64_t min_unit = [] {
    const char* e = getenv("TILES_ST_MINUNIT");
    return e ? std::max<int64_t>(1, atoll(e)) : (int64_t)16;
  }();
  const double r_sweep = d.r_sweep;  // calibrated per box (domain_setup)
  const double nz = (double)G.l[2], Td = (double)T;
  int64_t unit = G.t[2];
  double best = 1e300;
  for (int64_t u = 1; u <= G.t[2]; ++u) {
    if (G.t[2] % u || u < (int64_t)T || u < std::min<int64_t>(min_unit, G.t[2])) continue;
    const double est = std::max(nz, r_sweep * nz * (Td + (Td * Td - Td) / (double)u)) + 3.0 * (double)u;
    if (est < best) best = est, unit = u;
  }
  // the caller compares with the batched resident schedule (both link
  // directions in sequence, 2 nz, plus T whole-domain steps partly
  // overlapped, 0.011 per plane-step, same fit) and the wavefront
  *est_out = best;
  if (G.l[2] / unit + 4 > G.ntiles) unit = G.t[2];  // event budget (one per unit)
  sp->unit = unit;
  // thin tail units first; uniform units if those do not fit
  for (int thin : {st_thin_default(), 0}) {
    sp->u = make_units(G, unit, T, thin);
    if ((int64_t)sp->u.size() > G.ntiles) sp->u = make_units(G, G.t[2], T, 0);
    sp->units = (int64_t)sp->u.size();
    int64_t mx = 0;
    for (const auto& x : sp->u) mx = std::max(mx, x.np);
    sp->slab_tiles = ((mx + 2 * (int64_t)T) * plane + G.tile_elems - 1) / G.tile_elems;
    sp->sub_tiles = (G.layer_tiles * mx * G.t[0] * G.t[1] + G.tile_elems - 1) / G.tile_elems;
    if (2 * sp->slab_tiles + 3 * sp->sub_tiles <= G.ntiles) return true;
  }
  return false;
}

// Stream-through over units of `unit` planes (a unit is a slice of one tile
// layer: planes [p0, p0+unit) of each of its tiles, contiguous per tile, so
// its H2D/D2H are single strided 2-D copies). Per unit u, in z order: T
// sweeps over u and T halo planes with the valid range shrinking by one plane
// per end (the first reads the resident array, the middle ones ping-pong
// between two dense slabs, the last writes the exact core into packed
// sub-tiles), then the D2H. Unit u's result is written back into the resident
// array after unit u+1's first sweep (unit 0, read by the last unit through
// the periodic wrap, at the end).
static Status run_streamthrough(Domain& d, double alpha, int T, int S, const StreamPlan& sp) {
  (void)alpha;
  Exec& X = *d.exec;
  const Geometry& G = d.G;
  const int64_t U = sp.units, lt = G.layer_tiles, tz = G.t[2];
  const Pipes P(S, false);
  const int bit = d.res_bit;                       // H2D target array
  const int sb = bit ? 0 : (int)G.ntiles;          // scratch array (the other one)
  d.slab_depth = sp.slab_tiles * G.tile_elems / (G.l[0] * G.l[1]);  // planes a slab holds
  const int slab[2] = {sb, sb + (int)sp.slab_tiles};
  const int out[2] = {sb + 2 * (int)sp.slab_tiles, sb + 2 * (int)sp.slab_tiles + (int)sp.sub_tiles};
  const int keep0 = sb + 2 * (int)sp.slab_tiles + 2 * (int)sp.sub_tiles;
  (void)tz;
  auto layer_of = [&](int64_t u) { return sp.u[(size_t)u].layer; };
  auto p0_of = [&](int64_t u) { return sp.u[(size_t)u].p0; };
  auto np_of = [&](int64_t u) { return sp.u[(size_t)u].np; };
  auto z0_of = [&](int64_t u) { return layer_of(u) * G.t[2] + p0_of(u); };  // first local plane
  auto cur_slot = [&](int64_t u) {
    const int64_t t0 = layer_of(u) * lt;
    return bit ? (int)(G.ntiles + t0) : (int)t0;
  };
  auto res_of = [&](int64_t u) { return u == 0 ? keep0 : out[u & 1]; };
  auto ev_unit_done = [&](int64_t u) { return ev_host(d, u); };  // compute of unit u
  const int ring_ev[2] = {d.ev_misc_base + 4 + d.halo_stream + 1, d.ev_misc_base + 5 + d.halo_stream + 1};
  const int cs = P.comp(0), os = P.out(0);
  const bool multi = G.nranks > 1;  // z-slab ranks: halo layers replace the periodic wrap
  // two sweeps per kernel (heat2_band_slab shrink mode) with two_step = 1:
  // half the HBM traffic of the unit sweeps, but the C2 step is link-bound
  // and measured the same (24.82 vs 24.84 ms, four alternating pairs), while
  // the short two-level launches reach 0.53 of HBM against the single
  // sweeps' 0.67-0.76 — single sweeps by default
  const bool two = d.opt.two_step > 0 && !multi && X.sweep2s_ok(d);
  const int hs = d.halo_stream;
  const int ev_push = d.ev_misc_base + 6 + d.halo_stream + 1;
  if (multi) ++d.st_epoch;
  Status r;
  // one copy-in stream, so the copy engine runs the H2Ds in this order (it
  // may not across streams): the last unit first (unit 0's wrap neighbour),
  // then the planes below it in z order. Past the fill, the copies are cut
  // after every `merge` units (TILES_ST_H2D_MERGE): with D2H running, each
  // copy costs a ~40 us gap on the H2D side (profiles/r01/pcie_gap.json), and
  // H2D is the bottleneck of the steady state. With offset cuts
  // (TILES_ST_OFFSET=1; default 0) a copy ending after unit v also carries
  // the first T planes of unit v+1 (same tile layer), the top of unit v's
  // halo, so unit v's sweeps and D2H can start when that copy lands; with
  // 16-plane units in 64-plane layers this only moves one unit per layer and
  // lengthens that copy (C2: no gain measured). The thin end
  // units stay separate.
  static const int offset = [] {
    const char* e = getenv("TILES_ST_OFFSET");
    return e ? atoi(e) : 0;
  }();
  const int merge = st_h2d_merge();
  // units uploaded one per copy at the head (TILES_ST_HEAD, default 2: the
  // fill's units 0 and 1; more lets the first D2Hs follow unit by unit)
  static const int head = [] {
    const char* e = getenv("TILES_ST_HEAD");
    return e ? std::max(0, atoi(e)) : 2;
  }();
  const int64_t nzl = G.l[2];
  struct Copy {
    int64_t layer, p0, np;
  };
  std::vector<Copy> cps;
  std::vector<int> cp_of((size_t)nzl, 0);  // plane -> index of the copy that uploads it
  auto plan_copies = [&](bool off) {
    cps.clear();
    auto add = [&](int64_t zlo, int64_t zhi) {  // planes [zlo, zhi), one copy per tile layer
      while (zlo < zhi) {
        const int64_t L = zlo / tz, e = std::min(zhi, (L + 1) * tz);
        for (int64_t z = zlo; z < e; ++z) cp_of[(size_t)z] = (int)cps.size();
        cps.push_back({L, zlo - L * tz, e - zlo});
        zlo = e;
      }
    };
    const int64_t zend = z0_of(U - 1);
    add(zend, zend + np_of(U - 1));
    int64_t f = 0;
    int since = 0;
    for (int64_t v = 0; v + 1 < U; ++v) {
      ++since;
      const bool last = v + 2 >= U;
      const bool regular = np_of(v) == sp.unit && !last && np_of(v + 1) == sp.unit && layer_of(v + 1) == layer_of(v);
      if (!(v < head || !regular || since >= merge)) continue;
      int64_t e = last ? zend : z0_of(v + 1);
      if (off && !last && layer_of(v + 1) == layer_of(v)) e = std::min(zend, e + T);
      if (e > f) add(f, e);
      f = std::max(f, e);
      since = 0;
    }
  };
  plan_copies(offset != 0);
  if ((int64_t)cps.size() > G.ntiles) plan_copies(false);  // one ev_in event per copy
  for (size_t k = 0; k < cps.size(); ++k) {
    const Copy& c = cps[k];
    const int is = P.in(0);
    r = X.h2d_part(d, c.layer * lt, lt, bit ? (int)(G.ntiles + c.layer * lt) : (int)(c.layer * lt), c.p0, c.np, is);
    if (r.bad()) return r;
    r = X.record(d, ev_in(d, (int64_t)k), is);
    if (r.bad()) return r;
  }
  // the copy a set of planes waits for: the latest one (one stream, in order)
  auto need = [&](int64_t zlo, int64_t zhi) {
    int k = 0;
    for (int64_t z = zlo; z < zhi; ++z) k = std::max(k, cp_of[(size_t)(((z % nzl) + nzl) % nzl)]);
    return (int64_t)k;
  };
  if (multi) {  // my slab-end planes of initial data to the neighbours, on the halo stream
    for (int side : {1, 0}) {
      r = X.wait(d, ev_in(d, side ? need(nzl - T, nzl) : need(0, T)), hs);
      if (r.bad()) return r;
      r = X.st_halo(d, 0, side, T, hs);
      if (r.bad()) return r;
    }
    r = X.record(d, ev_push, hs);
    if (r.bad()) return r;
  }
  for (int64_t u = 0; u < U; ++u) {
    r = X.wait(d, ev_in(d, need(z0_of(u) - T, z0_of(u) + np_of(u) + T)), cs);
    if (r.bad()) return r;
    if (u >= 2) {  // the ring buffer u%2 was last read by unit u-2's D2H
      r = X.wait(d, ring_ev[u & 1], cs);
      if (r.bad()) return r;
    }
    if (multi)  // the slab-end units read the neighbours' planes (halo layers)
      for (int side : {0, 1})
        if (u == (side ? U - 1 : 0)) {
          r = X.st_halo(d, 1, side, T, cs);
          if (r.bad()) return r;
        }
    // sweep i reads planes [i-1, n+2T-i+1) and writes [i, n+2T-i); the
    // first reads the resident array directly (gather fused), the last writes
    // the unit's packed sub-tiles (scatter fused). On grids 512 wide two
    // sweeps run per kernel (heat2_band_slab, level i kept on chip).
    int cur = -1;  // dense slab holding the last level written (-1: the resident array)
    for (int i = 1; i <= T;) {
      const bool pair = two && i + 1 <= T;
      const int last = pair ? i + 1 : i;  // the level this kernel writes
      const int out = cur == 0 ? 1 : 0;
      const SlabRef src = i == 1 ? SlabRef{SlabRef::RESIDENT, bit, z0_of(u) - T} : SlabRef{SlabRef::DENSE, slab[cur], 0};
      const SlabRef dst = last == T ? SlabRef{SlabRef::SUB, res_of(u), 0} : SlabRef{SlabRef::DENSE, slab[out], 0};
      d.st_unit = np_of(u);  // packed sub-tile depth of the last sweep
      const int hi = (int)(np_of(u) + 2 * T - i);
      r = pair ? X.slab_sweep2s(d, src, dst, i, hi, cs) : X.slab_sweep(d, src, dst, i, hi, cs);
      if (r.bad()) return r;
      if (i == 1 && u >= 2) {  // unit u-1's initial data has no reader left
        r = X.copy_part(d, res_of(u - 1), cur_slot(u - 1), lt, p0_of(u - 1), np_of(u - 1), cs);
        if (r.bad()) return r;
      }
      if (i == 1 && multi)  // halo layers read: their senders may reuse them
        for (int side : {0, 1})
          if (u == (side ? U - 1 : 0)) {
            r = X.st_halo(d, 2, side, T, cs);
            if (r.bad()) return r;
          }
      cur = out;
      i = last + 1;
    }
    r = X.record(d, ev_unit_done(u), cs);
    if (r.bad()) return r;
    r = X.wait(d, ev_unit_done(u), os);
    if (r.bad()) return r;
    r = X.d2h_part(d, layer_of(u) * lt, lt, res_of(u), p0_of(u), np_of(u), os);
    if (r.bad()) return r;
    if (u >= 1) {
      r = X.record(d, ring_ev[u & 1], os);
      if (r.bad()) return r;
    }
  }
  if (multi) {  // the pushes read units 0 and U-1's initial data, overwritten below
    r = X.wait(d, ev_push, cs);
    if (r.bad()) return r;
  }
  if (U >= 2) {
    r = X.copy_part(d, res_of(U - 1), cur_slot(U - 1), lt, p0_of(U - 1), np_of(U - 1), cs);
    if (r.bad()) return r;
  }
  r = X.copy_part(d, keep0, cur_slot(0), lt, p0_of(0), np_of(0), cs);
  if (r.bad()) return r;
  for (int64_t k = 0; k < G.ntiles; ++k) {
    d.tile_dirty[k] = 0;  // the host received u^T through the D2H above
    d.tile_slot[k] = bit ? (int)(G.ntiles + k) : (int)k;
  }
  d.resident_valid = true;
  d.faces_valid = d.xfaces_valid = false;  // faces are re-extracted by the next resident run
  d.last_batches.clear();
  return Status::ok();
}

// ------------------------------------------- out-of-core stream-through
// The stream (out-of-core) schedule streams every tile through the device
// once per step. Temporal blocking: a
// pass of k steps over units of `un` >= k planes needs, per unit, only its
// own and its two neighbour units' data from the host, so each pass moves
// every cell across the link once per direction for k steps. Device memory:
// the input units in a ring (units 0 and U-1 fixed: the periodic wrap reads
// them at both ends), two dense slabs of un + 2k planes, two packed output
// units. (k, un) minimise the same estimate as the resident stream-through
// under the device budget; taken when k >= 2.
struct OocPlan {
  int64_t un = 0, U = 0, k = 0, passes = 0, R = 0;
  int64_t unit_slots = 0, slab_slots = 0;
};

static bool ooc_streamthrough_ok(const Domain& d, int T, OocPlan* op) {
  const Geometry& G = d.G;
  if (d.opt.stream_through < 0 || G.nranks != 1 || G.bc != TILE_BC_PERIODIC || T < 2) return false;
  if (G.t[0] % 2 || G.l[2] > (1 << 30)) return false;
  const double nz = (double)G.l[2];
  const int64_t plane = G.l[0] * G.l[1];
  const double r_sweep = d.r_sweep;
  double best = 1e300;
  for (int64_t k = 2; k <= std::min<int64_t>(T, G.t[2]); ++k)
    for (int64_t un = k; un <= G.t[2]; ++un) {
      if (G.t[2] % un || un < std::min<int64_t>(16, G.t[2])) continue;
      const int64_t U = G.l[2] / un;
      if (U > G.ntiles || U < 4) continue;  // one event per unit; ring of >= 2 besides the wrap units
      const int64_t us = (G.layer_tiles * un * G.t[0] * G.t[1] + G.tile_elems - 1) / G.tile_elems;
      const int64_t ss = ((un + 2 * k) * plane + G.tile_elems - 1) / G.tile_elems;
      // 2 fixed input units + R ring units (4, else 3) + 2 output units + 2 slabs
      const int64_t ring_max = U - 2;
      int64_t R = std::min<int64_t>(4, ring_max);
      if ((4 + R) * us + 2 * ss > d.nslots && R > std::min<int64_t>(3, ring_max)) --R;
      if ((4 + R) * us + 2 * ss > d.nslots) continue;
      const int64_t P = (T + k - 1) / k;
      const double kd = (double)(T + P - 1) / P;  // steps per pass (balanced)
      const double est = (double)P * (std::max(nz, r_sweep * nz * (kd + (kd * kd - kd) / (double)un)) + 3.0 * un);
      if (est < best) {
        best = est;
        op->un = un, op->U = U, op->k = k, op->passes = P, op->R = R, op->unit_slots = us,
        op->slab_slots = ss;
      }
    }
  if (best >= 1e300) return false;
  // the per-step stream schedule moves every cell once per direction per
  // step: T link passes at best
  if (d.opt.stream_through == 0 && best > (double)T * nz) return false;
  return true;
}

static Status run_streamthrough_ooc(Domain& d, int T, int S, const OocPlan& op) {
  Exec& X = *d.exec;
  const Geometry& G = d.G;
  const Pipes P(S, false);
  const int64_t U = op.U, un = op.un, lt = G.layer_tiles, tz = G.t[2], R = op.R;
  const int cs = P.comp(0), os = P.out(0), is = P.in(0);
  d.slab_depth = op.slab_slots * G.tile_elems / (G.l[0] * G.l[1]);  // planes a slab holds
  Status r;
  // flush: dirty resident tiles to the host, then nothing is resident
  {
    Sched sc(d, P);
    for (int64_t t = 0; t < G.ntiles; ++t)
      if (d.tile_slot[t] >= 0 && d.tile_dirty[t]) {
        r = sc.writeback(t);
        if (r.bad()) return r;
      }
  }
  for (int s = 0; s < d.nslots; ++s) {  // every slot's previous use before this run
    r = X.wait(d, ev_slot(d, s), is);
    if (r.bad()) return r;
    r = X.wait(d, ev_slot(d, s), cs);
    if (r.bad()) return r;
  }
  for (int64_t t = 0; t < G.ntiles; ++t) {
    r = X.wait(d, ev_host(d, t), is);  // host copy complete (earlier D2H)
    if (r.bad()) return r;
  }
  // slot layout (unit-sized packed buffers, then slabs)
  const int us = (int)op.unit_slots, ss = (int)op.slab_slots;
  const int F0 = 0, F1 = us, ring0 = 2 * us, out0 = ring0 + (int)R * us;
  const int outb[2] = {out0, out0 + us};
  const int slab[2] = {out0 + 2 * us, out0 + 2 * us + ss};
  auto inbuf = [&](int64_t u) {
    u = (u % U + U) % U;
    if (u == 0) return F0;
    if (u == U - 1) return F1;
    return ring0 + (int)((u - 1) % R) * us;
  };
  auto layer_of = [&](int64_t u) { return (u * un) / tz; };
  auto p0_of = [&](int64_t u) { return (u * un) % tz; };
  const int ring_ev[2] = {d.ev_misc_base + 4 + d.halo_stream + 1, d.ev_misc_base + 5 + d.halo_stream + 1};
  auto h2d_unit = [&](int64_t u, int pass) -> Status {
    if (pass > 0) {
      Status q = X.wait(d, ev_host(d, u), is);  // previous pass's D2H of u
      if (q.bad()) return q;
    }
    Status q = X.h2d_pack(d, layer_of(u) * lt, lt, inbuf(u), p0_of(u), un, is);
    if (q.bad()) return q;
    return X.record(d, ev_in(d, u), is);
  };
  for (int pass = 0; pass < (int)op.passes; ++pass) {
    const int k = (int)(T / op.passes + (pass < T % op.passes ? 1 : 0));
    if (pass > 0) {  // every buffer of the previous pass is free
      r = X.wait(d, ev_tile(d, U - 1, 1), is);
      if (r.bad()) return r;
    }
    // H2D order: the wrap neighbour first, then z order; units 1..R fill the
    // ring, unit u >= R+1 reuses unit u-R's buffer after the first sweep of
    // unit u-R+1 (its last reader)
    std::vector<char> issued((size_t)U, 0);
    auto issue = [&](int64_t u) -> Status {
      if (u < 0 || u >= U || issued[(size_t)u]) return Status::ok();
      issued[(size_t)u] = 1;
      return h2d_unit(u, pass);
    };
    r = issue(U - 1);
    if (r.bad()) return r;
    for (int64_t u = 0; u <= std::min<int64_t>(R, U - 1); ++u) {
      r = issue(u);
      if (r.bad()) return r;
    }
    for (int64_t u = 0; u < U; ++u) {
      for (int64_t du : {(int64_t)-1, (int64_t)0, (int64_t)1}) {
        r = X.wait(d, ev_in(d, (u + du + U) % U), cs);
        if (r.bad()) return r;
      }
      if (u >= 2 || pass > 0) {  // output buffer u%2 was last read by unit u-2's D2H
        r = X.wait(d, ring_ev[u & 1], cs);
        if (r.bad()) return r;
      }
      for (int i = 1; i <= k; ++i) {
        SlabRef src{SlabRef::DENSE, slab[(i - 1) & 1], 0, {0, 0, 0}, 0, 0};
        if (i == 1) src = SlabRef{SlabRef::UNITS, 0, u * un - k, {inbuf(u - 1), inbuf(u), inbuf(u + 1)}, u, un};
        const SlabRef dst = i == k ? SlabRef{SlabRef::SUB, outb[u & 1], 0, {0, 0, 0}, 0, 0}
                                   : SlabRef{SlabRef::DENSE, slab[i & 1], 0, {0, 0, 0}, 0, 0};
        d.st_unit = un;
        r = X.slab_sweep(d, src, dst, i, (int)(un + 2 * k - i), cs);
        if (r.bad()) return r;
        if (i == 1) {
          r = X.record(d, ev_tile(d, u, 0), cs);
          if (r.bad()) return r;
        }
      }
      r = X.record(d, ev_tile(d, u, 1), cs);
      if (r.bad()) return r;
      r = X.wait(d, ev_tile(d, u, 1), os);
      if (r.bad()) return r;
      r = X.d2h_part(d, layer_of(u) * lt, lt, outb[u & 1], p0_of(u), un, os);
      if (r.bad()) return r;
      r = X.record(d, ring_ev[u & 1], os);
      if (r.bad()) return r;
      r = X.record(d, ev_host(d, u), os);
      if (r.bad()) return r;
      // unit u+R's buffer held unit u; its last reader (unit u+1's first
      // sweep) is issued next iteration -> issue H2D(u+R) after that
      if (u >= 2 && u - 1 + R <= U - 2) {
        r = X.wait(d, ev_tile(d, u, 0), is);
        if (r.bad()) return r;
        r = issue(u - 1 + R);
        if (r.bad()) return r;
      }
    }
    for (int64_t u = 0; u < U; ++u) {  // any left (small U)
      r = issue(u);
      if (r.bad()) return r;
    }
  }
  // the host store now holds u^T; nothing is resident. Every slot's and
  // every tile's host events mark the end of this run for later schedules.
  r = X.record(d, ev_phase(d), cs);
  if (r.bad()) return r;
  r = X.wait(d, ev_phase(d), os);
  if (r.bad()) return r;
  for (int s = 0; s < d.nslots; ++s) {
    r = X.record(d, ev_slot(d, s), os);
    if (r.bad()) return r;
  }
  for (int64_t t = 0; t < G.ntiles; ++t) {
    r = X.record(d, ev_host(d, t), os);
    if (r.bad()) return r;
    d.tile_slot[t] = -1;
    d.tile_dirty[t] = 0;
  }
  d.free_slots.clear();
  for (int s = 0; s < d.nslots; ++s) {
    d.slot_owner[s] = -1;
    d.free_slots.push_back(s);
  }
  d.faces_valid = d.xfaces_valid = false;
  d.host_faces_valid = false;
  d.host_pending = true;
  return Status::ok();
}

// ---------------------------------------------------------------- wavefront
// Fresh-upload heat runs beyond the stream-through's reach (T > tz, or where
// its redundant halo sweeps cost more than they save): a
// time-skewed march over chunks of c planes. Level s (the grid after s
// steps) of iteration i covers planes [c*i - s, c*i + c - s), in unwrapped
// coordinates: a plane z < 0 is the ring's top plane nz + z, kept in a
// scratch of whole tile layers. Computing it reads level s-1 on
// [c*i - s - 1, c*i + c - s + 1): level s-1 of the same iteration plus the
// top two planes of iteration i-1. So iteration i depends only on its own
// chunk's upload and on iteration i-1, every cell is updated once per level
// (no redundant halo sweeps), and iteration i's level-T chunk is final when
// the iteration ends: its D2H starts then, while later chunks are still
// uploading. Iteration 0 reads level s-1 at planes -s-1, -s, which the ring
// computes last: a bootstrap trapezoid computes them first from the initial
// data of the top 2T planes (uploaded first) — T sweeps over [-2T + t, -t),
// t = 1..T-1, about T^2 plane updates (the dependency cone of the seam).
// Buffers: level s in resident array bit ^ (s & 1) for z >= 0, in scratch
// parity s & 1 (nlo = ceil(2T / tz) tile layers) for z < 0; level 0 is read
// through the wrapped resident view. Level s+2 overwrites level s only where
// no reader of level s remains (level s+1 of the same iteration runs before
// it; the two planes iteration i+1 reads lie above level s+2's chunk of
// iteration i) — checked on CPU by the random-order replay of the trace.
struct WavePlan {
  bool fused = false;  // two levels per pass (three level buffers)
  int64_t c = 0;    // chunk planes (divides tz)
  int64_t B = 0;    // bootstrap region: the top B planes, uploaded first (multiple of c, >= 2T)
  int64_t nlo = 0;  // scratch tile layers per parity
  double est = 0;   // estimated time in link-plane units (streamthrough_ok's scale)
};

static int64_t wave_chunk() {
  static const int64_t c = [] {
    const char* e = getenv("TILES_WAVE_C");
    return e ? std::max<int64_t>(1, atoll(e)) : (int64_t)32;  // C2 Fig. 5: 32 > 64 > 16 planes
  }();
  return c;
}


static bool wavefront_ok(const Domain& d, int T, WavePlan* wp) {
  const Geometry& G = d.G;
  if (d.opt.wavefront < 0 || G.nranks != 1 || G.bc != TILE_BC_PERIODIC || d.mode != MODE_RESIDENT) return false;
  if (T < 1 || G.t[0] % 2 || G.l[2] > (1 << 28)) return false;
  const int64_t nz = G.l[2], tz = G.t[2];
  int64_t c = std::min<int64_t>(wave_chunk(), tz);
  while (tz % c) --c;
  while (nz / c > G.ntiles) c *= 2;  // one event per chunk (ev_in / ev_host)
  if (tz % c || nz / c > G.ntiles) return false;
  const int64_t B = (2 * (int64_t)T + c - 1) / c * c;
  if (B + c > nz) return false;  // the seam's cone would cover the ring
  const int64_t nlo = (2 * (int64_t)T + tz - 1) / tz;
  // two levels per pass take a third level array (ntiles slots) and three
  // scratch parities, when the budget has them: by default where the band
  // kernel runs them (heat2_band_slab: grids 512 wide), with wavefront = 2
  // everywhere (slab_sweep2_tile elsewhere), never with wavefront = 3
  const uint64_t avail = d.budget_left + (uint64_t)d.wave_slots * G.tile_elems * 8;
  const int64_t slots3 = G.ntiles + 3 * nlo * G.layer_tiles, slots2 = 2 * nlo * G.layer_tiles;
  const bool band = band2_shape_ok(G.l[0], G.l[1], (int)G.t[0], (int)G.t[1]) && d.exec->band2_ok(const_cast<Domain&>(d));
  wp->fused = (d.opt.wavefront == 2 || (d.opt.wavefront != 3 && band)) && T >= 2 &&
              (d.wave_slots >= slots3 || (uint64_t)slots3 * G.tile_elems * 8 <= avail);
  const int64_t need_slots = wp->fused ? slots3 : slots2;
  if (d.wave_slots < need_slots && (uint64_t)need_slots * G.tile_elems * 8 > avail) return false;
  const double r = d.r_sweep, Td = (double)T, n = (double)nz;
  wp->c = c;
  wp->B = B;
  wp->nlo = nlo;
  // the bootstrap waits for the top B planes and sweeps ~T^2 planes; then
  // the march is bound by the link (every plane down once, the rest up) or
  // by its T sweeps per plane; one chunk of fill/drain
  // (the bootstrap's sweeps are thick, about 0.7 of a chunk sweep's cost per
  // plane, fitted on the Fig. 5 sweep at T = 64 and 100)
  const double rm = wp->fused ? 0.6 * r : r;  // two levels per pass: ~0.6 of the sweep time per level (C2: 0.6)
  wp->est = (double)B + 0.7 * r * Td * Td + std::max(n, rm * n * Td) + (double)c * (1.0 + rm * Td);
  return true;
}

static Status ensure_wave_scratch(Domain& d, int64_t slots) {
  if (d.wave_slots >= slots) return Status::ok();
  // room for up to 4 tile layers per parity when the budget allows, so runs
  // with growing T do not reallocate (a reallocation synchronises)
  const int64_t roomy = 2 * std::min<int64_t>(4, d.G.n[2] / 2) * d.G.layer_tiles;
  const uint64_t avail = d.budget_left + (uint64_t)d.wave_slots * d.G.tile_elems * 8;
  if (roomy > slots && (uint64_t)roomy * d.G.tile_elems * 8 <= avail / 2) slots = roomy;
  const uint64_t bytes = (uint64_t)slots * d.G.tile_elems * 8;
  if (d.own_wave && d.wave_base) {
    Status r = d.exec->sync_all(d);  // the old scratch may still be read
    if (r.bad()) return r;
    d.exec->free_device(d, d.wave_base);
    d.budget_left += (uint64_t)d.wave_slots * d.G.tile_elems * 8;
    d.wave_base = nullptr;
    d.wave_slots = 0;
  }
  if (bytes > d.budget_left) return make_err(TILE_ENOMEM_DEVICE, "wavefront scratch exceeds the device budget");
  if (d.opt.device_pool) {  // the caller's pool: its tail past the domain's carve
    d.wave_base = reinterpret_cast<double*>(d.pool + d.pool_bytes);
    d.own_wave = false;
  } else {
    void* p = nullptr;
    Status r = d.exec->alloc_device(d, bytes, &p);
    if (r.bad()) return r;
    d.wave_base = static_cast<double*>(p);
    d.own_wave = true;
  }
  d.budget_left -= bytes;
  d.wave_slots = (int)slots;
  return Status::ok();
}

// h2d = false: level 0 is already in the resident array (no uploads; the
// upload events are still recorded); d2h = false: the chunks' level-T planes
// stay on the device (no D2H; the tiles are left dirty for tile_sync). The
// large-T fresh-upload schedule runs the wavefront twice this way around the
// resident two-step passes (run_heat_resident).
static Status run_wavefront(Domain& d, int T, int S, const WavePlan& wp, bool h2d = true, bool d2h = true) {
  Exec& X = *d.exec;
  const Geometry& G = d.G;
  const int64_t nz = G.l[2], tz = G.t[2], lt = G.layer_tiles, c = wp.c, B = wp.B, nlo = wp.nlo;
  const int64_t U = nz / c, iB = (nz - B) / c;  // iterations; first chunk inside the bootstrap region
  // level buffers: two (level s in array bit ^ (s & 1)) or, with two levels
  // per pass, three (s % 3: the arrays bit, bit ^ 1 and a third one in the
  // wave scratch) — a fused pass writes level s+1 while its other CTAs still
  // read level s-1, so the two may not share memory. Scratch parities for
  // planes z < 0 likewise.
  const int nbuf = wp.fused ? 3 : 2;
  Status r = ensure_wave_scratch(d, wp.fused ? G.ntiles + 3 * nlo * lt : 2 * nlo * lt);
  if (r.bad()) return r;
  const Pipes P(S, false);
  const int cs = P.comp(0), os = P.out(0), is = P.in(0);
  const int bit = d.res_bit;
  const int arrA = bit ? (int)G.ntiles : 0, arrB = bit ? 0 : (int)G.ntiles;
  const int sc0 = d.nslots + (wp.fused ? (int)G.ntiles : 0);
  const int arr[3] = {arrA, arrB, d.nslots};
  const int scr[3] = {sc0, sc0 + (int)(nlo * lt), sc0 + 2 * (int)(nlo * lt)};
  const int ib = T % nbuf;                  // buffer holding level T
  const int fin = ib == 1 ? bit ^ 1 : bit;  // resident array that ends up holding it
  auto arr0 = [&](int a, int64_t L) { return (int)((a ? G.ntiles : 0) + L * lt); };
  // planes [z0, z1) of the ring (physical, 0 <= z0 < z1 <= nz) in tile-layer pieces
  auto pieces = [&](int64_t z0, int64_t z1, auto&& f) -> Status {
    for (int64_t z = z0; z < z1;) {
      const int64_t L = z / tz, lz = z - L * tz, np = std::min(z1 - z, tz - lz);
      Status q = f(L, lz, np);
      if (q.bad()) return q;
      z += np;
    }
    return Status::ok();
  };
  auto upload = [&](int64_t z0, int64_t z1) {
    if (!h2d) return Status::ok();
    return pieces(z0, z1, [&](int64_t L, int64_t lz, int64_t np) {
      return X.h2d_part(d, L * lt, lt, arr0(bit, L), lz, np, is);
    });
  };
  // Uploads on one copy-in stream: the seam's cone [-B, 0) in chunks going
  // down from the seam (region chunk k = planes [-(k+1)c, -kc) = ring chunk
  // U-1-k), chunk 0 right after the first of them, then chunks 1.. in march
  // order. The bootstrap runs in rounds as the region chunks land (a
  // downward skewed march: round k extends level t to [-(k+1)c + t, ...)),
  // and iteration 0's level s runs as soon as its seam strip (level s-1 at
  // planes -s-1, -s, complete once (k+1)c >= 2s) exists, so the bootstrap's
  // compute overlaps the cone's upload instead of following it.
  const int64_t nB = B / c;
  auto region_chunk = [&](int64_t k) { return U - 1 - k; };
  for (int64_t k = 0; k < nB; ++k) {
    const int64_t ch = region_chunk(k);
    r = upload(ch * c, (ch + 1) * c);
    if (r.bad()) return r;
    r = X.record(d, ev_in(d, ch), is);
    if (r.bad()) return r;
    if (k == 0 && iB > 0) {
      r = upload(0, c);
      if (r.bad()) return r;
      r = X.record(d, ev_in(d, 0), is);
      if (r.bad()) return r;
    }
  }
  for (int64_t i = 1; i < iB; ++i) {
    r = upload(i * c, (i + 1) * c);
    if (r.bad()) return r;
    r = X.record(d, ev_in(d, i), is);
    if (r.bad()) return r;
  }
  auto lvl = [&](int s) {  // view of level s (s = 0: the initial data, wrapped)
    const int k = s % nbuf;
    return s == 0 ? SlabRef{SlabRef::RESIDENT, bit, 0, {0, 0, 0}, 0, 0}
                  : SlabRef{SlabRef::WAVE, arr[k], 0, {scr[k], 0, 0}, 0, nlo};
  };
  auto level_of_iteration = [&](int64_t i, int s) {
    return X.slab_sweep(d, lvl(s - 1), lvl(s), (int)(c * i - s), (int)(c * i + c - s), cs);
  };
  // levels s, s+1 of iteration i in one pass
  auto levels_of_iteration = [&](int64_t i, int s) {
    return X.slab_sweep2(d, lvl(s - 1), lvl(s), lvl(s + 1), (int)(c * i - s), (int)(c * i + c - s), cs);
  };
  // the next pass of an iteration from level s: two levels when fused; returns the levels done
  auto pass_of_iteration = [&](int64_t i, int s, int* done) {
    if (wp.fused && s + 1 <= T) {
      *done = 2;
      return levels_of_iteration(i, s);
    }
    *done = 1;
    return level_of_iteration(i, s);
  };
  // bootstrap rounds, with iteration 0's levels interleaved
  int s0 = 1;  // next level of iteration 0
  for (int64_t k = 0; k < nB; ++k) {
    r = X.wait(d, ev_in(d, region_chunk(k)), cs);
    if (r.bad()) return r;
    for (int t = 1; t < T; ++t) {  // level t over [-2T + t, -t), the part this chunk makes computable
      const int64_t lo = std::max<int64_t>(-2 * (int64_t)T + t, -(k + 1) * c + t);
      const int64_t hi = std::min<int64_t>(-t, -k * c + t);
      const int64_t lo_prev = std::max<int64_t>(-2 * (int64_t)T + t, -k * c + t);  // computed before
      const int64_t h = k == 0 ? hi : std::min(hi, lo_prev);
      if (lo < h) {
        r = X.slab_sweep(d, lvl(t - 1), lvl(t), (int)lo, (int)h, cs);
        if (r.bad()) return r;
      }
    }
    if (k == 0 && iB > 0) {
      r = X.wait(d, ev_in(d, 0), cs);
      if (r.bad()) return r;
    }
    // iteration 0's levels whose seam strips are complete: level s needs
    // level s-1 at -s-1, -s, i.e. (k+1)c >= 2s (level 0: region chunk 0); a
    // fused pass (s, s+1) also level s at -s-2, -s-1: (k+1)c >= 2(s+1)
    while (s0 <= T) {
      const int last = (wp.fused && s0 + 1 <= T) ? s0 + 1 : s0;
      if ((k + 1) * c < 2 * (int64_t)last) break;
      int done = 0;
      r = pass_of_iteration(0, s0, &done);
      if (r.bad()) return r;
      s0 += done;
    }
  }
  while (s0 <= T) {
    int done = 0;
    r = pass_of_iteration(0, s0, &done);
    if (r.bad()) return r;
    s0 += done;
  }
  // the march
  for (int64_t i = 0; i < U; ++i) {
    if (i > 0) {
      if (i < iB) {
        r = X.wait(d, ev_in(d, i), cs);
        if (r.bad()) return r;
      }
      int s = 1;
      if (wp.fused && T >= 2 && X.wave_iter_ok(d)) {  // every pair of levels in one launch
        const SlabRef lv[4] = {lvl(3), lvl(1), lvl(2), lvl(0)};
        r = X.wave_iteration(d, lv, c * i, (int)c, 1, T / 2, cs);
        if (r.bad()) return r;
        s = 2 * (T / 2) + 1;
      }
      while (s <= T) {
        int done = 0;
        r = pass_of_iteration(i, s, &done);
        if (r.bad()) return r;
        s += done;
      }
    }
    if (!d2h) continue;
    r = X.record(d, ev_host(d, i), cs);
    if (r.bad()) return r;
    r = X.wait(d, ev_host(d, i), os);
    if (r.bad()) return r;
    // level-T planes [c*i - T, c*i + c - T): z < 0 from the scratch (the
    // ring's top planes), z >= 0 from the resident array
    const int64_t a = c * i - T, b = c * i + c - T;
    if (a < 0) {
      r = pieces(nz + a, nz + std::min<int64_t>(b, 0), [&](int64_t L, int64_t lz, int64_t np) {
        const int64_t Ls = L - (nz / tz - nlo);  // scratch layer of physical layer L
        return X.d2h_planes(d, L * lt, lt, scr[ib] + (int)(Ls * lt), lz, np, os);
      });
      if (r.bad()) return r;
    }
    if (b > 0) {
      r = pieces(std::max<int64_t>(a, 0), b, [&](int64_t L, int64_t lz, int64_t np) {
        return X.d2h_planes(d, L * lt, lt, arr[ib] + (int)(L * lt), lz, np, os);
      });
      if (r.bad()) return r;
    }
  }
  // leave the domain resident at level T: the ring's top T planes from the
  // scratch (and, when level T is in the third array, the rest from it)
  r = pieces(nz - T, nz, [&](int64_t L, int64_t lz, int64_t np) {
    const int64_t Ls = L - (nz / tz - nlo);
    return X.copy_planes(d, scr[ib] + (int)(Ls * lt), arr0(fin, L), lt, lz, np, cs);
  });
  if (r.bad()) return r;
  if (ib == 2) {
    r = pieces(0, nz - T, [&](int64_t L, int64_t lz, int64_t np) {
      return X.copy_planes(d, arr[2] + (int)(L * lt), arr0(fin, L), lt, lz, np, cs);
    });
    if (r.bad()) return r;
  }
  d.res_bit = fin;
  for (int64_t k = 0; k < G.ntiles; ++k) {
    d.tile_dirty[k] = d2h ? 0 : 1;  // with d2h the host received u^T through the D2H above
    d.tile_slot[k] = fin ? (int)(G.ntiles + k) : (int)k;
  }
  d.resident_valid = true;
  d.faces_valid = d.xfaces_valid = false;  // faces are re-extracted by the next resident run
  d.last_batches.clear();
  if (!d2h) {  // tile_sync copies the whole grid back after this run's last kernel
    const int ev = ev_layer(d, 0, 0);
    r = X.record(d, ev, cs);
    if (r.bad()) return r;
    d.last_batches.push_back({0, G.n[2], cs, os, ev});
  }
  return Status::ok();
}

// Two steps per kernel over the resident periodic grid (heat2_band,
// DESIGN.md §4): the whole grid is one kernel's work, so each pass reads u^s
// and writes u^{s+2} once (16 B per cell for two steps) and needs no faces;
// the faces go stale (re-extracted by the next face-reading run).
// TILES_BAND2=0 turns it off.
static bool band2_fits(Domain& d, bool serial) {
  static const int on = [] {
    const char* e = getenv("TILES_BAND2");
    return e ? atoi(e) : 1;
  }();
  const Geometry& G = d.G;
  return on && !serial && d.opt.two_step >= 0 && G.nranks == 1 && G.bc == TILE_BC_PERIODIC &&
         d.mode == MODE_RESIDENT && !d.user_fn && band2_shape_ok(G.l[0], G.l[1], (int)G.t[0], (int)G.t[1]) &&
         d.exec->band2_ok(d);
}
static bool band2_use(Domain& d, int steps, bool load, bool serial) {
  return !load && steps >= 2 && band2_fits(d, serial);
}

static Status run_band2(Domain& d, int steps, int S) {
  Exec& X = *d.exec;
  const Geometry& G = d.G;
  int bit = d.res_bit;
  for (int s = 0; s + 1 < steps; s += 2) {  // stream 0: every stream was joined into it (domain_run)
    Status r = X.band2(d, bit, bit ^ 1, 0);
    if (r.bad()) return r;
    bit ^= 1;
  }
  const int ev = ev_layer(d, 0, 0);
  Status r = X.record(d, ev, 0);
  if (r.bad()) return r;
  d.res_bit = bit;
  d.resident_valid = true;
  d.faces_valid = d.xfaces_valid = false;
  for (int64_t k = 0; k < G.ntiles; ++k) {
    d.tile_slot[k] = bit == 0 ? (int)k : (int)(G.ntiles + k);
    d.tile_dirty[k] = 1;
  }
  d.last_batches.clear();
  d.last_batches.push_back({0, G.n[2], 0, Pipes(S, false).out(0), ev});
  return Status::ok();
}

static Status run_heat_resident(Domain& d, double alpha, int steps, int S, bool serial) {
  const bool load = !d.resident_valid;
  if (band2_use(d, steps, load, serial)) {
    Status r = run_band2(d, steps & ~1, S);
    if (r.bad()) return r;
    if (steps & 1) r = run_heat_resident(d, alpha, 1, S, serial);  // the odd step: face-ghost single step
    d.last_schedule = 7;
    return r;
  }
  const int64_t nL = d.G.n[2];
  StreamPlan sp{};
  if (load && !serial) {  // fresh upload: stream-through, wavefront or the batched schedule
    double est_st = 0;
    WavePlan wp;
    const bool st = streamthrough_ok(d, steps, &sp, &est_st);
    const bool wf = wavefront_ok(d, steps, &wp);
    const double nz = (double)d.G.l[2];
    // the batched schedule: both link directions in sequence plus T
    // whole-domain steps partly overlapped (0.52 r per plane-step: the
    // persistent heat7 step per plane over the duplex link-plane time, fitted
    // with r on the Fig. 5 sweep)
    // (0.6 r when the middle steps run two per kernel on heat2_band, fitted
    // on the Fig. 5 sweep with heat2_band: T = 100 58.8 ms, T = 1000 257 ms;
    // the wavefront's 53.4 ms wins at T = 100)
    const double est_batched = 2.0 * nz + (band2_fits(d, serial) ? 0.6 : 0.52) * d.r_sweep * nz * steps;
    bool take_wf = wf && (d.opt.wavefront > 0 || (d.opt.stream_through <= 0 && wp.est < est_batched &&
                                                  (!st || wp.est < est_st)));
    bool take_st = !take_wf && st && (d.opt.stream_through > 0 || est_st < est_batched);
    if (take_wf) {
      d.last_schedule = 6;
      return run_wavefront(d, steps, S, wp);
    }
    if (take_st) {
      d.last_schedule = 2;
      return run_streamthrough(d, alpha, steps, S, sp);
    }
    // large T (the batched schedule's range): a wavefront of Tw levels while
    // the grid uploads (nothing downloaded), the middle steps two per kernel
    // on the resident grid, and a wavefront of the last Tw (+1) levels while
    // it downloads (nothing uploaded) — both link directions overlap compute
    // instead of bracketing it (TILES_WAVE_SPLIT=0: the batched schedule)
    static const int split = [] {
      const char* e = getenv("TILES_WAVE_SPLIT");
      return e ? atoi(e) : 1;
    }();
    if (split && d.opt.wavefront >= 0 && band2_fits(d, serial)) {
      int Tw = 64;
      WavePlan w0;
      while (Tw >= 8 && !wavefront_ok(d, Tw, &w0)) Tw /= 2;
      const int mid = steps - 2 * Tw;
      WavePlan w1;
      if (Tw >= 8 && mid >= 2 && wavefront_ok(d, Tw + (mid & 1), &w1)) {
        Status r = run_wavefront(d, Tw, S, w0, true, false);
        if (r.bad()) return r;
        r = run_band2(d, mid & ~1, S);
        if (r.bad()) return r;
        r = run_wavefront(d, Tw + (mid & 1), S, w1, false, true);
        d.last_schedule = 8;
        return r;
      }
    }
  }
  d.last_schedule = serial ? 5 : 1;
  const std::vector<int> kp = plan_passes(d, steps);
  const int T = (int)kp.size();  // passes
  struct Phase {
    int steps;
    bool layered;
    bool band2;  // whole-domain steps two per kernel (heat2_band, stream 0)
  };
  std::vector<Phase> ph;
  if (serial || !load) {
    ph.push_back({T, false, false});
  } else {
    const int k1 = (int)std::min<int64_t>(T, nL / 2 + 1);
    const int mid = T - k1 - 1;
    const bool all1 = std::find(kp.begin(), kp.end(), 2) == kp.end();
    if (T <= k1 + 1) {
      ph.push_back({T, true, false});
    } else if (mid >= 2 && all1 && band2_fits(d, serial)) {
      // the middle steps in pairs on heat2_band, an odd one with the last step
      ph.push_back({k1, true, false});
      ph.push_back({mid & ~1, false, true});
      ph.push_back({1 + (mid & 1), true, false});
    } else {
      ph.push_back({k1, true, false});
      ph.push_back({mid, false, false});
      ph.push_back({1, true, false});
    }
  }
  int bit = d.res_bit, fp = d.face_parity;
  // passes of two steps read every face; direct single steps only the x faces
  const bool any_x2 = std::find(kp.begin(), kp.end(), 2) != kp.end();
  std::vector<std::pair<Batch, int>> last;  // batches of the last phase + final event
  size_t pass0 = 0;
  for (size_t pi = 0; pi < ph.size(); ++pi) {
    if (ph[pi].band2) {  // after the join below (stream 0 waited for every batch)
      for (int s = 0; s + 1 < ph[pi].steps; s += 2) {
        Status r = d.exec->band2(d, bit, bit ^ 1, 0);
        if (r.bad()) return r;
        bit ^= 1;
      }
      pass0 += (size_t)ph[pi].steps;
      d.faces_valid = d.xfaces_valid = false;  // the next phase re-extracts them
      Status r = d.exec->record(d, ev_phase(d), 0);
      if (r.bad()) return r;
      continue;
    }
    ResidentRun R(d);
    R.alpha = alpha;
    R.T = ph[pi].steps;
    R.kpass.assign(kp.begin() + (long)pass0, kp.begin() + (long)(pass0 + (size_t)R.T));
    pass0 += (size_t)R.T;
    R.need_load = pi == 0 && load;
    R.need_extract = (pi == 0 || ph[pi - 1].band2) && !(any_x2 || !d.direct_ok ? d.faces_valid : d.xfaces_valid);
    R.multi = d.G.nranks > 1;
    R.entry_wait = pi > 0;
    R.bit0 = bit;
    R.fp0 = fp;
    R.build(S, serial, ph[pi].layered);
    Status r = R.run();
    if (r.bad()) return r;
    bit ^= (R.T & 1);
    fp ^= (R.T & 1);
    last.clear();
    for (size_t i = 0; i < R.B.size(); ++i)
      last.push_back({R.B[i], ev_layer(d, (int64_t)i, R.T > 0 ? (R.T - 1) & 1 : 1)});
    if (pi + 1 < ph.size()) {  // join: stream 0 waits for every batch, then ev_phase
      for (auto& e : last) {
        r = d.exec->wait(d, e.second, 0);
        if (r.bad()) return r;
      }
      r = d.exec->record(d, ev_phase(d), 0);
      if (r.bad()) return r;
    }
  }
  d.res_bit = bit;
  d.face_parity = fp;
  d.resident_valid = true;
  if (T > 0) {  // a direct last pass leaves the y/z exports stale
    d.xfaces_valid = true;
    d.faces_valid = kp.back() == 2 || !d.direct_ok;
  }
  for (int64_t k = 0; k < d.G.ntiles; ++k) {
    d.tile_slot[k] = bit == 0 ? (int)k : (int)(d.G.ntiles + k);
    if (T > 0) d.tile_dirty[k] = 1;
  }
  // where each layer's last kernel ran and its event (for tile_sync's D2H)
  d.last_batches.clear();
  for (auto& e : last) d.last_batches.push_back({e.first.L0, e.first.L1, e.first.stream, e.first.out, e.second});
  return Status::ok();
}

// -------------------------------------------------- streaming (out-of-core)
static Status run_stream(Domain& d, const tile_kernel& k, int T, int S) {
  Exec& X = *d.exec;
  const Geometry& G = d.G;
  const Pipes P(S, false);
  Sched sc(d, P);
  const bool heat = k.kind == TILE_KERNEL_HEAT7 || k.kind == TILE_KERNEL_USER_STENCIL;
  const bool fuse = !heat && d.opt.fuse_pointwise_steps;
  const std::vector<int> kp = heat ? plan_passes(d, T) : std::vector<int>();
  const int passes = heat ? (int)kp.size() : fuse ? (T > 0 ? 1 : 0) : T;
  const int64_t iters = fuse ? (int64_t)k.inner_iters * T : k.inner_iters;
  const int64_t N = G.ntiles;
  const bool multi = G.nranks > 1;
  Status r;

  if (d.host_pending) {  // host store still being written by an earlier run
    r = X.sync_all(d);
    if (r.bad()) return r;
    d.host_pending = false;
  }
  if (heat && !d.faces_valid) {
    if (!d.host_faces_valid) {
      // the faces come from the host store, so it must hold every tile's
      // current values first: tiles still dirty on the device (an earlier
      // pointwise run's kept window) are written back — GPU-disabled
      // requests, P:L90 — and every queued D2H completes
      for (int64_t t = 0; t < N; ++t) {
        if (!d.tile_dirty[t] || d.tile_slot[t] < 0) continue;
        r = sc.writeback(t);
        if (r.bad()) return r;
      }
      r = X.sync_all(d);
      if (r.bad()) return r;
      d.host_pending = false;
      host_extract_faces(G, d.host, d.host_faces);
      d.host_faces_valid = true;
    }
    r = X.faces_h2d(d, d.face_parity, 0);
    if (r.bad()) return r;
    r = X.record(d, ev_faces_init(d), 0);
    if (r.bad()) return r;
    d.faces_valid = d.xfaces_valid = true;
  } else if (heat) {
    r = X.record(d, ev_faces_init(d), 0);
    if (r.bad()) return r;
  }
  const int fp0 = d.face_parity;
  auto issue_halo = [&](int s) -> Status {  // faces written at pass s (s=-1: current)
    const int hs = d.halo_stream;
    for (int64_t t = 0; t < N; ++t) {
      int64_t ix, iy, iz;
      G.tile_coords(t, &ix, &iy, &iz);
      if (iz != 0 && iz != G.n[2] - 1) continue;
      Status q = X.wait(d, s < 0 ? ev_faces_init(d) : ev_tile(d, t, s & 1), hs);
      if (q.bad()) return q;
    }
    Status q = X.halo(d, fp0 ^ ((s + 1) & 1), hs);
    if (q.bad()) return q;
    return X.record(d, ev_halo(d, s & 1), hs);
  };
  if (heat && multi && passes > 0) {
    r = issue_halo(-1);
    if (r.bad()) return r;
  }

  // keep window: the last W tiles of a pass stay dirty on the device; the
  // snake order makes them the first (cache hits) of the next pass.
  const int64_t W = std::max<int64_t>(0, std::min<int64_t>(N - 1, d.nslots - 4 * (int64_t)S - 2));
  for (int s = 0; s < passes; ++s) {
    const int rp = fp0 ^ (s & 1);
    for (int64_t j = 0; j < N; ++j) {
      const int64_t t = (s & 1) ? N - 1 - j : j;
      const int st = P.comp(t);
      int in = d.tile_slot[t];
      if (in >= 0) {
        d.stats.hits++;
        r = X.note(d, TILE_OP_HIT, t, in, st);
        if (r.bad()) return r;
      } else {
        d.stats.misses++;
        const int is = P.in(t);
        r = sc.acquire(t, is, -1, &in);
        if (r.bad()) return r;
        r = X.wait(d, ev_host(d, t), is);  // host copy of t complete (previous D2H)
        if (r.bad()) return r;
        r = X.h2d(d, t, 1, in, is);
        if (r.bad()) return r;
        r = X.record(d, ev_slot(d, in), is);
        if (r.bad()) return r;
        d.tile_slot[t] = in;
        d.tile_dirty[t] = 0;
        sc.touch(t);
      }
      r = X.wait(d, ev_slot(d, in), st);  // after the slot's previous op (H2D or D2H)
      if (r.bad()) return r;
      if (heat) {
        int out;
        r = sc.acquire(t, st, in, &out);
        if (r.bad()) return r;
        // ghost sources: neighbours' previous pass (RAW) and their reads of
        // the parity this kernel overwrites (WAR)
        bool halo_wait = false;
        for (int f = 0; f < 6; ++f) {
          FaceSrc fs = face_source(G, t, f);
          if (fs.kind == 0 && fs.val != t) {
            r = X.wait(d, s == 0 ? ev_faces_init(d) : ev_tile(d, fs.val, (s - 1) & 1), st);
            if (r.bad()) return r;
          } else if (fs.kind >= 2) {
            halo_wait = true;
          }
        }
        if (s == 0) {
          r = X.wait(d, ev_faces_init(d), st);
          if (r.bad()) return r;
        }
        if (halo_wait && multi) {
          r = X.wait(d, ev_halo(d, (s - 1) & 1), st);
          if (r.bad()) return r;
        }
        const int64_t tl[1] = {t};
        const int is[1] = {in}, os[1] = {out};
        r = kp[(size_t)s] == 2 ? X.heat2(d, tl, is, os, 1, rp, nullptr, st)
                               : X.heat(d, tl, is, os, 1, rp, nullptr, st);
        if (r.bad()) return r;
        r = X.record(d, ev_tile(d, t, s & 1), st);
        if (r.bad()) return r;
        r = X.record(d, ev_slot(d, in), st);
        if (r.bad()) return r;
        r = X.record(d, ev_slot(d, out), st);
        if (r.bad()) return r;
        sc.release(in);
        d.tile_slot[t] = out;
        d.slot_owner[out] = (int)t;
      } else {
        r = X.sincos(d, t, in, iters, st);
        if (r.bad()) return r;
        r = X.record(d, ev_slot(d, in), st);
        if (r.bad()) return r;
      }
      d.tile_dirty[t] = 1;
      sc.touch(t);
      if (j < N - W) {
        r = sc.writeback(t);
        if (r.bad()) return r;
      }
    }
    if (heat && multi && s < passes - 1) {
      r = issue_halo(s);
      if (r.bad()) return r;
    }
  }
  if (heat) d.face_parity ^= (passes & 1);
  return Status::ok();
}

// ------------------------------------------------------------ public runs
static Status upload_dirichlet_if_needed(Domain& d) {
  if (d.G.bc != TILE_BC_DIRICHLET || d.dir_uploaded) return Status::ok();
  Status r = d.exec->upload_dir(d);
  if (r.bad()) return r;
  d.dir_uploaded = true;
  return Status::ok();
}

Status domain_run(Domain& d, const tile_kernel& k, int steps, int nstreams) {
  if (k.kind == TILE_KERNEL_HEAT7) {
    if (!(k.alpha > 0.0 && k.alpha <= 1.0 / 6.0))
      return make_err(TILE_EINVAL, "HEAT7 alpha must be in (0, 1/6]");
  } else if (k.kind == TILE_KERNEL_SINCOS || k.kind == TILE_KERNEL_USER) {
    if (k.inner_iters < 0) return make_err(TILE_EINVAL, "inner_iters must be >= 0");
    if (k.kind == TILE_KERNEL_USER && !d.user_fn) return make_err(TILE_EINVAL, "USER kernel without a function");
  } else if (k.kind == TILE_KERNEL_USER_STENCIL) {
    if (!d.user_fn) return make_err(TILE_EINVAL, "USER_STENCIL kernel without a function");
    if (d.G.ghost != 1) return make_err(TILE_EINVAL, "USER_STENCIL: ghost = 1 only");
  } else {
    return make_err(TILE_EINVAL, "unknown kernel kind");
  }
  if (steps < 0) return make_err(TILE_EINVAL, "steps must be >= 0");
  if (nstreams < 1 || nstreams > 64) return make_err(TILE_EINVAL, "nstreams must be in [1, 64]");
  d.kernel_alpha = k.alpha;
  Status r = upload_dirichlet_if_needed(d);
  if (r.bad()) return r;
  const bool serial = d.opt.sched == TILE_SCHED_SYNC;
  const int S = serial ? 1 : nstreams;
  const Pipes P(S, serial);
  r = join_streams(d, std::max(P.used(), d.streams_used));
  if (r.bad()) return r;
  d.streams_used = std::max(d.streams_used, P.used());
  d.last_S = S;
  d.last_serial = serial;
  d.in_flight = true;
  if (k.kind == TILE_KERNEL_USER_STENCIL) {
    // the heat kernel's specialised paths (direct ghosts, persistent and
    // two-step launches, stream-through sweeps) compute HEAT7 itself: a user
    // stencil runs the face-ghost single-step schedule of the same machinery
    // z-slab ranks exchange the exported slab-end faces by copies (the fused
    // transport's in-kernel push is HEAT7's; its exchange counters are
    // monotonic, so copy and fused exchanges interleave across runs)
    const bool direct = d.direct_ok, persist = d.persist_ok, x2 = d.x2_ok, fused = d.peer_fused;
    const int32_t st_opt = d.opt.stream_through, wf_opt = d.opt.wavefront;
    d.direct_ok = d.persist_ok = d.x2_ok = d.peer_fused = false;
    d.opt.stream_through = d.opt.wavefront = -1;
    r = d.mode == MODE_RESIDENT ? run_heat_resident(d, 0.0, steps, S, serial) : run_stream(d, k, steps, S);
    d.direct_ok = direct;
    d.persist_ok = persist;
    d.x2_ok = x2;
    d.peer_fused = fused;
    d.opt.stream_through = st_opt;
    d.opt.wavefront = wf_opt;
    if (r.bad()) return r;
    d.stats.steps_done += (uint64_t)steps;
    return Status::ok();
  }
  if (k.kind == TILE_KERNEL_HEAT7 && d.mode == MODE_RESIDENT) {
    r = run_heat_resident(d, k.alpha, steps, S, serial);
  } else if (d.mode == MODE_RESIDENT) {
    // pointwise kernel on resident tiles: per-tile H2D -> kernel, in place
    Exec& X = *d.exec;
    const bool fuse = d.opt.fuse_pointwise_steps;
    const int passes = fuse ? (steps > 0 ? 1 : 0) : steps;
    const int64_t iters = fuse ? (int64_t)k.inner_iters * steps : k.inner_iters;
    for (int s = 0; s < passes; ++s)
      for (int64_t t = 0; t < d.G.ntiles; ++t) {
        const int st = P.comp(t);
        const int slot = (int)(d.res_bit == 0 ? t : d.G.ntiles + t);
        if (!d.resident_valid && s == 0) {
          r = X.h2d(d, t, 1, slot, P.in(t));
          if (r.bad()) return r;
          if (P.in(t) != st) {
            r = X.record(d, ev_in(d, t), P.in(t));
            if (r.bad()) return r;
            r = X.wait(d, ev_in(d, t), st);
            if (r.bad()) return r;
          }
        }
        r = X.sincos(d, t, slot, iters, st);
        if (r.bad()) return r;
        r = X.record(d, ev_tile(d, t, 0), st);
        if (r.bad()) return r;
      }
    if (passes > 0) {
      d.resident_valid = true;
      d.faces_valid = d.xfaces_valid = false;  // interiors changed without faces
      for (int64_t t = 0; t < d.G.ntiles; ++t) {
        d.tile_slot[t] = (int)(d.res_bit == 0 ? t : d.G.ntiles + t);
        d.tile_dirty[t] = 1;
      }
      d.last_batches.clear();
      for (int64_t L = 0; L < d.G.n[2]; ++L) d.last_batches.push_back({L, L + 1, -1, -1, -1});
    }
  } else {
    OocPlan op;
    if (k.kind == TILE_KERNEL_HEAT7 && !serial && ooc_streamthrough_ok(d, steps, &op)) {
      d.last_schedule = 4;
      r = run_streamthrough_ooc(d, steps, S, op);
    } else {
      d.last_schedule = serial ? 5 : 3;
      r = run_stream(d, k, steps, S);
      if (k.kind != TILE_KERNEL_HEAT7 && steps > 0) {
        // tiles changed without their faces (device or host copies)
        d.faces_valid = d.xfaces_valid = false;
        d.host_faces_valid = false;
      }
    }
  }
  if (r.bad()) return r;
  if (k.kind == TILE_KERNEL_HEAT7) d.stats.steps_done += (uint64_t)steps;
  return Status::ok();
}

// -------------------------------------------------------------- sync/store
Status domain_sync(Domain& d) {
  Exec& X = *d.exec;
  Status r;
  if (d.mode == MODE_RESIDENT) {
    for (auto& b : d.last_batches) {
      const int64_t t0 = b.L0 * d.G.layer_tiles, n = (b.L1 - b.L0) * d.G.layer_tiles;
      bool any = false;
      for (int64_t t = t0; t < t0 + n; ++t) any |= d.tile_dirty[t] != 0;
      if (!any) continue;
      if (b.stream >= 0) {
        if (b.out != b.stream) {
          r = X.wait(d, b.ev, b.out);  // after the batch's last kernel
          if (r.bad()) return r;
        }
        r = X.d2h(d, t0, n, d.tile_slot[t0], b.out);
        if (r.bad()) return r;
      } else {  // per-tile pipelines (pointwise kernel)
        const Pipes P(d.last_S, d.last_serial);
        for (int64_t t = t0; t < t0 + n; ++t) {
          r = X.wait(d, ev_tile(d, t, 0), P.out(t));
          if (r.bad()) return r;
          r = X.d2h(d, t, 1, d.tile_slot[t], P.out(t));
          if (r.bad()) return r;
        }
      }
      for (int64_t t = t0; t < t0 + n; ++t) d.tile_dirty[t] = 0;
    }
  } else {
    const Pipes P(d.last_S, false);
    for (int64_t t = 0; t < d.G.ntiles; ++t) {
      if (!d.tile_dirty[t] || d.tile_slot[t] < 0) continue;
      const int st = P.out(t);
      const int sl = d.tile_slot[t];
      r = X.wait(d, ev_slot(d, sl), st);
      if (r.bad()) return r;
      r = X.d2h(d, t, 1, sl, st);
      if (r.bad()) return r;
      d.tile_dirty[t] = 0;
      r = X.record(d, ev_slot(d, sl), st);
      if (r.bad()) return r;
      r = X.record(d, ev_host(d, t), st);
      if (r.bad()) return r;
    }
  }
  r = X.sync_all(d);
  if (r.bad()) return r;
  d.in_flight = false;
  d.host_pending = false;
  d.host_faces_valid = false;  // host store changed
  return Status::ok();
}

Status domain_invalidate(Domain& d) {
  if (d.in_flight) {
    Status r = domain_sync(d);
    if (r.bad()) return r;
  }
  for (int64_t t = 0; t < d.G.ntiles; ++t) {
    if (d.tile_dirty[t]) return make_err(TILE_ESTATE, "dirty tiles; call tile_sync first");
  }
  d.resident_valid = false;
  d.faces_valid = d.xfaces_valid = false;
  if (d.mode == MODE_STREAM) {
    for (int64_t t = 0; t < d.G.ntiles; ++t) d.tile_slot[t] = -1;
    d.free_slots.clear();
    for (int s = 0; s < d.nslots; ++s) {
      d.slot_owner[s] = -1;
      d.free_slots.push_back(s);
    }
  }
  return Status::ok();
}

// GPU-disabled request of one region (§IV.B.4: "If programmer
// requests a region on CPU ... TileAcc performs a check on cache list to see
// if the region is on device", and if so copies it back first; the
// D2H is waited for before the host pointer is returned). READ keeps the
// device copy (now clean); WRITE also drops it, since the caller's CPU code
// will change the host data (stream mode: the tile's slot is freed; resident
// mode: every other device-newer tile is written back too and the next run
// re-uploads the domain).
Status domain_host_region(Domain& d, int64_t t, int mode, double** ptr) {
  Exec& X = *d.exec;
  Status r;
  if (d.tile_dirty[t] && d.tile_slot[t] >= 0) {
    const int sl = d.tile_slot[t];
    int st = 0;
    if (d.mode == MODE_STREAM) {
      const Pipes P(d.last_S, false);
      st = P.out(t);
      r = X.wait(d, ev_slot(d, sl), st);
      if (r.bad()) return r;
    } else {
      // after the kernel of the tile's layer that wrote it last
      int64_t ix, iy, iz;
      d.G.tile_coords(t, &ix, &iy, &iz);
      bool found = false;
      for (auto& b : d.last_batches)
        if (iz >= b.L0 && iz < b.L1 && b.stream >= 0) {
          st = b.out;
          r = X.wait(d, b.ev, st);
          if (r.bad()) return r;
          found = true;
        }
      if (!found) {  // per-tile pipelines (pointwise kernels)
        const Pipes P(d.last_S, d.last_serial);
        st = P.out(t);
        r = X.wait(d, ev_tile(d, t, 0), st);
        if (r.bad()) return r;
      }
    }
    r = X.d2h(d, t, 1, sl, st);
    if (r.bad()) return r;
    if (d.mode == MODE_STREAM) {
      r = X.record(d, ev_slot(d, sl), st);
      if (r.bad()) return r;
      r = X.record(d, ev_host(d, t), st);
      if (r.bad()) return r;
    }
    d.tile_dirty[t] = 0;
    d.stats.writebacks++;
  }
  r = X.sync_all(d);  // the D2H above and any write-back still in flight
  if (r.bad()) return r;
  d.host_pending = false;
  if (mode == TILE_HOST_WRITE) {
    d.host_faces_valid = false;
    if (d.mode == MODE_STREAM) {
      const int sl = d.tile_slot[t];
      if (sl >= 0) {
        d.tile_slot[t] = -1;
        d.slot_owner[sl] = -1;
        d.free_slots.push_back(sl);
      }
      d.faces_valid = d.xfaces_valid = false;  // the tile's exported faces are stale too
    } else if (d.resident_valid) {
      r = domain_sync(d);  // the other device-newer tiles reach the host first
      if (r.bad()) return r;
      d.resident_valid = false;
      d.faces_valid = d.xfaces_valid = false;
      for (int64_t k = 0; k < d.G.ntiles; ++k) d.tile_slot[k] = -1;
    }
  }
  if (d.in_flight) {
    bool any = false;
    for (int64_t k = 0; k < d.G.ntiles; ++k) any |= d.tile_dirty[k] != 0;
    d.in_flight = any;
  }
  *ptr = d.host_tile(t);
  return Status::ok();
}

// Host-side ghost update (§III, §IV.B.6: regions on the host get
// their ghost cells updated on the host): tile t with its g-deep shell,
// gathered from the host store through the ghost map — the periodic wrap, the
// Dirichlet fixed faces (edge and corner cells outside the domain in two or
// three axes are not stored: NaN), or, with z-slab ranks, only shells inside
// the rank's slab (others: EINVAL). Device-newer tiles are written back first.
Status domain_host_ghosts(Domain& d, int64_t t, double* out) {
  const Geometry& G = d.G;
  int64_t c[3];
  G.tile_coords(t, &c[0], &c[1], &c[2]);
  const int64_t g = G.ghost;
  if (G.nranks > 1 && G.bc == TILE_BC_PERIODIC && (c[2] == 0 || c[2] == G.n[2] - 1))
    return make_err(TILE_EINVAL, "ghost cells of this tile live on another rank");
  if (G.nranks > 1 && G.bc == TILE_BC_DIRICHLET && ((c[2] == 0 && G.rank > 0) || (c[2] == G.n[2] - 1 && G.rank < G.nranks - 1)))
    return make_err(TILE_EINVAL, "ghost cells of this tile live on another rank");
  bool dirty = d.host_pending;
  for (int64_t k = 0; k < G.ntiles && !dirty; ++k) dirty = d.tile_dirty[k] && d.tile_slot[k] >= 0;
  if (dirty || d.in_flight) {
    Status r = domain_sync(d);
    if (r.bad()) return r;
  }
  const int64_t ex = G.t[0] + 2 * g, ey = G.t[1] + 2 * g, ez = G.t[2] + 2 * g;
  std::vector<int64_t> map((size_t)(ex * ey * ez));
  ghost_map(G, t, map.data());
  const int64_t tx = G.t[0], ty = G.t[1], tz = G.t[2], nx = G.g[0], ny = G.g[1];
  const int64_t D = G.depth;
  for (int64_t k = 0; k < ez; ++k)
    for (int64_t j = 0; j < ey; ++j)
      for (int64_t i = 0; i < ex; ++i) {
        const int64_t m = map[(size_t)((k * ey + j) * ex + i)];
        double v;
        if (m >= 0) {
          const int64_t x = m % nx, y = (m / nx) % ny, z = m / (nx * ny) - G.zoff;  // local z
          const int64_t k2 = ((z / tz) * G.n[1] + y / ty) * G.n[0] + x / tx;
          v = d.host_tile(k2)[((z % tz) * ty + y % ty) * tx + x % tx];
        } else {  // Dirichlet: the fixed face of the domain boundary (nearest layer)
          int64_t p[3] = {c[0] * tx + i - g, c[1] * ty + j - g, c[2] * tz + k - g};  // local coords
          const int64_t lim[3] = {G.l[0], G.l[1], G.l[2]};
          int axis = -1, nout = 0;
          for (int a = 0; a < 3; ++a)
            if (p[a] < 0 || p[a] >= lim[a]) ++nout, axis = a;
          v = std::nan("");  // outside in two or three axes: not stored
          if (nout == 1) {
            const int f = 2 * axis + (p[axis] < 0 ? 0 : 1);
            p[axis] = p[axis] < 0 ? 0 : lim[axis] - 1;  // the adjacent interior cell
            const int64_t k2 = ((p[2] / tz) * G.n[1] + p[1] / ty) * G.n[0] + p[0] / tx;
            const int64_t lx = p[0] % tx, ly = p[1] % ty, lz = p[2] % tz;
            const double* fc = d.host_dir[f] + k2 * G.face_elems[f];
            const int64_t l = (f & 1) ? 0 : D - 1;  // the layer nearest the tile
            if (f <= XP) v = fc[(lz * ty + ly) * D + l];
            else if (f <= YP) v = fc[(lz * D + l) * tx + lx];
            else v = fc[(l * ty + ly) * tx + lx];
          }
        }
        out[(k * ey + j) * ex + i] = v;
      }
  return Status::ok();
}

// GPU-disabled iteration (§IV.B.5: compute(tile, lambda) with the
// iterator's GPU flag off; the regions' newest data is brought to the
// host first; their ghost cells are updated on the host). The
// library only moves data and calls the caller's function: no cell update of
// its own runs on the CPU. With `ghosted`, every listed tile's shell is
// gathered before the first call, so an update that writes its tile in
// place still reads only old values through the shells (Jacobi order, as
// the paper's separate old/new tile arrays give). WRITE hands the host store
// the newest data: device copies are dropped (as tile_mark_host_dirty).
Status domain_host_compute(Domain& d, const int64_t* ids, int64_t n, int mode, int ghosted, tile_host_fn fn,
                           void* ctx) {
  const Geometry& G = d.G;
  std::vector<int64_t> list;
  if (ids) list.assign(ids, ids + n);
  else for (int64_t k = 0; k < G.ntiles; ++k) list.push_back(k);
  bool dirty = d.host_pending || d.in_flight;
  for (int64_t k = 0; k < G.ntiles && !dirty; ++k) dirty = d.tile_dirty[k] && d.tile_slot[k] >= 0;
  if (dirty) {
    Status r = domain_sync(d);
    if (r.bad()) return r;
  }
  const int64_t g = G.ghost;
  const int64_t box = (G.t[0] + 2 * g) * (G.t[1] + 2 * g) * (G.t[2] + 2 * g);
  // WRITE: every shell before the first call (Jacobi order); READ: one at a
  // time (nothing changes between the calls)
  const bool all_first = ghosted && mode == TILE_HOST_WRITE;
  std::vector<double> shells;
  if (ghosted) {
    try {
      shells.resize((size_t)(box * (all_first ? (int64_t)list.size() : 1)));
    } catch (const std::bad_alloc&) {
      return make_err(TILE_ENOMEM_HOST, "host ghost shells for the listed tiles");
    }
    for (size_t i = 0; all_first && i < list.size(); ++i) {
      Status r = domain_host_ghosts(d, list[i], shells.data() + i * (size_t)box);
      if (r.bad()) return r;
    }
  }
  for (size_t i = 0; i < list.size(); ++i) {
    int64_t c[3];
    G.tile_coords(list[i], &c[0], &c[1], &c[2]);
    const int64_t origin[3] = {c[0] * G.t[0], c[1] * G.t[1], c[2] * G.t[2] + G.zoff};
    const double* sh = nullptr;
    if (ghosted && all_first) sh = shells.data() + i * (size_t)box;
    if (ghosted && !all_first) {
      Status r = domain_host_ghosts(d, list[i], shells.data());
      if (r.bad()) return r;
      sh = shells.data();
    }
    fn(ctx, list[i], d.host_tile(list[i]), sh, G.t, origin, (int32_t)g);
  }
  if (mode == TILE_HOST_WRITE) {
    d.host_faces_valid = false;
    for (auto& x : d.tile_dirty) x = 0;
    return domain_invalidate(d);
  }
  return Status::ok();
}

Status domain_load(Domain& d, const double* src) {
  if (d.in_flight) {
    Status r = domain_sync(d);
    if (r.bad()) return r;
  }
  const Geometry& G = d.G;
  const bool dir = G.bc == TILE_BC_DIRICHLET;
  const int64_t h = dir ? 1 : 0;
  const int64_t ex = G.l[0] + 2 * h, ey = G.l[1] + 2 * h;
  const int64_t tx = G.t[0], ty = G.t[1], tz = G.t[2];
  host_parallel_for(G.ntiles, [&](int64_t b, int64_t e) {
    for (int64_t k = b; k < e; ++k) {
      int64_t ix, iy, iz;
      G.tile_coords(k, &ix, &iy, &iz);
      double* dst = d.host_tile(k);
      for (int64_t z = 0; z < tz; ++z)
        for (int64_t y = 0; y < ty; ++y) {
          const double* s =
              src + ((iz * tz + z + h) * ey + (iy * ty + y + h)) * ex + ix * tx + h;
          std::memcpy(dst + (z * ty + y) * tx, s, (size_t)tx * 8);
        }
    }
  });
  if (dir) {  // fixed Dirichlet faces from the halo (only boundary faces used)
    host_parallel_for(G.ntiles, [&](int64_t b, int64_t e) {
      for (int64_t k = b; k < e; ++k) {
        int64_t ix, iy, iz;
        G.tile_coords(k, &ix, &iy, &iz);
        const int64_t ox = ix * tx + h, oy = iy * ty + h, oz = iz * tz + h;
        auto at = [&](int64_t z, int64_t y, int64_t x) { return src[(z * ey + y) * ex + x]; };
        const int64_t D = G.depth;
        for (int f = 0; f < 6; ++f) {
          if (face_source(G, k, f).kind != 1) continue;
          // the fixed halo value goes to the layer nearest the tile (the
          // minus faces' last layer, the plus faces' first); others unused
          double* o = d.host_dir[f] + k * G.face_elems[f];
          const int64_t l = (f & 1) ? 0 : D - 1;
          if (f <= XP) {
            const int64_t x = f == XM ? ox - 1 : ox + tx;
            for (int64_t z = 0; z < tz; ++z)
              for (int64_t y = 0; y < ty; ++y) o[(z * ty + y) * D + l] = at(oz + z, oy + y, x);
          } else if (f <= YP) {
            const int64_t y = f == YM ? oy - 1 : oy + ty;
            for (int64_t z = 0; z < tz; ++z)
              for (int64_t x = 0; x < tx; ++x) o[(z * D + l) * tx + x] = at(oz + z, y, ox + x);
          } else {
            const int64_t z = f == ZM ? oz - 1 : oz + tz;
            for (int64_t y = 0; y < ty; ++y)
              for (int64_t x = 0; x < tx; ++x) o[(l * ty + y) * tx + x] = at(z, oy + y, ox + x);
          }
        }
      }
    });
    d.dir_uploaded = false;
  }
  d.host_faces_valid = false;
  for (int64_t t = 0; t < G.ntiles; ++t) d.tile_dirty[t] = 0;
  return domain_invalidate(d);
}

Status domain_store(Domain& d, double* dst) {
  Status r = domain_sync(d);
  if (r.bad()) return r;
  const Geometry& G = d.G;
  const int64_t h = G.bc == TILE_BC_DIRICHLET ? 1 : 0;
  const int64_t ex = G.l[0] + 2 * h, ey = G.l[1] + 2 * h;
  const int64_t tx = G.t[0], ty = G.t[1], tz = G.t[2];
  host_parallel_for(G.ntiles, [&](int64_t b, int64_t e) {
    for (int64_t k = b; k < e; ++k) {
      int64_t ix, iy, iz;
      G.tile_coords(k, &ix, &iy, &iz);
      const double* s = d.host_tile(k);
      for (int64_t z = 0; z < tz; ++z)
        for (int64_t y = 0; y < ty; ++y) {
          double* o = dst + ((iz * tz + z + h) * ey + (iy * ty + y + h)) * ex + ix * tx + h;
          std::memcpy(o, s + (z * ty + y) * tx, (size_t)tx * 8);
        }
    }
  });
  return Status::ok();
}

}  // namespace tiles
