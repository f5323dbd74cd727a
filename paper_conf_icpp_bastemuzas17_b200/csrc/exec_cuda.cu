// exec_cuda.cu — the CUDA executor: maps the scheduler's operations onto
// CUDA streams, events, cudaMemcpyAsync from pinned memory
// and the sm_100a kernels of kernels.cu. No CPU fallback exists: every
// compute operation is a kernel launch.
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "runtime.hpp"

namespace tiles {
namespace {

Status cuda_err(cudaError_t e, const char* what) {
  char buf[256];
  std::snprintf(buf, sizeof buf, "%s: %s", what, cudaGetErrorString(e));
  return make_err(TILE_ECUDA, buf);
}
#define CK(call)                                  \
  do {                                            \
    cudaError_t e_ = (call);                      \
    if (e_ != cudaSuccess) return cuda_err(e_, #call); \
  } while (0)

struct CudaExec final : Exec {
  int dev = 0;
  int sms = 148;
  int heat_occ = 1;
  std::vector<cudaStream_t> streams;
  std::vector<char> own_stream;
  std::vector<cudaEvent_t> events;
  std::vector<cudaEvent_t> tpool;                 // timing events (free list)
  struct Timed {
    cudaEvent_t a, b;
    uint64_t cells;  // cells read + written once by the launches (stencil sweeps), else 0
    uint32_t n;      // launches inside [a, b]
  };
  std::vector<Timed> tpending;
  // a run of consecutive sweep launches on one stream shares one event pair:
  // an event between two launches would end programmatic dependent launch
  // (the next sweep's ramp overlapping the previous one's drain), so a
  // per-launch pair times each sweep alone. The interval is closed (its end
  // event recorded) by the next other operation on that stream (S() below),
  // a join or a synchronize.
  std::vector<int> open_iv;  // per stream: index into tpending, or -1
  bool in_launch = false;    // S() inside a timed launch does not close
  uint64_t next_cells = 0;   // cells of the next timed launch (set just before it)
  cudaEvent_t t_begin = nullptr, t_end = nullptr;
  cudaEvent_t local_ready = nullptr;  // in-process transport

  Status timing_event(cudaEvent_t* e) {
    if (!tpool.empty()) {
      *e = tpool.back();
      tpool.pop_back();
      return Status::ok();
    }
    CK(cudaEventCreate(e));
    return Status::ok();
  }
  Status close_iv(int st) {
    if (open_iv.size() <= (size_t)st || open_iv[(size_t)st] < 0) return Status::ok();
    Timed& t = tpending[(size_t)open_iv[(size_t)st]];
    open_iv[(size_t)st] = -1;
    Status r = timing_event(&t.b);
    if (r.bad()) return r;
    CK(cudaEventRecord(t.b, streams[(size_t)st]));
    return Status::ok();
  }
  Status close_all() {
    for (size_t i = 0; i < open_iv.size(); ++i) {
      Status r = close_iv((int)i);
      if (r.bad()) return r;
    }
    return Status::ok();
  }
  // bracket a kernel launch with timing events on its stream (a sweep joins
  // the stream's open interval)
  template <class F>
  Status timed(Domain& d, int st, F&& launch) {
    return timed_status(d, st, [&]() -> Status {
      CK(launch());
      return Status::ok();
    });
  }
  // the same for a launch that reports a library Status (user kernels: the
  // real cause — ENOSYS, module load, launch — reaches the caller unchanged)
  template <class F>
  Status timed_status(Domain& d, int st, F&& launch) {
    const uint64_t cells = next_cells;
    next_cells = 0;
    if (!d.kernel_timing) {
      Status r = close_iv(st);
      if (r.bad()) return r;
      in_launch = true;
      r = launch();
      in_launch = false;
      return r;
    }
    if (open_iv.size() < streams.size()) open_iv.resize(streams.size(), -1);
    if (!cells || open_iv[(size_t)st] < 0) {
      Status r = close_iv(st);
      if (r.bad()) return r;
      cudaEvent_t a;
      r = timing_event(&a);
      if (r.bad()) return r;
      CK(cudaEventRecord(a, streams[(size_t)st]));
      tpending.push_back({a, nullptr, 0, 0});
      open_iv[(size_t)st] = (int)tpending.size() - 1;
    }
    in_launch = true;
    Status r = launch();
    in_launch = false;
    if (r.bad()) return r;  // the open interval is closed by the sync that reports it
    Timed& t = tpending[(size_t)open_iv[(size_t)st]];
    t.cells += cells;
    t.n++;
    if (!cells) return close_iv(st);
    return Status::ok();
  }
  Status collect(Domain& d) {  // after a synchronize
    for (auto& pr : tpending) {
      float ms = 0;
      if (pr.b) CK(cudaEventElapsedTime(&ms, pr.a, pr.b));
      d.stats.kernel_ms += ms;
      d.stats.kernel_timed += pr.n;
      if (pr.cells) {
        d.stats.sweep_ms += ms;
        d.stats.sweep_cells += pr.cells;
        d.stats.sweep_timed += pr.n;
      }
      tpool.push_back(pr.a);
      if (pr.b) tpool.push_back(pr.b);
    }
    tpending.clear();
    return Status::ok();
  }
  Status join_into0(Domain& d) {
    Status r0 = close_all();
    if (r0.bad()) return r0;
    for (size_t i = 1; i < streams.size(); ++i) {
      CK(cudaEventRecord(events[(size_t)(d.ev_misc_base + 4 + i)], streams[i]));
      CK(cudaStreamWaitEvent(streams[0], events[(size_t)(d.ev_misc_base + 4 + i)], 0));
    }
    return Status::ok();
  }
  Status timer_start(Domain& d) override {
    if (!t_begin) CK(cudaEventCreate(&t_begin));
    if (!t_end) CK(cudaEventCreate(&t_end));
    Status r = join_into0(d);
    if (r.bad()) return r;
    CK(cudaEventRecord(t_begin, streams[0]));
    // later work on any stream starts after t_begin
    for (size_t i = 1; i < streams.size(); ++i) CK(cudaStreamWaitEvent(streams[i], t_begin, 0));
    return Status::ok();
  }
  Status timer_stop(Domain& d, double* ms) override {
    Status r = join_into0(d);
    if (r.bad()) return r;
    CK(cudaEventRecord(t_end, streams[0]));
    CK(cudaEventSynchronize(t_end));
    float f = 0;
    CK(cudaEventElapsedTime(&f, t_begin, t_end));
    *ms = f;
    r = sync_all(d);
    if (r.bad()) return r;
    return Status::ok();
  }

  // the stream of an operation; any operation but a timed sweep ends the
  // stream's open timing interval first
  cudaStream_t S(int i) {
    if (!in_launch && (size_t)i < open_iv.size() && open_iv[(size_t)i] >= 0) (void)close_iv(i);
    return streams[(size_t)i];
  }

  // TILES_FAULT: the n-th operation of a kind fails with a real CUDA error
  // (an invalid copy queued on the same stream), reported through CK.
  Status inject(Domain& d, int kind, int st) {
    if (!fault_fires(d, kind)) return Status::ok();
    CK(cudaMemcpyAsync(nullptr, nullptr, 8, cudaMemcpyDeviceToDevice, S(st < 0 ? 0 : st)));
    return make_err(TILE_ECUDA, "injected fault did not fail");
  }
#define INJECT(kind, st)                 \
  do {                                   \
    Status f_ = inject(d, kind, st);     \
    if (f_.bad()) return f_;             \
  } while (0)

  Status h2d(Domain& d, int64_t t0, int64_t n, int s0, int st) override {
    INJECT(FAULT_H2D, st);
    if (d.measure == TILE_MEASURE_COMP_ONLY) return Status::ok();
    const size_t bytes = (size_t)n * d.G.tile_elems * 8;
    CK(cudaMemcpyAsync(d.slot_ptr(s0), d.host_tile(t0), bytes, cudaMemcpyHostToDevice, S(st)));
    d.stats.bytes_h2d += bytes;
    d.stats.n_h2d++;
    return Status::ok();
  }
  Status d2h(Domain& d, int64_t t0, int64_t n, int s0, int st) override {
    INJECT(FAULT_D2H, st);
    if (d.measure == TILE_MEASURE_COMP_ONLY) return Status::ok();
    const size_t bytes = (size_t)n * d.G.tile_elems * 8;
    CK(cudaMemcpyAsync(d.host_tile(t0), d.slot_ptr(s0), bytes, cudaMemcpyDeviceToHost, S(st)));
    d.stats.bytes_d2h += bytes;
    d.stats.n_d2h++;
    return Status::ok();
  }
  Status record(Domain&, int ev, int st) override {
    CK(cudaEventRecord(events[(size_t)ev], S(st)));
    return Status::ok();
  }
  Status wait(Domain&, int ev, int st) override {
    CK(cudaStreamWaitEvent(S(st), events[(size_t)ev], 0));
    return Status::ok();
  }
  Status heat(Domain& d, const int64_t* tiles, const int* in, const int* out, int n, int rp,
              const TileItem* dev_items, int st, int direct_bit, int nstack, int nsteps) override {
    INJECT(FAULT_KERNEL, st);
    if (d.measure == TILE_MEASURE_XFER_ONLY || n == 0) return Status::ok();
    if (d.user_fn && userfn_is_stencil(d.user_fn)) {  // TILE_KERNEL_USER_STENCIL (face ghosts)
      double* fx[6];
      for (int f = 0; f < 6; ++f) fx[f] = d.faces[f][rp ^ 1];
      const double* const* gs = d.gsrc_dev[rp];
      Status r;
      if (dev_items) {
        r = timed_status(d, st, [&] {
          return userfn_launch_stencil(d.user_fn, dev_items, n, nullptr, nullptr, 0, gs, fx, d.G.face_elems,
                                       d.G.t, d.G.depth, S(st));
        });
        if (r.bad()) return r;
        d.stats.n_kernels++;
      } else {
        for (int i = 0; i < n; ++i) {
          r = timed_status(d, st, [&] {
            return userfn_launch_stencil(d.user_fn, nullptr, 1, d.slot_ptr(in[i]), d.slot_ptr(out[i]),
                                         (int)tiles[i], gs, fx, d.G.face_elems, d.G.t, d.G.depth, S(st));
          });
          if (r.bad()) return r;
          d.stats.n_kernels++;
        }
      }
      return Status::ok();
    }
    if (nsteps > 1 && (!coop || direct_bit < 0 || !dev_items || (int64_t)sms * heat_occ > kMaxProgCtas)) {
      // no persistent launch possible: one launch per step (buffers and face
      // parities alternate)
      const int64_t off = dev_items - d.items_dev[direct_bit];
      for (int s = 0; s < nsteps; ++s) {
        const int b = direct_bit ^ (s & 1);
        Status r = heat(d, tiles, in, out, n, rp ^ (s & 1), d.items_dev[b] + off, st, b, nstack, 1);
        if (r.bad()) return r;
      }
      return Status::ok();
    }
    HeatParams p{};
    p.tx = (int)d.G.t[0];
    p.ty = (int)d.G.t[1];
    p.tz = (int)d.G.t[2];
    p.band = d.band;
    p.nbands = p.ty / d.band;
    p.nitems = n;
    p.alpha = d.kernel_alpha;
    p.cache_flags = d.heat_cache_flags;
    p.depth = d.G.depth;
    if (dev_items) {
      p.items = dev_items;
    } else {
      if (n > kMaxInlineItems) return make_err(TILE_ESTATE, "internal: too many inline items");
      p.items = nullptr;
      for (int i = 0; i < n; ++i)
        p.inline_items[i] = {d.slot_ptr(in[i]), d.slot_ptr(out[i]), (int32_t)tiles[i], 0};
    }
    p.gsrc = d.gsrc_dev[rp];
    for (int f = 0; f < 6; ++f) {
      p.fexp[f] = d.faces[f][rp ^ 1];
      p.face_elems[f] = d.G.face_elems[f];
    }
    if (nstack < 1 || n % nstack) return make_err(TILE_ESTATE, "internal: bad tile stack");
    p.nstack = nstack;
    p.lt = n / nstack;
    if (direct_bit >= 0) {  // y/z ghosts from the neighbours' interiors; export x (+ slab-end z)
      p.gdir = d.gdir_dev[direct_bit][rp];
      p.ystr = d.ystr_dev;
      p.exp_y = 0;
      const bool multi = d.G.nranks > 1;
      p.exp_zlo_below = multi ? (int32_t)d.G.layer_tiles : 0;
      p.exp_zhi_from = multi ? (int32_t)(d.G.ntiles - d.G.layer_tiles) : INT32_MAX;
      if (multi && d.peer_fused && d.peer_connected && d.measure != TILE_MEASURE_COMP_ONLY) {
        // write parity rp^1 of the neighbours' receive buffers: the lower
        // rank's halo[1] (from above) and the upper rank's halo[0]
        const int wp = rp ^ 1;
        const uint64_t hb = d.peer_halo_bytes;
        char* lo = static_cast<char*>(d.peer_base[0]);
        char* up = static_cast<char*>(d.peer_base[1]);
        p.zpush_lo = lo ? reinterpret_cast<double*>(lo + (2 + wp) * hb) : nullptr;
        p.zpush_hi = up ? reinterpret_cast<double*>(up + (0 + wp) * hb) : nullptr;
      }
    } else {
      p.gdir = nullptr;
      p.ystr = nullptr;
      p.exp_y = 1;
      p.exp_zlo_below = INT32_MAX;
      p.exp_zhi_from = 0;
    }
    // persistent grid: one wave of CTAs, >= 4 planes each
    const int64_t planes = (int64_t)n * p.nbands * p.tz;
    int64_t grid = (int64_t)sms * heat_occ;
    static const int64_t grid_cap = [] {  // experiment knob: cap the persistent grid
      const char* e = std::getenv("TILES_HEAT_GRID");
      return e ? (int64_t)std::atoll(e) : (int64_t)0;
    }();
    if (grid_cap > 0) grid = std::min(grid, grid_cap);
    grid = std::max<int64_t>(1, std::min<int64_t>(grid, (planes + 3) / 4));
    // banded tiles: adjacent bands side by side in time (their shared halo
    // rows from L2); TILES_HEAT_RR=0 keeps contiguous plane ranges
    static const int rr_on = [] {
      const char* e = std::getenv("TILES_HEAT_RR");
      return e ? std::atoi(e) : 1;
    }();
    p.rr_rounds = rr_on && p.nbands > 1 ? (int32_t)((int64_t)p.lt * p.nbands / grid) : 0;
    {  // z-chunked round-robin items (TILES_HEAT_ZCHUNK planes; experiment)
      static const int zc = [] {
        const char* e = std::getenv("TILES_HEAT_ZCHUNK");
        return e ? std::atoi(e) : 0;
      }();
      const int64_t NZ = (int64_t)nstack * p.tz;
      if (zc > 0 && NZ % zc == 0) {
        p.zchunk = zc;
        p.rr_rounds = (int32_t)((int64_t)p.lt * p.nbands * (NZ / zc) / grid);
      }
    }
    p.nsteps = 1;
    if (nsteps > 1) {  // one persistent launch for all steps (CTA progress counters)
      const int b1 = direct_bit ^ 1;
      p.nsteps = nsteps;
      // snake order across steps (TILES_SNAKE=0: off; TILES_SNAKE_KEEP: planes
      // per CTA stored evict_last at the end of a step, default 16)
      static const int snake = [] {
        const char* e = std::getenv("TILES_SNAKE");
        return e ? std::atoi(e) : 1;
      }();
      static const int keep_tail = [] {
        const char* e = std::getenv("TILES_SNAKE_KEEP");
        return e ? std::atoi(e) : 16;
      }();
      p.snake = snake;
      p.keep_tail = snake ? keep_tail : 0;
      p.ntx = (int32_t)d.G.n[0];
      p.nty = (int32_t)d.G.n[1];
      p.epoch = d.prog_epoch;
      p.prog = d.prog_dev;
      p.items_odd = d.items_dev[b1] + (dev_items - d.items_dev[direct_bit]);
      p.gdir_odd = d.gdir_dev[b1][rp ^ 1];
      for (int f = 0; f < 6; ++f) p.fexp_odd[f] = d.faces[f][rp];
      d.prog_epoch += (uint32_t)(nsteps - 1);  // barrier rounds of this launch
      if (d.prog_grid && d.prog_grid != grid) return make_err(TILE_ESTATE, "internal: persistent grid changed");
      d.prog_grid = grid;
    }
    cudaError_t le = cudaSuccess;
    next_cells = d.kernel_timing ? (uint64_t)n * d.G.tile_elems * (uint64_t)p.nsteps : 0;
    Status r = timed(d, st, [&] {
      le = launch_heat7(p, d.stages, d.heat_smem, (int)grid, S(st));
      return le == cudaErrorCooperativeLaunchTooLarge ? cudaSuccess : le;
    });
    if (r.bad()) return r;
    if (le == cudaErrorCooperativeLaunchTooLarge) {
      // SMs held by another context: no co-residency guarantee, so no
      // persistent launches on this domain; run the steps one launch each
      (void)cudaGetLastError();
      coop = 0;
      d.prog_epoch -= (uint32_t)(nsteps - 1);
      return heat(d, tiles, in, out, n, rp, dev_items, st, direct_bit, nstack, nsteps);
    }
    d.stats.n_kernels++;
    return Status::ok();
  }
  int coop = 0;  // cudaDevAttrCooperativeLaunch
  SweepMaps maps{};
  bool maps_tried = false;
  const double* maps_wave = nullptr;
  int64_t maps_wave_slots = 0;
  // tensor maps of the slot pool and the wavefront scratch (x halos of the
  // tile-column sweep), encoded once per allocation
  void ensure_maps(Domain& d) {
    if (!maps_tried) {
      maps_tried = true;
      sweep_map_encode(&maps, 0, d.slot_base, (uint64_t)d.nslots * d.G.tile_elems * 8, (int)d.G.t[0],
                       sweep_tile_band());
    }
    // (re-encoded when the scratch moves or grows: a reallocation may return
    // the same address with more slots, which a stale map would read as
    // out-of-bounds zeros)
    if (d.wave_base && (maps_wave != d.wave_base || maps_wave_slots != d.wave_slots)) {
      maps_wave = d.wave_base;
      maps_wave_slots = d.wave_slots;
      sweep_map_encode(&maps, 1, d.wave_base, (uint64_t)d.wave_slots * d.G.tile_elems * 8, (int)d.G.t[0],
                       sweep_tile_band());
    }
  }
  SlabView slab_view(Domain& d, const SlabRef& r, int lo) {
    const Geometry& G = d.G;
    SlabView v{};
    v.ntx = (int)G.n[0];
    v.nty = (int)G.n[1];
    v.tx = (int)G.t[0];
    v.ty = (int)G.t[1];
    v.tz = 1 << 30;
    if (r.kind == SlabRef::DENSE) {
      // scratch slab, tile-blocked like the packed sub-tiles: [tile (x, y)]
      // [plane < slab_depth][ty][tx], so the sweep kernels stage bands of
      // rows as single contiguous ranges
      v.base = d.slot_ptr(r.slot);
      v.te = d.slab_depth * G.t[0] * G.t[1];
    } else if (r.kind == SlabRef::RESIDENT) {
      v.base = d.slot_ptr(r.slot ? (int)G.ntiles : 0);
      v.te = G.tile_elems;
      v.tz = (int)G.t[2];
      v.zbase = (int)r.zbase;
      v.nz = (int)G.l[2];
      if (G.nranks > 1) {  // multi-rank stream-through: no wrap inside the slab
        v.hlo = d.st_halo[0];
        v.hhi = d.st_halo[1];
      }
    } else if (r.kind == SlabRef::WAVE) {
      v.base = d.slot_ptr(r.slot);  // the level's tile-blocked array (its first slot)
      v.te = G.tile_elems;
      v.tz = (int)G.t[2];
      v.zbase = 0;
      v.nz = (int)G.l[2];
      v.hlo = d.slot_ptr(r.ring[0]);
      v.nlo = (int)r.un;
    } else if (r.kind == SlabRef::UNITS) {
      v.ring = 1;
      v.te = r.un * G.t[0] * G.t[1];
      v.zbase = (int)r.zbase;
      v.nz = (int)G.l[2];
      v.u = (int)r.u;
      v.un = (int)r.un;
      v.U = (int)(G.l[2] / r.un);
      for (int k = 0; k < 3; ++k) v.ubase[k] = d.slot_ptr(r.ring[k]);
    } else {  // SUB: packed sub-tiles of st_unit planes; sweep plane lo -> 0
      v.base = d.slot_ptr(r.slot);
      v.te = d.st_unit * G.t[0] * G.t[1];
      v.zbase = -lo;
    }
    return v;
  }
  Status slab_sweep(Domain& d, const SlabRef& src, const SlabRef& dst, int lo, int hi, int st) override {
    INJECT(FAULT_KERNEL, st);
    if (d.measure == TILE_MEASURE_XFER_ONLY) return Status::ok();
    const SlabView s = slab_view(d, src, lo), t = slab_view(d, dst, lo);
    next_cells = d.kernel_timing ? (uint64_t)(hi - lo) * d.G.l[0] * d.G.l[1] : 0;
    ensure_maps(d);
    Status r = timed(d, st, [&] {
      return launch_slab_sweep(s, t, (int)d.G.l[0], (int)d.G.l[1], lo, hi, d.kernel_alpha, sms, S(st), &maps);
    });
    if (r.bad()) return r;
    d.stats.n_kernels++;
    return Status::ok();
  }
  Band2Maps bmaps[2];
  int bmaps_state = 0;  // 0 not tried, 1 encoded, -1 not available
  // tensor maps of other tile-blocked regions (wavefront level arrays and
  // scratch layers, stream-through slabs), by base pointer, tile depth and
  // tile layers
  struct MapEntry {
    const double* base;
    int tz, layers;
    bool ok;
    Band2Maps m;
  };
  std::vector<MapEntry> band_maps;
  bool band_maps_for(Domain& d, const double* base, int tz, int layers, Band2Maps* out) {
    for (auto& e : band_maps)
      if (e.base == base && e.tz == tz && e.layers == layers) {
        if (e.ok) *out = e.m;
        return e.ok;
      }
    const Geometry& G = d.G;
    MapEntry e{base, tz, layers, false, {}};
    e.ok = band2_maps_encode(&e.m, base, (int)G.t[0], (int)G.t[1], tz, (int)G.n[0], (int)G.n[1], layers);
    band_maps.push_back(e);
    if (e.ok) *out = e.m;
    return e.ok;
  }
  bool band2_slab_on(Domain& d) {
    static const int on = [] {
      const char* e = getenv("TILES_BAND2_SLAB");
      return e ? atoi(e) : 1;
    }();
    const Geometry& G = d.G;
    return on && G.nranks == 1 && band2_shape_ok(G.l[0], G.l[1], (int)G.t[0], (int)G.t[1]);
  }
  // a view read by heat2_band_slab: RESIDENT (wrapped, plane offset zbase),
  // WAVE (level array + scratch layers), DENSE (one layer of slab_depth)
  bool band2_in(Domain& d, const SlabRef& r, Band2View* v) {
    const Geometry& G = d.G;
    v->nlo = 0;
    v->wrap = r.kind == SlabRef::RESIDENT;
    v->zbase = 0;
    v->nz = (int)G.l[2];
    v->tz = (int)G.t[2];
    if (r.kind == SlabRef::RESIDENT) {
      v->zbase = (int)r.zbase;
      return band_maps_for(d, d.slot_ptr(r.slot ? (int)G.ntiles : 0), v->tz, (int)G.n[2], &v->main);
    }
    if (r.kind == SlabRef::WAVE) {
      v->nlo = (int)r.un;
      return band_maps_for(d, d.slot_ptr(r.slot), v->tz, (int)G.n[2], &v->main) &&
             band_maps_for(d, d.slot_ptr(r.ring[0]), v->tz, (int)r.un, &v->scr);
    }
    if (r.kind == SlabRef::DENSE) {
      v->tz = (int)d.slab_depth;
      return band_maps_for(d, d.slot_ptr(r.slot), v->tz, 1, &v->main);
    }
    return false;
  }
  // a view written by heat2_band_slab; SUB: plane `first` -> sub-tile plane 0
  bool band2_out(Domain& d, const SlabRef& r, int first, Band2Out* o) {
    const Geometry& G = d.G;
    o->base = d.slot_ptr(r.slot);
    o->hlo = nullptr;
    o->nlo = 0;
    o->zbase = 0;
    if (r.kind == SlabRef::WAVE) {
      o->hlo = d.slot_ptr(r.ring[0]);
      o->nlo = (int)r.un;
      o->tz = (int)G.t[2];
    } else if (r.kind == SlabRef::DENSE) {
      o->tz = (int)d.slab_depth;
    } else if (r.kind == SlabRef::SUB) {
      o->tz = (int)d.st_unit;
      o->zbase = -first;
    } else {
      return false;
    }
    o->te = (int64_t)o->tz * G.t[0] * G.t[1];
    return true;
  }
  bool sweep2s_ok(Domain& d) override { return band2_slab_on(d); }
  unsigned long long* iter_flags = nullptr;
  unsigned long long iter_epoch = 0;
  bool wave_iter_ok(Domain& d) override {
    // one launch per wavefront iteration (TILES_WAVE_ITER=1): correct, but
    // slower than a launch per pass with programmatic dependent launch
    // (Fig. 5 T = 100: 48.2 vs 42.3 ms) — off by default
    static const int on = [] {
      const char* e = getenv("TILES_WAVE_ITER");
      return e ? atoi(e) : 0;
    }();
    return on && band2_slab_on(d) && d.G.l[1] / 4 <= sms;
  }
  Status wave_iteration(Domain& d, const SlabRef* lv, int64_t ci, int c, int s0, int P, int st) override {
    INJECT(FAULT_KERNEL, st);
    if (d.measure == TILE_MEASURE_XFER_ONLY) return Status::ok();
    const Geometry& G = d.G;
    Band2Iter p{};
    for (int k = 0; k < 4; ++k)
      if (!band2_in(d, lv[k], &p.v[k])) return make_err(TILE_ESTATE, "internal: wavefront views without band maps");
    for (int k = 0; k < 3; ++k)
      if (!band2_out(d, lv[k], 0, &p.o[k])) return make_err(TILE_ESTATE, "internal: wavefront views without band maps");
    if (!iter_flags) {
      const size_t nb = (size_t)(G.l[1] / 4);
      CK(cudaMalloc(reinterpret_cast<void**>(&iter_flags), nb * sizeof(unsigned long long)));
      CK(cudaMemset(iter_flags, 0, nb * sizeof(unsigned long long)));
    }
    p.flags = iter_flags;
    p.epoch = ++iter_epoch;
    p.ty = (int)G.t[1];
    p.nty = (int)G.n[1];
    p.ci = (int)ci;
    p.c = c;
    p.s0 = s0;
    p.P = P;
    p.alpha = d.kernel_alpha;
    next_cells = d.kernel_timing ? (uint64_t)P * c * G.l[0] * G.l[1] : 0;  // one pass over each level pair's cells
    Status r = timed(d, st, [&] { return launch_heat2_band_iter(p, S(st)); });
    if (r.bad()) return r;
    d.stats.n_kernels++;
    return Status::ok();
  }
  Status slab_sweep2s(Domain& d, const SlabRef& src, const SlabRef& dst, int lo, int hi, int st) override {
    INJECT(FAULT_KERNEL, st);
    if (d.measure == TILE_MEASURE_XFER_ONLY) return Status::ok();
    Band2View bv;
    Band2Out bo;
    if (!band2_in(d, src, &bv) || !band2_out(d, dst, lo + 1, &bo))
      return make_err(TILE_ESTATE, "internal: two-sweep pass on views without band maps");
    next_cells = d.kernel_timing ? (uint64_t)(hi - lo) * d.G.l[0] * d.G.l[1] : 0;  // one pass over the cells
    Status r = timed(d, st, [&] {
      return launch_heat2_band_slab(0, bv, bv, bo, bo, (int)d.G.t[1], (int)d.G.n[1], lo, hi, d.kernel_alpha, S(st));
    });
    if (r.bad()) return r;
    d.stats.n_kernels++;
    return Status::ok();
  }
  bool band2_ok(Domain& d) override {
    if (bmaps_state == 0) {
      const Geometry& G = d.G;
      bmaps_state = -1;
      if (d.nslots >= 2 * G.ntiles &&
          band2_maps_encode(&bmaps[0], d.slot_ptr(0), (int)G.t[0], (int)G.t[1], (int)G.t[2], (int)G.n[0],
                            (int)G.n[1], (int)G.n[2]) &&
          band2_maps_encode(&bmaps[1], d.slot_ptr((int)G.ntiles), (int)G.t[0], (int)G.t[1], (int)G.t[2],
                            (int)G.n[0], (int)G.n[1], (int)G.n[2]))
        bmaps_state = 1;
    }
    return bmaps_state == 1;
  }
  Status band2(Domain& d, int sbit, int dbit, int st) override {
    INJECT(FAULT_KERNEL, st);
    if (d.measure == TILE_MEASURE_XFER_ONLY) return Status::ok();
    if (!band2_ok(d)) return make_err(TILE_ESTATE, "internal: heat2_band without its tensor maps");
    const Geometry& G = d.G;
    next_cells = d.kernel_timing ? (uint64_t)(G.l[0] * G.l[1] * G.l[2]) : 0;  // one pass over the cells
    Status r = timed(d, st, [&] {
      return launch_heat2_band(bmaps[sbit], d.slot_ptr(dbit ? (int)G.ntiles : 0), (int)G.t[1], (int)G.t[2],
                               (int)G.n[1], (int)G.n[2], d.kernel_alpha, S(st));
    });
    if (r.bad()) return r;
    d.stats.n_kernels++;
    return Status::ok();
  }
  Status slab_sweep2(Domain& d, const SlabRef& src, const SlabRef& mid, const SlabRef& dst, int a, int b,
                     int st) override {
    INJECT(FAULT_KERNEL, st);
    if (d.measure == TILE_MEASURE_XFER_ONLY) return Status::ok();
    ensure_maps(d);
    const SlabView s = slab_view(d, src, a), m = slab_view(d, mid, a), t = slab_view(d, dst, a);
    bool fused = true;
    next_cells = d.kernel_timing ? (uint64_t)(b - a) * d.G.l[0] * d.G.l[1] : 0;  // one pass over the cells
    // the band layout (heat2_band_slab) when the grid is 512 wide and every
    // view has its tensor maps; else the tile-column kernel
    Band2View bv[2];
    Band2Out bo[2];
    const bool band = band2_slab_on(d) && band2_in(d, src, &bv[0]) && band2_in(d, mid, &bv[1]) &&
                      band2_out(d, mid, 0, &bo[0]) && band2_out(d, dst, 0, &bo[1]);
    Status r = timed(d, st, [&] {
      const Geometry& G = d.G;
      const cudaError_t e =
          band ? launch_heat2_band_slab(1, bv[0], bv[1], bo[0], bo[1], (int)G.t[1], (int)G.n[1], a, b,
                                        d.kernel_alpha, S(st))
               : launch_slab_sweep2(s, m, t, (int)G.l[0], (int)G.l[1], a, b, d.kernel_alpha, sms, S(st), &maps);
      if (e == cudaErrorNotSupported) {
        fused = false;
        cudaGetLastError();
        return cudaSuccess;
      }
      return e;
    });
    if (r.bad()) return r;
    if (!fused) {  // shapes the fused kernel does not cover: both levels in full, one after the other
      r = slab_sweep(d, src, mid, a, b, st);
      if (r.bad()) return r;
      return slab_sweep(d, mid, dst, a - 1, b - 1, st);
    }
    d.stats.n_kernels++;
    return Status::ok();
  }
  Status h2d_part(Domain& d, int64_t t0, int64_t n, int s0, int64_t p0, int64_t np, int st) override {
    INJECT(FAULT_H2D, st);
    if (d.measure == TILE_MEASURE_COMP_ONLY) return Status::ok();
    const size_t pl = (size_t)d.G.t[0] * d.G.t[1] * 8, tb = (size_t)d.G.tile_elems * 8;
    CK(cudaMemcpy2DAsync(reinterpret_cast<char*>(d.slot_ptr(s0)) + p0 * pl, tb,
                         reinterpret_cast<const char*>(d.host_tile(t0)) + p0 * pl, tb, np * pl,
                         (size_t)n, cudaMemcpyHostToDevice, S(st)));
    d.stats.bytes_h2d += (uint64_t)n * np * pl;
    d.stats.n_h2d++;
    return Status::ok();
  }
  // TILES_D2H_KERNEL=N (N > 0 CTAs): partial D2H copies by the SMs into the
  // mapped host store instead of the copy engine (experiment)
  int push_ctas() {
    static const int n = [] {
      const char* e = getenv("TILES_D2H_KERNEL");
      return e ? atoi(e) : 0;
    }();
    return n;
  }
  double* host_dev(Domain& d, int64_t t) {
    if (!host_dptr) {
      void* p = nullptr;
      if (cudaHostGetDevicePointer(&p, d.host, 0) != cudaSuccess) return nullptr;
      host_dptr = static_cast<double*>(p);
    }
    return host_dptr + t * d.G.tile_elems;
  }
  double* host_dptr = nullptr;
  Status d2h_part(Domain& d, int64_t t0, int64_t n, int ps, int64_t p0, int64_t np, int st) override {
    INJECT(FAULT_D2H, st);
    if (d.measure == TILE_MEASURE_COMP_ONLY) return Status::ok();
    const size_t pl = (size_t)d.G.t[0] * d.G.t[1] * 8, tb = (size_t)d.G.tile_elems * 8;
    if (push_ctas() > 0 && !d.opt.pageable_host && host_dev(d, t0)) {
      const int64_t pe = (int64_t)(pl / 8);
      CK(launch_push_rows(d.slot_ptr(ps), np * pe, host_dev(d, t0) + p0 * pe, d.G.tile_elems, n, np * pe,
                          push_ctas(), S(st)));
      d.stats.bytes_d2h += (uint64_t)n * np * pl;
      d.stats.n_d2h++;
      return Status::ok();
    }
    CK(cudaMemcpy2DAsync(reinterpret_cast<char*>(d.host_tile(t0)) + p0 * pl, tb, d.slot_ptr(ps),
                         np * pl, np * pl, (size_t)n, cudaMemcpyDeviceToHost, S(st)));
    d.stats.bytes_d2h += (uint64_t)n * np * pl;
    d.stats.n_d2h++;
    return Status::ok();
  }
  Status h2d_pack(Domain& d, int64_t t0, int64_t n, int ps, int64_t p0, int64_t np, int st) override {
    INJECT(FAULT_H2D, st);
    if (d.measure == TILE_MEASURE_COMP_ONLY) return Status::ok();
    const size_t pl = (size_t)d.G.t[0] * d.G.t[1] * 8, tb = (size_t)d.G.tile_elems * 8;
    CK(cudaMemcpy2DAsync(d.slot_ptr(ps), np * pl, reinterpret_cast<const char*>(d.host_tile(t0)) + p0 * pl,
                         tb, np * pl, (size_t)n, cudaMemcpyHostToDevice, S(st)));
    d.stats.bytes_h2d += (uint64_t)n * np * pl;
    d.stats.n_h2d++;
    return Status::ok();
  }
  Status copy_part(Domain& d, int ps, int s0, int64_t n, int64_t p0, int64_t np, int st) override {
    if (d.measure == TILE_MEASURE_XFER_ONLY) return Status::ok();
    const size_t pl = (size_t)d.G.t[0] * d.G.t[1] * 8, tb = (size_t)d.G.tile_elems * 8;
    CK(cudaMemcpy2DAsync(reinterpret_cast<char*>(d.slot_ptr(s0)) + p0 * pl, tb, d.slot_ptr(ps),
                         np * pl, np * pl, (size_t)n, cudaMemcpyDeviceToDevice, S(st)));
    return Status::ok();
  }
  Status d2h_planes(Domain& d, int64_t t0, int64_t n, int s0, int64_t p0, int64_t np, int st) override {
    INJECT(FAULT_D2H, st);
    if (d.measure == TILE_MEASURE_COMP_ONLY) return Status::ok();
    const size_t pl = (size_t)d.G.t[0] * d.G.t[1] * 8, tb = (size_t)d.G.tile_elems * 8;
    if (push_ctas() > 0 && !d.opt.pageable_host && host_dev(d, t0)) {
      const int64_t pe = (int64_t)(pl / 8);
      CK(launch_push_rows(d.slot_ptr(s0) + p0 * pe, d.G.tile_elems, host_dev(d, t0) + p0 * pe, d.G.tile_elems, n,
                          np * pe, push_ctas(), S(st)));
      d.stats.bytes_d2h += (uint64_t)n * np * pl;
      d.stats.n_d2h++;
      return Status::ok();
    }
    CK(cudaMemcpy2DAsync(reinterpret_cast<char*>(d.host_tile(t0)) + p0 * pl, tb,
                         reinterpret_cast<const char*>(d.slot_ptr(s0)) + p0 * pl, tb, np * pl, (size_t)n,
                         cudaMemcpyDeviceToHost, S(st)));
    d.stats.bytes_d2h += (uint64_t)n * np * pl;
    d.stats.n_d2h++;
    return Status::ok();
  }
  Status copy_planes(Domain& d, int src0, int dst0, int64_t n, int64_t p0, int64_t np, int st) override {
    if (d.measure == TILE_MEASURE_XFER_ONLY) return Status::ok();
    const size_t pl = (size_t)d.G.t[0] * d.G.t[1] * 8, tb = (size_t)d.G.tile_elems * 8;
    CK(cudaMemcpy2DAsync(reinterpret_cast<char*>(d.slot_ptr(dst0)) + p0 * pl, tb,
                         reinterpret_cast<const char*>(d.slot_ptr(src0)) + p0 * pl, tb, np * pl, (size_t)n,
                         cudaMemcpyDeviceToDevice, S(st)));
    return Status::ok();
  }
  Status copy_slots(Domain& d, int src, int dst, int64_t n, int st) override {
    if (d.measure == TILE_MEASURE_XFER_ONLY) return Status::ok();
    CK(cudaMemcpyAsync(d.slot_ptr(dst), d.slot_ptr(src), (size_t)n * d.G.tile_elems * 8,
                       cudaMemcpyDeviceToDevice, S(st)));
    return Status::ok();
  }
  int heat2_occ = 0;
  Status heat2(Domain& d, const int64_t* tiles, const int* in, const int* out, int n, int rp,
               const TileItem* dev_items, int st) override {
    INJECT(FAULT_KERNEL, st);
    if (d.measure == TILE_MEASURE_XFER_ONLY || n == 0) return Status::ok();
    Heat2Params P{};
    HeatParams& p = P.h;
    p.tx = (int)d.G.t[0];
    p.ty = (int)d.G.t[1];
    p.tz = (int)d.G.t[2];
    p.band = d.band2;
    p.nbands = p.ty / d.band2;
    p.nitems = n;
    p.alpha = d.kernel_alpha;
    p.cache_flags = d.heat_cache_flags;
    p.depth = 2;
    if (dev_items) {
      p.items = dev_items;
    } else {
      if (n > kMaxInlineItems) return make_err(TILE_ESTATE, "internal: too many inline items");
      for (int i = 0; i < n; ++i)
        p.inline_items[i] = {d.slot_ptr(in[i]), d.slot_ptr(out[i]), (int32_t)tiles[i], 0};
    }
    p.gsrc = d.gsrc_dev[rp];
    for (int f = 0; f < 6; ++f) {
      p.fexp[f] = d.faces[f][rp ^ 1];
      p.face_elems[f] = d.G.face_elems[f];
    }
    p.nstack = 1;
    p.lt = n;
    p.exp_y = 1;
    p.exp_zlo_below = INT32_MAX;
    P.esrc = d.esrc_dev[rp];
    P.fixed_mask = d.fixed_mask_dev;
    const int64_t planes = (int64_t)n * p.nbands * p.tz;
    int64_t grid = (int64_t)sms * heat2_occ;
    grid = std::max<int64_t>(1, std::min<int64_t>(grid, (planes + 3) / 4));
    next_cells = d.kernel_timing ? (uint64_t)n * d.G.tile_elems : 0;  // one pass for two steps
    Status r = timed(d, st, [&] { return launch_heat7x2(P, d.heat2_smem, (int)grid, S(st)); });
    if (r.bad()) return r;
    d.stats.n_kernels++;
    return Status::ok();
  }
  Status sincos(Domain& d, int64_t t, int slot, int64_t iters, int st) override {
    INJECT(FAULT_KERNEL, st);
    if (d.measure == TILE_MEASURE_XFER_ONLY) return Status::ok();
    if (d.user_fn) {  // TILE_KERNEL_USER: the caller's compiled pointwise function
      int64_t ix, iy, iz;
      d.G.tile_coords(t, &ix, &iy, &iz);
      const int64_t td[2] = {d.G.t[0], d.G.t[1]};
      const int64_t org[3] = {ix * d.G.t[0], iy * d.G.t[1], d.G.zoff + iz * d.G.t[2]};
      const int64_t gd[2] = {d.G.g[0], d.G.g[1]};
      const int64_t* b = d.user_box;
      for (int a = 0; a < 3; ++a)  // ranged compute: a tile outside the box launches nothing
        if (org[a] >= b[3 + a] || org[a] + d.G.t[a] <= b[a]) return Status::ok();
      Status r = timed_status(d, st, [&] {
        return userfn_launch(d.user_fn, d.slot_ptr(slot), d.G.tile_elems, td, org, gd, iters, b, S(st));
      });
      if (r.bad()) return r;
      d.stats.n_kernels++;
      return Status::ok();
    }
    SincosParams p{};
    p.tile_elems = d.G.tile_elems;
    p.nitems = 1;
    p.iters = iters;
    p.items = nullptr;
    p.inline_items[0] = {d.slot_ptr(slot), d.slot_ptr(slot), (int32_t)t, 0};
    const int64_t pairs = d.G.tile_elems / 2;
    int64_t grid = std::min<int64_t>((pairs + 255) / 256, (int64_t)sms * 8);
    Status r = timed(d, st, [&] { return launch_sincos(p, (int)std::max<int64_t>(1, grid), S(st)); });
    if (r.bad()) return r;
    d.stats.n_kernels++;
    return Status::ok();
  }
  Status extract(Domain& d, int64_t t0, int64_t n, int s0, int par, const TileItem* dev_items,
                 int st) override {
    if (d.measure == TILE_MEASURE_XFER_ONLY || n == 0) return Status::ok();
    ExtractParams p{};
    p.depth = d.G.depth;
    p.tx = (int)d.G.t[0];
    p.ty = (int)d.G.t[1];
    p.tz = (int)d.G.t[2];
    p.nitems = (int)n;
    if (dev_items) {
      p.items = dev_items;
    } else {
      if (n > kMaxInlineItems) return make_err(TILE_ESTATE, "internal: too many inline items");
      for (int64_t i = 0; i < n; ++i)
        p.inline_items[i] = {d.slot_ptr(s0 + (int)i), nullptr, (int32_t)(t0 + i), 0};
    }
    for (int f = 0; f < 6; ++f) {
      p.fexp[f] = d.faces[f][par];
      p.face_elems[f] = d.G.face_elems[f];
    }
    Status r = timed(d, st, [&] { return launch_extract(p, S(st)); });
    if (r.bad()) return r;
    d.stats.n_kernels++;
    return Status::ok();
  }
  Status faces_h2d(Domain& d, int par, int st) override {
    if (d.measure == TILE_MEASURE_COMP_ONLY) return Status::ok();
    for (int f = 0; f < 6; ++f) {
      const size_t bytes = (size_t)d.G.ntiles * d.G.face_elems[f] * 8;
      CK(cudaMemcpyAsync(d.faces[f][par], d.host_faces[f], bytes, cudaMemcpyHostToDevice, S(st)));
      d.stats.bytes_h2d += bytes;
      d.stats.n_h2d++;
    }
    return Status::ok();
  }
  Status halo(Domain& d, int par, int st, int mode) override {
    if (d.opt.local_group) {
      if (!local_ready) CK(cudaEventCreateWithFlags(&local_ready, cudaEventDisableTiming));
      Status r = local_halo(d, par, S(st), local_ready);
      if (r.bad()) return r;
      d.stats.n_halo++;
      return Status::ok();
    }
    Status r = d.opt.peer_transport ? peer_halo(d, par, S(st), mode) : nccl_halo(d, par, S(st));
    if (r.bad()) return r;
    d.stats.n_halo++;
    return Status::ok();
  }
  Status st_halo(Domain& d, int op, int side, int T, int st) override {
    Status r = peer_st_halo(d, op, side, T, S(st));
    if (r.bad()) return r;
    if (op == 0) d.stats.n_halo++;
    return Status::ok();
  }
  Status note(Domain&, int, int64_t, int64_t, int) override { return Status::ok(); }
  Status sync_all(Domain& d) override {
    INJECT(FAULT_SYNC, 0);
    Status r = close_all();
    if (r.bad()) return r;
    for (auto s : streams) CK(cudaStreamSynchronize(s));
    return collect(d);
  }
  // Link: best of 3 H2D copies of up to 64 MiB from the pinned tile store
  // (duplex H2D runs at ~0.87 of the solo rate on PCIe 5, pcie_gap.json).
  // Sweep: best of 3 sweeps of 32 planes between the two resident arrays
  // (zeroed first: no uninitialised reads). Both timed with events on
  // stream 0, before any user data exists.
  Status calibrate(Domain& d, double* r) override {
    *r = 0;
    const Geometry& G = d.G;
    const uint64_t plane_b = (uint64_t)G.l[0] * G.l[1] * 8;
    const uint64_t nb = std::min<uint64_t>(64ull << 20, (uint64_t)G.ntiles * G.tile_elems * 8);
    const int planes = (int)std::min<int64_t>(32, G.l[2] - 2);  // a wavefront chunk
    cudaStream_t s0 = S(0);
    cudaEvent_t a, b;
    CK(cudaEventCreate(&a));
    CK(cudaEventCreate(&b));
    float best_l = 1e30f, best_s = 1e30f;
    Status res = Status::ok();
    ensure_maps(d);
    auto run = [&]() -> cudaError_t {
      cudaError_t e = cudaMemsetAsync(d.slot_ptr(0), 0, (size_t)planes * plane_b + plane_b, s0);
      if (e != cudaSuccess) return e;
      for (int i = 0; i < 4; ++i) {  // first rep warms the pinned pages
        if ((e = cudaEventRecord(a, s0)) != cudaSuccess) return e;
        if ((e = cudaMemcpyAsync(d.slot_ptr(0), d.host, nb, cudaMemcpyHostToDevice, s0)) != cudaSuccess) return e;
        if ((e = cudaEventRecord(b, s0)) != cudaSuccess) return e;
        if ((e = cudaEventSynchronize(b)) != cudaSuccess) return e;
        float ms = 0;
        cudaEventElapsedTime(&ms, a, b);
        if (i) best_l = std::min(best_l, ms);
      }
      SlabView v{};
      v.base = d.slot_ptr(0);
      v.te = G.tile_elems;
      v.tx = (int)G.t[0];
      v.ty = (int)G.t[1];
      v.tz = (int)G.t[2];
      v.ntx = (int)G.n[0];
      v.nty = (int)G.n[1];
      v.nz = (int)G.l[2];
      SlabView w = v;
      w.base = d.slot_ptr((int)G.ntiles);
      if ((e = cudaMemsetAsync(d.slot_ptr(0), 0, (size_t)G.ntiles * G.tile_elems * 8, s0)) != cudaSuccess) return e;
      for (int i = 0; i < 4; ++i) {
        if ((e = cudaEventRecord(a, s0)) != cudaSuccess) return e;
        if ((e = launch_slab_sweep(v, w, (int)G.l[0], (int)G.l[1], 1, 1 + planes, 0.125, sms, s0, &maps)) !=
            cudaSuccess)
          return e;
        if ((e = cudaEventRecord(b, s0)) != cudaSuccess) return e;
        if ((e = cudaEventSynchronize(b)) != cudaSuccess) return e;
        float ms = 0;
        cudaEventElapsedTime(&ms, a, b);
        if (i) best_s = std::min(best_s, ms);
      }
      return cudaSuccess;
    };
    const cudaError_t e = run();
    cudaEventDestroy(a);
    cudaEventDestroy(b);
    if (e != cudaSuccess) return cuda_err(e, "calibration");
    const double link_plane = (double)best_l / ((double)nb / (double)plane_b) / 0.87;  // ms per plane, duplex
    const double sweep_plane = (double)best_s / planes;
    if (link_plane > 0 && sweep_plane > 0) *r = sweep_plane / link_plane;
    return res;
  }
  Status mem_info(Domain&, uint64_t* fr, uint64_t* tot) override {
    size_t f = 0, t = 0;
    CK(cudaMemGetInfo(&f, &t));
    *fr = f;
    *tot = t;
    return Status::ok();
  }
  Status alloc_host(Domain& d, uint64_t bytes, void** p) override {
    if (d.opt.pageable_host) {  // baseline only: pageable memory
      *p = std::malloc(bytes ? bytes : 1);
      if (!*p) return make_err(TILE_ENOMEM_HOST, "malloc failed");
      std::memset(*p, 0, bytes);
      return Status::ok();
    }
    // pinned (page-locked) host regions, P:L73 (cudaMallocHost); an injected
    // fault asks for more than any host has
    const uint64_t req = fault_fires(d, FAULT_HOST_ALLOC) ? (1ull << 62) : (bytes ? bytes : 1);
    cudaError_t e = cudaHostAlloc(p, req, cudaHostAllocPortable | cudaHostAllocMapped);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return make_err(TILE_ENOMEM_HOST, std::string("cudaHostAlloc: ") + cudaGetErrorString(e));
    }
    return Status::ok();
  }
  void free_host(Domain& d, void* p) override {
    if (d.opt.pageable_host)
      std::free(p);
    else
      cudaFreeHost(p);
  }
  Status alloc_device(Domain&, uint64_t bytes, void** p) override {
    cudaError_t e = cudaMalloc(p, bytes);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return make_err(TILE_ENOMEM_DEVICE, std::string("cudaMalloc: ") + cudaGetErrorString(e));
    }
    return Status::ok();
  }
  void free_device(Domain&, void* p) override { cudaFree(p); }

  Status setup(Domain& d) override {
    const int nst = d.halo_stream + 1;
    streams.assign((size_t)nst, nullptr);
    own_stream.assign((size_t)nst, 0);
    for (int i = 0; i < nst; ++i) {
      if (i < d.opt.nstreams_provided && d.opt.streams && d.opt.streams[i]) {
        streams[(size_t)i] = static_cast<cudaStream_t>(d.opt.streams[i]);
      } else {
        CK(cudaStreamCreateWithFlags(&streams[(size_t)i], cudaStreamNonBlocking));
        own_stream[(size_t)i] = 1;
      }
    }
    events.assign((size_t)d.nevents, nullptr);
    for (auto& e : events) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    // events start "completed": record each once on stream 0
    for (auto& e : events) CK(cudaEventRecord(e, streams[0]));
    for (int p = 0; p < 2; ++p) {
      CK(cudaMemcpy(d.gsrc_dev[p], d.gsrc_host[p].data(), d.gsrc_host[p].size() * sizeof(void*),
                    cudaMemcpyHostToDevice));
      if (d.mode == MODE_RESIDENT)
        CK(cudaMemcpy(d.items_dev[p], d.items_host[p].data(),
                      d.items_host[p].size() * sizeof(TileItem), cudaMemcpyHostToDevice));
    }
    if (d.direct_ok) {
      for (int b = 0; b < 2; ++b)
        for (int p = 0; p < 2; ++p)
          CK(cudaMemcpy(d.gdir_dev[b][p], d.gdir_host[b][p].data(), d.gdir_host[b][p].size() * sizeof(void*),
                        cudaMemcpyHostToDevice));
      CK(cudaMemcpy(d.ystr_dev, d.ystr_host.data(), d.ystr_host.size() * sizeof(int64_t),
                    cudaMemcpyHostToDevice));
    }
    CK(heat_configure((int)d.G.t[0], (int)d.G.t[1], d.band, d.stages, d.heat_smem, &heat_occ));
    {
      int dev = 0;
      CK(cudaGetDevice(&dev));
      CK(cudaDeviceGetAttribute(&coop, cudaDevAttrCooperativeLaunch, dev));
    }
    CK(cudaMemset(d.prog_dev, 0, (size_t)kMaxProgCtas * sizeof(unsigned long long)));
    if (d.x2_ok) {
      CK(heat2_configure((int)d.G.t[0], d.band2, d.heat2_smem, &heat2_occ));
      if (heat2_occ < 1) {  // cannot be resident (e.g. profiler-reserved shared memory)
        std::fprintf(stderr, "libtiles: two-step kernel (band %d, %zu B shared) not resident on an SM; "
                     "using single steps\n", d.band2, d.heat2_smem);
        d.x2_ok = false;
      }
      for (int p = 0; p < 2 && d.x2_ok; ++p)
        CK(cudaMemcpy(d.esrc_dev[p], d.esrc_host[p].data(), d.esrc_host[p].size() * sizeof(EdgePtr),
                      cudaMemcpyHostToDevice));
      if (d.x2_ok)
        CK(cudaMemcpy(d.fixed_mask_dev, d.fixed_mask_host.data(), d.fixed_mask_host.size(),
                      cudaMemcpyHostToDevice));
    }
    if (heat_occ < 1) return make_err(TILE_EINVAL, "heat kernel cannot be resident on an SM");
    CK(cudaStreamSynchronize(streams[0]));
    return Status::ok();
  }
  Status upload_dir(Domain& d) override {
    for (int f = 0; f < 6; ++f)
      CK(cudaMemcpy(d.dir_faces[f], d.host_dir[f], (size_t)d.G.ntiles * d.G.face_elems[f] * 8,
                    cudaMemcpyHostToDevice));
    return Status::ok();
  }
  void destroy(Domain&) override {
    for (auto& pr : tpending) {
      tpool.push_back(pr.a);
      tpool.push_back(pr.b);
    }
    tpending.clear();
    for (auto e : tpool) cudaEventDestroy(e);
    tpool.clear();
    if (local_ready) cudaEventDestroy(local_ready);
    if (t_begin) cudaEventDestroy(t_begin);
    if (t_end) cudaEventDestroy(t_end);
    for (auto e : events)
      if (e) cudaEventDestroy(e);
    for (size_t i = 0; i < streams.size(); ++i)
      if (own_stream[i] && streams[i]) cudaStreamDestroy(streams[i]);
    events.clear();
    streams.clear();
    if (iter_flags) cudaFree(iter_flags);
    iter_flags = nullptr;
  }
};

}  // namespace

Exec* make_cuda_exec(Domain& d, Status* st) {
  auto* x = new CudaExec();
  int dev = d.opt.device;
  cudaError_t e = cudaSuccess;
  if (dev < 0) e = cudaGetDevice(&dev);
  if (e == cudaSuccess) e = cudaSetDevice(dev);
  if (e == cudaSuccess) e = cudaDeviceGetAttribute(&x->sms, cudaDevAttrMultiProcessorCount, dev);
  if (e != cudaSuccess) {
    *st = cuda_err(e, "device setup (is a CUDA device visible?)");
    delete x;
    return nullptr;
  }
  x->dev = dev;
  d.device = dev;
  d.sm_count = x->sms;
  *st = Status::ok();
  return x;
}

}  // namespace tiles
