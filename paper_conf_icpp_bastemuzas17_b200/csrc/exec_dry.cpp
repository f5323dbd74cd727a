// exec_dry.cpp — dry-run executor: no CUDA call at all; every operation the
// scheduler issues is appended to the domain's op trace (tile_trace), so the
// residency protocol and the dependency structure can be checked on a CPU.
#include <cstdlib>
#include <cstring>

#include "runtime.hpp"

namespace tiles {
namespace {

struct DryExec final : Exec {
  // TILES_FAULT in a dry run: the failing operation reports TILE_ECUDA as
  // the CUDA executor's would (nothing is recorded for it)
  static Status inject(Domain& d, int kind) {
    return fault_fires(d, kind) ? make_err(TILE_ECUDA, "injected fault (TILES_FAULT, dry run)") : Status::ok();
  }
  void put(Domain& d, int kind, int stream, int64_t a, int64_t b, int64_t c, int64_t dd) {
    tile_op op;
    op.kind = kind;
    op.stream = stream;
    op.a = a;
    op.b = b;
    op.c = c;
    op.d = dd;
    d.trace.push_back(op);
  }
  Status h2d(Domain& d, int64_t t0, int64_t n, int s0, int st) override {
    if (Status f_ = inject(d, FAULT_H2D); f_.bad()) return f_;
    d.stats.bytes_h2d += (uint64_t)n * d.G.tile_elems * 8;
    d.stats.n_h2d++;
    put(d, TILE_OP_H2D, st, t0, s0, n, 0);
    return Status::ok();
  }
  Status d2h(Domain& d, int64_t t0, int64_t n, int s0, int st) override {
    if (Status f_ = inject(d, FAULT_D2H); f_.bad()) return f_;
    d.stats.bytes_d2h += (uint64_t)n * d.G.tile_elems * 8;
    d.stats.n_d2h++;
    put(d, TILE_OP_D2H, st, t0, s0, n, 0);
    return Status::ok();
  }
  Status record(Domain& d, int ev, int st) override {
    put(d, TILE_OP_RECORD, st, ev, 0, 0, 0);
    return Status::ok();
  }
  Status wait(Domain& d, int ev, int st) override {
    put(d, TILE_OP_WAIT, st, ev, 0, 0, 0);
    return Status::ok();
  }
  Status heat(Domain& d, const int64_t* tiles, const int* in, const int* out, int n, int rp,
              const TileItem* dev_items, int st, int direct_bit, int nstack, int nsteps) override {
    if (Status f_ = inject(d, FAULT_KERNEL); f_.bad()) return f_;
    if (nsteps > 1) {  // a persistent launch: the same ops as nsteps single steps
      const int64_t off = dev_items - d.items_dev[direct_bit];
      for (int s = 0; s < nsteps; ++s) {
        const int b = direct_bit ^ (s & 1);
        Status r = heat(d, tiles, in, out, n, rp ^ (s & 1), d.items_dev[b] + off, st, b, nstack, 1);
        if (r.bad()) return r;
      }
      d.stats.n_kernels -= (uint64_t)nsteps - 1;  // one launch
      return Status::ok();
    }
    d.stats.n_kernels++;
    if (nstack < 1 || n % nstack) return make_err(TILE_ESTATE, "internal: bad tile stack");
    const int kind = direct_bit >= 0 ? TILE_OP_KERNELD : TILE_OP_KERNEL;
    // d of a direct op: read parity | 0x100 when the launch pushes its slab-end
    // z exports into the neighbour ranks' receive buffers (fused halo)
    const int push = direct_bit >= 0 && d.G.nranks > 1 && d.peer_fused ? 0x100 : 0;
    if (dev_items) {  // resident batch: items are a slice of items_host[bit]
      const int bit = dev_items >= d.items_dev[1] && d.items_dev[1] ? 1 : 0;
      const int64_t k0 = dev_items - d.items_dev[bit];
      for (int i = 0; i < n; ++i) {
        const TileItem& it = d.items_host[bit][(size_t)(k0 + i)];
        const int is = (int)((it.in - d.slot_base) / d.G.tile_elems);
        const int os = (int)((it.out - d.slot_base) / d.G.tile_elems);
        put(d, kind, st, it.tile, is, os, rp | push);
      }
    } else {
      for (int i = 0; i < n; ++i) put(d, kind, st, tiles[i], in[i], out[i], rp | push);
    }
    return Status::ok();
  }
  Status heat2(Domain& d, const int64_t* tiles, const int* in, const int* out, int n, int rp,
               const TileItem* dev_items, int st) override {
    if (Status f_ = inject(d, FAULT_KERNEL); f_.bad()) return f_;
    const size_t mark = d.trace.size();
    Status r = heat(d, tiles, in, out, n, rp, dev_items, st, -1, 1, 1);
    for (size_t i = mark; i < d.trace.size(); ++i) d.trace[i].kind = TILE_OP_KERNEL2;
    return r;
  }
  Status slab_sweep(Domain& d, const SlabRef& src, const SlabRef& dst, int lo, int hi, int st) override {
    if (Status f_ = inject(d, FAULT_KERNEL); f_.bad()) return f_;
    d.stats.n_kernels++;
    if (src.kind == SlabRef::UNITS) {
      // a: destination code as below; b: unit slots (u-1, u, u+1) packed 21
      // bits each; c: lo | hi << 32; d: u | un << 32
      const int64_t b = dst.kind == SlabRef::DENSE ? dst.slot : -1 - (int64_t)dst.slot;
      put(d, TILE_OP_SWEEP_U, st, b,
          (int64_t)src.ring[0] | ((int64_t)src.ring[1] << 21) | ((int64_t)src.ring[2] << 42),
          (int64_t)lo | ((int64_t)hi << 32), src.u | (src.un << 32));
      return Status::ok();
    }
    if (src.kind == SlabRef::WAVE || dst.kind == SlabRef::WAVE) {
      // wavefront sweep: view codes (bit 0: 1 = WAVE, 0 = RESIDENT wrapped at
      // zbase 0; bit 1: the resident array; bits 2..: WAVE scratch slot);
      // c: lo, hi as two signed 32-bit halves; d: scratch layers (nlo)
      auto code = [](const SlabRef& r) {
        return r.kind == SlabRef::WAVE ? 1 | ((int64_t)r.slot << 1) | ((int64_t)r.ring[0] << 32)
                                       : ((int64_t)r.slot << 1);
      };
      put(d, TILE_OP_WSWEEP, st, code(src), code(dst),
          (int64_t)(uint32_t)lo | ((int64_t)(uint32_t)hi << 32), dst.kind == SlabRef::WAVE ? dst.un : src.un);
      return Status::ok();
    }
    // a: slab slot, or -1-bit for the resident array (slab plane 0 at z = d)
    // b: slab slot, or -1-slot for packed sub-tiles (sweep plane lo -> 0)
    const int64_t a = src.kind == SlabRef::DENSE ? src.slot : -1 - (int64_t)src.slot;
    const int64_t b = dst.kind == SlabRef::DENSE ? dst.slot : -1 - (int64_t)dst.slot;
    put(d, TILE_OP_SWEEP, st, a, b, (int64_t)lo | ((int64_t)hi << 32),
        src.kind == SlabRef::RESIDENT ? src.zbase : 0);
    return Status::ok();
  }
  bool band2_ok(Domain&) override { return true; }
  bool wave_iter_ok(Domain& d) override { return sweep2s_ok(d); }
  Status wave_iteration(Domain& d, const SlabRef* lv, int64_t ci, int c, int s0, int P, int st) override {
    for (int k = 0; k < P; ++k) {
      const int s = s0 + 2 * k;
      const SlabRef& src = s - 1 == 0 ? lv[3] : lv[(s - 1) % 3];
      Status r = slab_sweep2(d, src, lv[s % 3], lv[(s + 1) % 3], (int)(ci - s), (int)(ci - s + c), st);
      if (r.bad()) return r;
    }
    return Status::ok();
  }
  bool sweep2s_ok(Domain& d) override {
    const Geometry& G = d.G;
    return G.nranks == 1 && band2_shape_ok(G.l[0], G.l[1], (int)G.t[0], (int)G.t[1]);
  }
  Status slab_sweep2s(Domain& d, const SlabRef& src, const SlabRef& dst, int lo, int hi, int st) override {
    if (Status f_ = inject(d, FAULT_KERNEL); f_.bad()) return f_;
    d.stats.n_kernels++;
    // codes as TILE_OP_SWEEP: a slab slot or -1-bit (resident, slab plane 0
    // at z = d); b slab slot or -1-slot (packed sub-tiles from plane lo+1)
    const int64_t a = src.kind == SlabRef::DENSE ? src.slot : -1 - (int64_t)src.slot;
    const int64_t b = dst.kind == SlabRef::DENSE ? dst.slot : -1 - (int64_t)dst.slot;
    put(d, TILE_OP_SWEEP2S, st, a, b, (int64_t)lo | ((int64_t)hi << 32),
        src.kind == SlabRef::RESIDENT ? src.zbase : 0);
    return Status::ok();
  }
  Status band2(Domain& d, int sbit, int dbit, int st) override {
    if (Status f_ = inject(d, FAULT_KERNEL); f_.bad()) return f_;
    d.stats.n_kernels++;
    put(d, TILE_OP_BAND2, st, (int64_t)sbit << 1, (int64_t)dbit << 1, d.G.l[2] << 32, 0);
    return Status::ok();
  }
  Status slab_sweep2(Domain& d, const SlabRef& src, const SlabRef& mid, const SlabRef& dst, int a, int b,
                     int st) override {
    if (Status f_ = inject(d, FAULT_KERNEL); f_.bad()) return f_;
    d.stats.n_kernels++;
    auto code = [](const SlabRef& r) {
      return r.kind == SlabRef::WAVE ? 1 | ((int64_t)r.slot << 1) | ((int64_t)r.ring[0] << 32) : ((int64_t)r.slot << 1);
    };
    // one kernel, two records (a trace entry has four operands): the
    // parameters, then the destination view (the replay executes at the second)
    put(d, TILE_OP_WSWEEP2, st, code(src), code(mid), (int64_t)(uint32_t)a | ((int64_t)(uint32_t)b << 32), dst.un);
    put(d, TILE_OP_WSWEEP2_DST, st, code(dst), 0, 0, 0);
    return Status::ok();
  }
  Status h2d_pack(Domain& d, int64_t t0, int64_t n, int ps, int64_t p0, int64_t np, int st) override {
    if (Status f_ = inject(d, FAULT_H2D); f_.bad()) return f_;
    d.stats.bytes_h2d += (uint64_t)n * np * d.G.t[0] * d.G.t[1] * 8;
    d.stats.n_h2d++;
    put(d, TILE_OP_H2D_PACK, st, t0, ps, n, p0 | (np << 32));
    return Status::ok();
  }
  Status h2d_part(Domain& d, int64_t t0, int64_t n, int s0, int64_t p0, int64_t np, int st) override {
    if (Status f_ = inject(d, FAULT_H2D); f_.bad()) return f_;
    d.stats.bytes_h2d += (uint64_t)n * np * d.G.t[0] * d.G.t[1] * 8;
    d.stats.n_h2d++;
    put(d, TILE_OP_H2D_PART, st, t0, s0, n, p0 | (np << 32));
    return Status::ok();
  }
  Status d2h_part(Domain& d, int64_t t0, int64_t n, int ps, int64_t p0, int64_t np, int st) override {
    if (Status f_ = inject(d, FAULT_D2H); f_.bad()) return f_;
    d.stats.bytes_d2h += (uint64_t)n * np * d.G.t[0] * d.G.t[1] * 8;
    d.stats.n_d2h++;
    put(d, TILE_OP_D2H_PART, st, t0, ps, n, p0 | (np << 32));
    return Status::ok();
  }
  Status copy_part(Domain& d, int ps, int s0, int64_t n, int64_t p0, int64_t np, int st) override {
    put(d, TILE_OP_COPY_PART, st, ps, s0, n, p0 | (np << 32));
    return Status::ok();
  }
  Status d2h_planes(Domain& d, int64_t t0, int64_t n, int s0, int64_t p0, int64_t np, int st) override {
    if (Status f_ = inject(d, FAULT_D2H); f_.bad()) return f_;
    d.stats.bytes_d2h += (uint64_t)n * np * d.G.t[0] * d.G.t[1] * 8;
    d.stats.n_d2h++;
    put(d, TILE_OP_D2H_PLANES, st, t0, s0, n, p0 | (np << 32));
    return Status::ok();
  }
  Status copy_planes(Domain& d, int src0, int dst0, int64_t n, int64_t p0, int64_t np, int st) override {
    put(d, TILE_OP_COPY_PLANES, st, src0, dst0, n, p0 | (np << 32));
    return Status::ok();
  }
  Status copy_slots(Domain& d, int src, int dst, int64_t n, int st) override {
    put(d, TILE_OP_COPY, st, src, dst, n, 0);
    return Status::ok();
  }
  Status sincos(Domain& d, int64_t t, int slot, int64_t iters, int st) override {
    if (Status f_ = inject(d, FAULT_KERNEL); f_.bad()) return f_;
    d.stats.n_kernels++;
    put(d, TILE_OP_POINTWISE, st, t, slot, iters, 0);
    return Status::ok();
  }
  Status extract(Domain& d, int64_t t0, int64_t n, int s0, int par, const TileItem*,
                 int st) override {
    d.stats.n_kernels++;
    for (int64_t i = 0; i < n; ++i) put(d, TILE_OP_EXTRACT, st, t0 + i, s0 + i, 0, par);
    return Status::ok();
  }
  Status faces_h2d(Domain& d, int par, int st) override {
    for (int f = 0; f < 6; ++f) d.stats.bytes_h2d += (uint64_t)d.G.ntiles * d.G.face_elems[f] * 8;
    put(d, TILE_OP_FACES_H2D, st, 0, 0, 0, par);
    return Status::ok();
  }
  Status halo(Domain& d, int par, int st, int mode) override {
    d.stats.n_halo++;
    d.stats.bytes_halo += 2ull * d.G.layer_tiles * d.G.face_elems[ZM] * 8;
    put(d, mode == 2 ? TILE_OP_HALO_SIGNAL : TILE_OP_HALO, st, mode, 0, 0, par);
    return Status::ok();
  }
  Status st_halo(Domain& d, int op, int side, int T, int st) override {
    if (op == 0) {
      d.stats.n_halo++;
      d.stats.bytes_halo += (uint64_t)d.G.layer_tiles * T * d.G.t[0] * d.G.t[1] * 8;
    }
    put(d, TILE_OP_ST_HALO, st, op, side, T, d.st_epoch);
    return Status::ok();
  }
  Status note(Domain& d, int kind, int64_t a, int64_t b, int st) override {
    put(d, kind, st, a, b, 0, 0);
    return Status::ok();
  }
  Status calibrate(Domain&, double* r) override {
    *r = 0;  // no device: the default fit
    return Status::ok();
  }
  Status sync_all(Domain& d) override {
    if (Status f_ = inject(d, FAULT_SYNC); f_.bad()) return f_;
    put(d, TILE_OP_SYNC, -1, 0, 0, 0, 0);
    return Status::ok();
  }
  Status mem_info(Domain& d, uint64_t* fr, uint64_t* tot) override {
    // a pretend device: the budget option (or 64 GiB) is all there is
    *tot = 180ull << 30;
    *fr = d.opt.device_budget_bytes ? d.opt.device_budget_bytes + (1ull << 30) : (64ull << 30);
    return Status::ok();
  }
  Status alloc_host(Domain& d, uint64_t bytes, void** p) override {
    if (fault_fires(d, FAULT_HOST_ALLOC)) return make_err(TILE_ENOMEM_HOST, "host allocation failed (injected)");
    *p = std::malloc(bytes ? bytes : 1);
    if (!*p) return make_err(TILE_ENOMEM_HOST, "host allocation failed");
    return Status::ok();
  }
  void free_host(Domain&, void* p) override { std::free(p); }
  Status alloc_device(Domain&, uint64_t, void** p) override {
    *p = reinterpret_cast<void*>(uintptr_t(1) << 40);  // never dereferenced
    return Status::ok();
  }
  void free_device(Domain&, void*) override {}
  Status setup(Domain&) override { return Status::ok(); }
  Status upload_dir(Domain& d) override {
    put(d, TILE_OP_FACES_H2D, 0, 1, 0, 0, -1);
    return Status::ok();
  }
  void destroy(Domain&) override {}
  Status timer_start(Domain&) override { return Status::ok(); }
  Status timer_stop(Domain&, double* ms) override {
    *ms = 0;
    return Status::ok();
  }
};

}  // namespace

Exec* make_dry_exec() { return new DryExec(); }

}  // namespace tiles
