// userfn.cpp — user pointwise kernels ("general
// kernels"; the paper's compute(tile) runs user code over a region,
// P:L126-L147). The caller supplies CUDA C source defining
//     __device__ double <name>(double u, long long gidx)
// which NVRTC compiles for sm_100a together with a grid-stride wrapper that
// applies it `iters` times to every cell of a tile in place; tile_run with
// TILE_KERNEL_USER then moves tiles through the same residency / streaming
// schedules as the compute-intensive kernel (pointwise, no ghosts). NVRTC is
// dlopen'ed (ENOSYS without it); the cubin is loaded per device with the
// driver API fetched through cudaGetDriverEntryPoint (the primary context
// cudart uses), so no -lcuda / -lnvrtc link dependency exists.
#include <cuda.h>
#include <cuda_runtime.h>
#include <dlfcn.h>

#include <algorithm>
#include <cctype>
#include <cstdio>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "runtime.hpp"

namespace tiles {
namespace {

// NVRTC entry points (nvrtc.h signatures, resolved with dlsym)
using nvrtcResult_t = int;
using nvrtcProgram_t = void*;
struct Nvrtc {
  nvrtcResult_t (*create)(nvrtcProgram_t*, const char*, const char*, int, const char* const*, const char* const*);
  nvrtcResult_t (*compile)(nvrtcProgram_t, int, const char* const*);
  nvrtcResult_t (*log_size)(nvrtcProgram_t, size_t*);
  nvrtcResult_t (*log)(nvrtcProgram_t, char*);
  nvrtcResult_t (*cubin_size)(nvrtcProgram_t, size_t*);
  nvrtcResult_t (*cubin)(nvrtcProgram_t, char*);
  nvrtcResult_t (*destroy)(nvrtcProgram_t*);
  bool ok = false;
};

Nvrtc& nvrtc() {
  static Nvrtc n;
  static std::once_flag once;
  std::call_once(once, [] {
    void* h = nullptr;
    for (const char* lib : {"libnvrtc.so.12", "libnvrtc.so", "/usr/local/cuda/lib64/libnvrtc.so.12"})
      if ((h = dlopen(lib, RTLD_NOW | RTLD_LOCAL))) break;
    if (!h) return;
    auto sym = [&](const char* s) { return dlsym(h, s); };
    n.create = reinterpret_cast<decltype(n.create)>(sym("nvrtcCreateProgram"));
    n.compile = reinterpret_cast<decltype(n.compile)>(sym("nvrtcCompileProgram"));
    n.log_size = reinterpret_cast<decltype(n.log_size)>(sym("nvrtcGetProgramLogSize"));
    n.log = reinterpret_cast<decltype(n.log)>(sym("nvrtcGetProgramLog"));
    n.cubin_size = reinterpret_cast<decltype(n.cubin_size)>(sym("nvrtcGetCUBINSize"));
    n.cubin = reinterpret_cast<decltype(n.cubin)>(sym("nvrtcGetCUBIN"));
    n.destroy = reinterpret_cast<decltype(n.destroy)>(sym("nvrtcDestroyProgram"));
    n.ok = n.create && n.compile && n.log_size && n.log && n.cubin_size && n.cubin && n.destroy;
  });
  return n;
}

// driver API through the runtime's entry-point query
struct Drv {
  CUresult (*load)(CUmodule*, const void*) = nullptr;
  CUresult (*get)(CUfunction*, CUmodule, const char*) = nullptr;
  CUresult (*launch)(CUfunction, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned, unsigned,
                     CUstream, void**, void**) = nullptr;
  CUresult (*unload)(CUmodule) = nullptr;
  bool ok = false;
};

Drv& drv() {
  static Drv d;
  static std::once_flag once;
  std::call_once(once, [] {
    cudaDriverEntryPointQueryResult q{};
    void* p = nullptr;
    if (cudaGetDriverEntryPoint("cuModuleLoadData", &p, cudaEnableDefault, &q) == cudaSuccess && p)
      d.load = reinterpret_cast<decltype(d.load)>(p);
    p = nullptr;
    if (cudaGetDriverEntryPoint("cuModuleGetFunction", &p, cudaEnableDefault, &q) == cudaSuccess && p)
      d.get = reinterpret_cast<decltype(d.get)>(p);
    p = nullptr;
    if (cudaGetDriverEntryPoint("cuLaunchKernel", &p, cudaEnableDefault, &q) == cudaSuccess && p)
      d.launch = reinterpret_cast<decltype(d.launch)>(p);
    p = nullptr;
    if (cudaGetDriverEntryPoint("cuModuleUnload", &p, cudaEnableDefault, &q) == cudaSuccess && p)
      d.unload = reinterpret_cast<decltype(d.unload)>(p);
    d.ok = d.load && d.get && d.launch && d.unload;
  });
  return d;
}

bool valid_identifier(const char* s) {
  if (!s || !*s || !(std::isalpha((unsigned char)s[0]) || s[0] == '_')) return false;
  for (const char* c = s; *c; ++c)
    if (!(std::isalnum((unsigned char)*c) || *c == '_')) return false;
  return std::strlen(s) < 128;
}

}  // namespace

struct UserFn {
  bool stencil = false;  // 7-point user stencil (tile_user_stencil_create)
  std::string name;
  std::vector<char> cubin;
  std::mutex m;
  std::vector<std::pair<int, CUmodule>> modules;  // per device
  std::vector<std::pair<int, CUfunction>> fns;
};

static Status compile(const std::string& src, const char* name, bool stencil, UserFn** out);

// 7-point user stencil: the face layouts and ghost conventions of the
// library's stencil kernels (HeatParams::gsrc / fexp, kernels.cuh), one
// thread per (x, y) column marching z (z-1, z in registers; in-plane
// neighbours through L1), ghosts from the read-parity faces, the new boundary
// layers exported to the write-parity faces for the next step's neighbours.
static const char* kStencilWrapper = R"(
struct TileItemJ { const double* in; double* out; int tile; int pad; };
extern "C" __global__ void tile_user_stencil(const TileItemJ* items, const double* in1, double* out1,
    int tile1, const double* const* gsrc, double* fx0, double* fx1, double* fy0, double* fy1,
    double* fz0, double* fz1, long long e0, long long e1, long long e2, long long e3, long long e4,
    long long e5, int tx, int ty, int tz, int D) {
  TileItemJ it;
  if (items) it = items[blockIdx.y]; else { it.in = in1; it.out = out1; it.tile = tile1; }
  const long long pl = (long long)tx * ty, t = it.tile;
  const double* const* gs = gsrc + t * 6;
  const double* u = it.in;
  // one thread per (x, y) column, marching z: z-1 and z stay in registers
  for (int col = blockIdx.x * blockDim.x + threadIdx.x; col < tx * ty; col += gridDim.x * blockDim.x) {
    const int x = col % tx, y = col / tx;
    double zm = gs[4][((long long)(D - 1) * ty + y) * tx + x];
    double c = u[col];
    for (int z = 0; z < tz; ++z) {
      const long long i = (long long)z * pl + col;
      const double zp = z < tz - 1 ? u[i + pl] : gs[5][(long long)y * tx + x];
      const double xm = x > 0 ? u[i - 1] : gs[0][((long long)z * ty + y) * D + (D - 1)];
      const double xp = x < tx - 1 ? u[i + 1] : gs[1][((long long)z * ty + y) * D];
      const double ym = y > 0 ? u[i - tx] : gs[2][((long long)z * D + (D - 1)) * tx + x];
      const double yp = y < ty - 1 ? u[i + tx] : gs[3][((long long)z * D) * tx + x];
      const double v = USER_STENCIL(c, xm, xp, ym, yp, zm, zp);
      it.out[i] = v;
      if (x < D) fx0[t * e0 + ((long long)z * ty + y) * D + x] = v;
      if (x >= tx - D) fx1[t * e1 + ((long long)z * ty + y) * D + (x - (tx - D))] = v;
      if (y < D) fy0[t * e2 + ((long long)z * D + y) * tx + x] = v;
      if (y >= ty - D) fy1[t * e3 + ((long long)z * D + (y - (ty - D))) * tx + x] = v;
      if (z < D) fz0[t * e4 + ((long long)z * ty + y) * tx + x] = v;
      if (z >= tz - D) fz1[t * e5 + ((long long)(z - (tz - D)) * ty + y) * tx + x] = v;
      zm = c;
      c = zp;
    }
  }
}
)";

Status userfn_create_stencil(const char* source, const char* name, UserFn** out) {
  if (!source || !out) return make_err(TILE_EINVAL, "null argument");
  if (!valid_identifier(name)) return make_err(TILE_EINVAL, "user function name must be a C identifier");
  std::string w = kStencilWrapper;
  const std::string key = "USER_STENCIL";
  w.replace(w.find(key), key.size(), name);
  return compile(std::string(source) + "\n" + w, name, true, out);
}

Status userfn_create(const char* source, const char* name, UserFn** out) {
  if (!source || !out) return make_err(TILE_EINVAL, "null argument");
  if (!valid_identifier(name)) return make_err(TILE_EINVAL, "user function name must be a C identifier");
  const std::string src = std::string(source) +
                          "\nextern \"C\" __global__ void tile_user_apply(double* __restrict__ u, long long n,"
                          " long long tx, long long ty, long long x0, long long y0, long long z0,"
                          " long long nx, long long ny, long long iters, long long bx0, long long by0,"
                          " long long bz0, long long bx1, long long by1, long long bz1) {\n"
                          "  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n;"
                          " i += (long long)gridDim.x * blockDim.x) {\n"
                          "    const long long lx = i % tx, r = i / tx, ly = r % ty, lz = r / ty;\n"
                          "    const long long X = x0 + lx, Y = y0 + ly, Z = z0 + lz;\n"
                          "    if (X < bx0 || X >= bx1 || Y < by0 || Y >= by1 || Z < bz0 || Z >= bz1) continue;\n"
                          "    const long long g = (Z * ny + Y) * nx + X;\n"
                          "    double v = u[i];\n"
                          "    for (long long k = 0; k < iters; ++k) v = " + std::string(name) + "(v, g);\n"
                          "    u[i] = v;\n  }\n}\n";
  return compile(src, name, false, out);
}

static Status compile(const std::string& src, const char* name, bool stencil, UserFn** out) {
  Nvrtc& n = nvrtc();
  if (!n.ok) return make_err(TILE_ENOSYS, "libnvrtc not available");
  nvrtcProgram_t prog = nullptr;
  if (n.create(&prog, src.c_str(), "tile_user.cu", 0, nullptr, nullptr) != 0)
    return make_err(TILE_EINVAL, "nvrtcCreateProgram failed");
  const char* opts[] = {"--gpu-architecture=sm_100a", "--std=c++17", "-default-device", "--fmad=false"};
  const int rc = n.compile(prog, 4, opts);
  size_t ls = 0;
  n.log_size(prog, &ls);
  std::string log(ls, '\0');
  if (ls) n.log(prog, &log[0]);
  if (rc != 0) {
    n.destroy(&prog);
    return make_err(TILE_EINVAL, "user kernel does not compile: " + log);
  }
  size_t cs = 0;
  n.cubin_size(prog, &cs);
  auto* f = new UserFn;
  f->stencil = stencil;
  f->name = name;
  f->cubin.resize(cs);
  n.cubin(prog, f->cubin.data());
  n.destroy(&prog);
  *out = f;
  return Status::ok();
}

void userfn_free(UserFn* f) {
  if (!f) return;
  Drv& d = drv();
  if (d.ok && !f->modules.empty()) {
    // each module was loaded in its device's primary context: make that
    // current for the unload (ranks of one process may use other devices)
    int cur = -1;
    const bool have_cur = cudaGetDevice(&cur) == cudaSuccess;
    for (auto& m : f->modules) {
      if (cudaSetDevice(m.first) != cudaSuccess || d.unload(m.second) != CUDA_SUCCESS)
        std::fprintf(stderr, "libtiles: user function module unload failed on device %d\n", m.first);
    }
    if (have_cur) cudaSetDevice(cur);
  }
  delete f;
}

static Status function_on_device(UserFn* f, CUfunction* out, int* dev_out) {
  Drv& d = drv();
  if (!d.ok) return make_err(TILE_ENOSYS, "driver entry points for module loading unavailable");
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return make_err(TILE_ECUDA, "cudaGetDevice");
  *dev_out = dev;
  std::lock_guard<std::mutex> lk(f->m);
  for (auto& p : f->fns)
    if (p.first == dev) {
      *out = p.second;
      return Status::ok();
    }
  CUmodule mod = nullptr;
  CUfunction fn = nullptr;
  if (d.load(&mod, f->cubin.data()) != CUDA_SUCCESS) return make_err(TILE_ECUDA, "cuModuleLoadData (user kernel)");
  if (d.get(&fn, mod, f->stencil ? "tile_user_stencil" : "tile_user_apply") != CUDA_SUCCESS) {
    d.unload(mod);
    return make_err(TILE_ECUDA, "cuModuleGetFunction");
  }
  f->modules.push_back({dev, mod});
  f->fns.push_back({dev, fn});
  *out = fn;
  return Status::ok();
}

bool userfn_is_stencil(const UserFn* f) { return f && f->stencil; }

Status userfn_launch_stencil(UserFn* f, const void* dev_items, int nitems, const double* in, double* out,
                             int tile, const double* const* gsrc, double* const fexp[6],
                             const int64_t face_elems[6], const int64_t t[3], int depth, void* stream) {
  CUfunction fn = nullptr;
  int dev = 0;
  Status s = function_on_device(f, &fn, &dev);
  if (s.bad()) return s;
  int tx = (int)t[0], ty = (int)t[1], tz = (int)t[2], D = depth, tl = tile;
  long long e[6];
  double* fx[6];
  for (int i = 0; i < 6; ++i) e[i] = face_elems[i], fx[i] = fexp[i];
  const void* items = dev_items;
  void* args[] = {&items, &in, &out, &tl, &gsrc, &fx[0], &fx[1], &fx[2], &fx[3], &fx[4], &fx[5],
                  &e[0], &e[1], &e[2], &e[3], &e[4], &e[5], &tx, &ty, &tz, &D};
  const long long cols = (long long)tx * ty;  // one thread per (x, y) column
  const long long bx = std::max<long long>(1, (cols + 255) / 256);
  // blockIdx.y = item: launch at most 65535 items at a time (gridDim.y limit;
  // the wrapper's TileItemJ has TileItem's layout)
  static_assert(sizeof(TileItem) == 24, "TileItemJ layout");
  constexpr int kMaxY = 65535;
  const int total = dev_items ? std::max(1, nitems) : 1;
  for (int i0 = 0; i0 < total; i0 += kMaxY) {
    const int ny = std::min(kMaxY, total - i0);
    items = dev_items ? static_cast<const void*>(static_cast<const TileItem*>(dev_items) + i0) : nullptr;
    if (drv().launch(fn, (unsigned)bx, (unsigned)ny, 1, 256, 1, 1, 0, static_cast<CUstream>(stream), args,
                     nullptr) != CUDA_SUCCESS)
      return make_err(TILE_ECUDA, "cuLaunchKernel (user stencil)");
  }
  return Status::ok();
}

Status userfn_launch(UserFn* f, double* data, int64_t n, const int64_t tdims[2], const int64_t org[3],
                     const int64_t gdims[2], int64_t iters, const int64_t box[6], void* stream) {
  Drv& d = drv();
  CUfunction fn = nullptr;
  int dev = 0;
  Status st = function_on_device(f, &fn, &dev);
  if (st.bad()) return st;
  long long a_n = n, tx = tdims[0], ty = tdims[1], x0 = org[0], y0 = org[1], z0 = org[2], nx = gdims[0],
            ny = gdims[1], it = iters;
  long long b[6];
  for (int i = 0; i < 6; ++i) b[i] = box[i];
  void* args[] = {&data, &a_n, &tx, &ty, &x0, &y0, &z0, &nx, &ny, &it, &b[0], &b[1], &b[2], &b[3], &b[4], &b[5]};
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  const long long blocks = std::min<long long>((n + 255) / 256, (long long)sms * 8);
  if (d.launch(fn, (unsigned)std::max<long long>(1, blocks), 1, 1, 256, 1, 1, 0, static_cast<CUstream>(stream),
               args, nullptr) != CUDA_SUCCESS)
    return make_err(TILE_ECUDA, "cuLaunchKernel (user kernel)");
  return Status::ok();
}

}  // namespace tiles
