/* synth/splitmix.c — C twin of synth/splitmix.py (counter-based splitmix64
 * input generator; no arithmetic of the method). OpenMP over z-planes. */
#include <stdint.h>

static inline uint64_t splitmix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

static inline int64_t wrap(int64_t i, int64_t n) { i %= n; return i < 0 ? i + n : i; }

void synth_fill_uniform(double* out, int64_t nx, int64_t ny, int64_t nz,
                        int64_t z0, int64_t bz, int64_t y0, int64_t by,
                        int64_t x0, int64_t bx, uint64_t seed) {
  const uint64_t key0 = seed * 0x9E3779B97F4A7C15ull;
#pragma omp parallel for schedule(static)
  for (int64_t k = 0; k < bz * by; ++k) {
    int64_t zz = wrap(z0 + k / by, nz), yy = wrap(y0 + k % by, ny);
    double* row = out + k * bx;
    uint64_t base = ((uint64_t)zz * (uint64_t)ny + (uint64_t)yy) * (uint64_t)nx;
    for (int64_t i = 0; i < bx; ++i) {
      uint64_t g = base + (uint64_t)wrap(x0 + i, nx);
      row[i] = (double)(splitmix64(g + key0) >> 11) * 0x1.0p-53;
    }
  }
}
