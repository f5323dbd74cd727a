// Pinned host memory flavours vs PCIe rate: cudaHostAllocDefault vs
// cudaHostAllocWriteCombined, H2D alone, D2H alone, and both at once (two
// streams), 1 GiB copies, best of 5. Probe for the host tile store's flags.
#include <cstdio>
#include <cstring>
#include <cuda_runtime.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s: %s\n", #x, cudaGetErrorString(e)); return 1; } } while (0)
int main() {
  const size_t B = 1ull << 30;
  void *d1, *d2;
  CK(cudaMalloc(&d1, B)); CK(cudaMalloc(&d2, B));
  cudaStream_t s1, s2; CK(cudaStreamCreate(&s1)); CK(cudaStreamCreate(&s2));
  cudaEvent_t a, b, c; cudaEventCreate(&a); cudaEventCreate(&b); cudaEventCreate(&c);
  for (unsigned flags : {cudaHostAllocDefault, cudaHostAllocWriteCombined, cudaHostAllocPortable}) {
    void *h1, *h2;
    CK(cudaHostAlloc(&h1, B, flags)); CK(cudaHostAlloc(&h2, B, flags));
    memset(h1, 1, B); memset(h2, 2, B);
    float best[3] = {1e9, 1e9, 1e9};
    for (int r = 0; r < 6; ++r) {
      float ms;
      cudaEventRecord(a, s1); cudaMemcpyAsync(d1, h1, B, cudaMemcpyHostToDevice, s1); cudaEventRecord(b, s1);
      cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b); if (r) best[0] = ms < best[0] ? ms : best[0];
      cudaEventRecord(a, s1); cudaMemcpyAsync(h2, d2, B, cudaMemcpyDeviceToHost, s1); cudaEventRecord(b, s1);
      cudaEventSynchronize(b); cudaEventElapsedTime(&ms, a, b); if (r) best[1] = ms < best[1] ? ms : best[1];
      cudaDeviceSynchronize();
      cudaEventRecord(a, 0);
      cudaStreamWaitEvent(s1, a, 0); cudaStreamWaitEvent(s2, a, 0);
      cudaMemcpyAsync(d1, h1, B, cudaMemcpyHostToDevice, s1);
      cudaMemcpyAsync(h2, d2, B, cudaMemcpyDeviceToHost, s2);
      cudaEventRecord(b, s1); cudaEventRecord(c, s2);
      cudaEventSynchronize(b); cudaEventSynchronize(c);
      float m1, m2; cudaEventElapsedTime(&m1, a, b); cudaEventElapsedTime(&m2, a, c);
      ms = m1 > m2 ? m1 : m2; if (r) best[2] = ms < best[2] ? ms : best[2];
    }
    printf("flags %u: H2D %.1f GB/s  D2H %.1f GB/s  bidir %.1f GB/s\n", flags, B / best[0] / 1e6, B / best[1] / 1e6,
           2 * B / best[2] / 1e6);
    cudaFreeHost(h1); cudaFreeHost(h2);
  }
  return 0;
}
