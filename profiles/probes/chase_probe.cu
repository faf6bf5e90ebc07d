// Dependent-load latency probe (diagnostic for wg_dsm_chase): one thread chases a pointer chain of
// 64 B-strided slots through a pre-touched span, with volatile (ld.volatile) and .cg loads.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__global__ void init(unsigned long long* p, unsigned long long n) {
  for (unsigned long long i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    p[i * 8] = (i * 0x9E3779B97F4A7C15ull) ^ 0x5555;
}
template <int MODE>
__global__ void chase(const unsigned long long* p, unsigned long long n, long long acc_n, unsigned long long* sink) {
  unsigned long long x = 0x243F6A8885A308D3ull, acc = 0;
  for (long long i = 0; i < acc_n; ++i) {
    const unsigned long long slot = __umul64hi(x, n);
    unsigned long long v;
    if (MODE == 0) v = *reinterpret_cast<const volatile unsigned long long*>(p + slot * 8);
    else v = __ldcg(p + slot * 8);
    acc += v;
    x = (v + (unsigned long long)i) * 0x9E3779B97F4A7C15ull;
  }
  *sink = acc;
}
int main() {
  const size_t maxb = 4ull << 30;
  unsigned long long *p, *sink;
  cudaMalloc(&p, maxb);
  cudaMalloc(&sink, 8);
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  size_t spans[] = {1 << 20, 4 << 20, 16 << 20, 64 << 20, 256 << 20, 1ull << 30, 4ull << 30};
  for (size_t sp : spans) {
    unsigned long long n = sp / 64;
    init<<<1184, 256>>>(p, n);
    for (int mode = 0; mode < 2; ++mode) {
      for (int rep = 0; rep < 2; ++rep) {
        const long long N = 50000;
        cudaEventRecord(a);
        if (mode == 0) chase<0><<<1, 1>>>(p, n, N, sink); else chase<1><<<1, 1>>>(p, n, N, sink);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (rep == 1) printf("span %8zu KB  %s  %.1f ns/access\n", sp >> 10, mode ? "ld.cg      " : "ld.volatile", ms * 1e6 / N);
      }
    }
  }
  return 0;
}
