// Probe: are 64-bit CAS / min and 32-bit add atomic on distributed shared memory (cluster of 2)?
// All 2 x 256 threads hit words that live in block 0's shared memory.
#include <cooperative_groups.h>
#include <cstdio>
namespace cg = cooperative_groups;
__device__ unsigned dsm_addr(const void* p, unsigned r) {
  unsigned o; asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(o) : "r"((unsigned)__cvta_generic_to_shared(p)), "r"(r)); return o; }
__global__ void __cluster_dims__(2, 1, 1) k(unsigned long long* out) {
  __shared__ unsigned long long w_cas, w_min, g_cas, g_min;
  __shared__ unsigned w_add, w_cas32, w_min32;
  cg::cluster_group cl = cg::this_cluster();
  if (threadIdx.x == 0) { w_cas = 0; w_min = ~0ull; g_cas = 0; g_min = ~0ull; w_add = 0; w_cas32 = 0; w_min32 = ~0u; }
  cl.sync();
  const unsigned t = cl.block_rank() * blockDim.x + threadIdx.x;
  unsigned a_cas = dsm_addr(&w_cas, 0), a_min = dsm_addr(&w_min, 0), a_add = dsm_addr(&w_add, 0);
  unsigned a_c32 = dsm_addr(&w_cas32, 0), a_m32 = dsm_addr(&w_min32, 0);
  for (int it = 0; it < 100; ++it) {
    // 64-bit CAS increment loop (explicit shared::cluster)
    unsigned long long cur, old;
    asm volatile("ld.shared::cluster.u64 %0, [%1];" : "=l"(cur) : "r"(a_cas) : "memory");
    for (;;) {
      asm volatile("atom.shared::cluster.cas.b64 %0, [%1], %2, %3;" : "=l"(old) : "r"(a_cas), "l"(cur), "l"(cur + 1) : "memory");
      if (old == cur) break;
      cur = old;
    }
    unsigned long long v = 1000000ull + (unsigned long long)((t * 7919u + it * 104729u) % 999983u);
    asm volatile("atom.shared::cluster.min.u64 %0, [%1], %2;" : "=l"(old) : "r"(a_min), "l"(v) : "memory");
    asm volatile("red.shared::cluster.add.u32 [%0], %1;" ::"r"(a_add), "r"(1u) : "memory");
    unsigned c32, o32;
    asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(c32) : "r"(a_c32) : "memory");
    for (;;) {
      asm volatile("atom.shared::cluster.cas.b32 %0, [%1], %2, %3;" : "=r"(o32) : "r"(a_c32), "r"(c32), "r"(c32 + 1) : "memory");
      if (o32 == c32) break;
      c32 = o32;
    }
    asm volatile("atom.shared::cluster.min.u32 %0, [%1], %2;" : "=r"(o32) : "r"(a_m32), "r"((unsigned)v) : "memory");
    // generic-pointer variants
    unsigned long long* gp = cl.map_shared_rank(&g_cas, 0);
    unsigned long long gc = *(volatile unsigned long long*)gp;
    for (;;) { unsigned long long o = atomicCAS(gp, gc, gc + 1); if (o == gc) break; gc = o; }
    atomicMin(cl.map_shared_rank(&g_min, 0), v);
  }
  cl.sync();
  if (cl.block_rank() == 0 && threadIdx.x == 0) {
    out[0] = w_cas; out[1] = w_min; out[2] = w_add; out[3] = w_cas32; out[4] = w_min32; out[5] = g_cas; out[6] = g_min;
  }
}
int main() {
  unsigned long long* d; cudaMalloc(&d, 64);
  k<<<2, 256>>>(d);
  unsigned long long h[7]; cudaMemcpy(h, d, 56, cudaMemcpyDeviceToHost);
  unsigned long long mn = ~0ull;
  for (unsigned t = 0; t < 512; ++t) for (int it = 0; it < 100; ++it) { unsigned long long v = 1000000ull + (unsigned long long)((t * 7919u + it * 104729u) % 999983u); if (v < mn) mn = v; }
  printf("expect cas=%d min=%llu add=%d | ptx cas64=%llu min64=%llu add32=%llu cas32=%llu min32=%llu | generic cas64=%llu min64=%llu  err=%s\n",
         512 * 100, mn, 512 * 100, h[0], h[1], h[2], h[3], h[4], h[5], h[6], cudaGetErrorString(cudaGetLastError()));
}
