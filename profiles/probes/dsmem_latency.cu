// Probe: dependent-load latency of distributed shared memory (cluster of 16 x 512 threads, like
// hop_small_kernel): ld.shared::cluster chains to the own block and to another block, and CAS chains.
#include <cooperative_groups.h>
#include <cstdio>
namespace cg = cooperative_groups;
__device__ unsigned dsm_addr(const void* p, unsigned r) {
  unsigned o; asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(o) : "r"((unsigned)__cvta_generic_to_shared(p)), "r"(r)); return o; }
__global__ void k(unsigned long long* out, int remote, int mode, int nthreads_active) {
  __shared__ unsigned tab[4096];
  cg::cluster_group cl = cg::this_cluster();
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) tab[i] = (i * 2654435761u + 12345u) & 4095u;
  cl.sync();
  const unsigned me = cl.block_rank();
  const unsigned tgt = remote ? (me + 1) % cl.num_blocks() : me;
  unsigned idx = threadIdx.x & 4095;
  unsigned base = dsm_addr(&tab[0], tgt);
  long long t0 = clock64();
  if ((int)threadIdx.x < nthreads_active) {
    for (int it = 0; it < 64; ++it) {
      unsigned v;
      if (mode == 0) {
        asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(base + idx * 4) : "memory");
      } else {
        asm volatile("atom.shared::cluster.cas.b32 %0, [%1], %2, %3;" : "=r"(v) : "r"(base + idx * 4), "r"(0xffffffffu), "r"(0u) : "memory");
      }
      idx = v & 4095;
    }
  }
  long long t1 = clock64();
  cl.sync();
  if (threadIdx.x == 0 && me == 0) { out[0] = (t1 - t0) / 64; out[1] = idx; }
}
int main() {
  unsigned long long* d; cudaMalloc(&d, 64);
  cudaFuncSetAttribute(k, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
  for (int mode = 0; mode < 2; ++mode)
    for (int remote = 0; remote < 2; ++remote)
      for (int act : {1, 32, 512}) {
        cudaLaunchConfig_t cfg = {};
        cfg.gridDim = dim3(16); cfg.blockDim = dim3(512);
        cudaLaunchAttribute at[1]; at[0].id = cudaLaunchAttributeClusterDimension;
        at[0].val.clusterDim.x = 16; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
        cfg.attrs = at; cfg.numAttrs = 1;
        cudaLaunchKernelEx(&cfg, k, d, remote, mode, act);
        unsigned long long h[2]; cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
        printf("%s %s threads %d: %llu cycles per dependent op (%s)\n", mode ? "cas" : "ld", remote ? "remote" : "own",
               act, h[0], cudaGetErrorString(cudaGetLastError()));
      }
}
