// device_util.cuh -- device helpers of the CUDA path: Philox, warp/block scans,
// look-back status format, last-block cleanup, cache-hinted vector loads, fast division.
#pragma once

#include <cuda_runtime.h>
#include <stdint.h>

#if defined(WG_KTIMING) && WG_KTIMING
#include <cstdio>
#endif

namespace wg {

constexpr unsigned FULL_MASK = 0xffffffffu;

// Programmatic dependent launch: wait for the previous kernel of the stream (no-op when
// the kernel was launched without the PDL attribute), then let the next one start.
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" :::); }
__device__ __forceinline__ void pdl_enter() {
  pdl_wait();
  pdl_trigger();
}

// Philox4x32-10 (Salmon et al. SC'11), the counter-based generator of reading A3.
__device__ __forceinline__ uint4 philox4x32_10(uint4 c, uint2 k) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    if (r) {
      k.x += 0x9E3779B9u;
      k.y += 0xBB67AE85u;
    }
    const unsigned hi0 = __umulhi(0xD2511F53u, c.x), lo0 = 0xD2511F53u * c.x;
    const unsigned hi1 = __umulhi(0xCD9E8D57u, c.z), lo1 = 0xCD9E8D57u * c.z;
    c = make_uint4(hi1 ^ c.y ^ k.x, lo1, hi0 ^ c.w ^ k.y, lo0);
  }
  return c;
}

__device__ __forceinline__ unsigned long long ld_volatile_u64(const unsigned long long* p) {
  return *reinterpret_cast<const volatile unsigned long long*>(p);
}
__device__ __forceinline__ void st_volatile_u64(unsigned long long* p, unsigned long long v) {
  *reinterpret_cast<volatile unsigned long long*>(p) = v;
}

// 16-byte read-only load that does not allocate in L1 (each feature byte is read once).
__device__ __forceinline__ uint4 ld_nc_na_v4(const void* p) {
  uint4 r;
  asm("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
      : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
      : "l"(p));
  return r;
}
__device__ __forceinline__ unsigned ld_nc_na_u32(const void* p) {
  unsigned r;
  asm("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(r) : "l"(p));
  return r;
}
__device__ __forceinline__ unsigned short ld_nc_na_u16(const void* p) {
  unsigned short r;
  asm("ld.global.nc.L1::no_allocate.u16 %0, [%1];" : "=h"(r) : "l"(p));
  return r;
}

template <typename T>
__device__ __forceinline__ T warp_inclusive_sum(T v, int lane) {
#pragma unroll
  for (int d = 1; d < 32; d <<= 1) {
    T o = __shfl_up_sync(FULL_MASK, v, d);
    if (lane >= d) v += o;
  }
  return v;
}

template <typename T>
__device__ __forceinline__ T warp_sum(T v) {
#pragma unroll
  for (int d = 16; d > 0; d >>= 1) v += __shfl_xor_sync(FULL_MASK, v, d);
  return v;
}

// Block-wide exclusive sum for NT threads (NT multiple of 32, <= 1024).
// warp_tot must have room for NT/32 values.  Returns the exclusive prefix;
// *total receives the block aggregate (in every thread).
template <int NT, typename T>
__device__ __forceinline__ T block_exclusive_sum(T v, T* warp_tot, T* total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  T inc = warp_inclusive_sum(v, lane);
  if (lane == 31) warp_tot[warp] = inc;
  __syncthreads();
  if (warp == 0) {
    T w = lane < NT / 32 ? warp_tot[lane] : T(0);
    T wi = warp_inclusive_sum(w, lane);
    if (lane < NT / 32) warp_tot[lane] = wi - w;  // exclusive warp offsets
    if (lane == NT / 32 - 1) warp_tot[NT / 32] = wi;
  }
  __syncthreads();
  *total = warp_tot[NT / 32];
  return warp_tot[warp] + inc - v;
}

// ---------------------------------------------------------------- decoupled look-back
// Tile status word: bits 63..62 = flag (0 none, 1 aggregate, 2 inclusive prefix),
// bits 61..0 = value.  Flag and value share one 64-bit word, so publication needs
// no fence.  The block-wide look-back itself is in scan.cuh.
constexpr unsigned long long LB_AGG = 1ull << 62, LB_PRE = 2ull << 62, LB_VAL = (1ull << 62) - 1;

// Last-block cleanup: every block calls this once at its very end (all threads).
// Returns true (in every thread of the block) for the block that finished last;
// by then no other block of this launch reads the look-back status any more.
__device__ __forceinline__ bool finish_block(unsigned* done, int* smem_flag) {
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const unsigned prev = atomicAdd(done, 1u);
    *smem_flag = (prev == gridDim.x - 1);
  }
  __syncthreads();
  return *smem_flag != 0;
}

__device__ __forceinline__ void latch_error(unsigned* ctrl_err, unsigned bits) { atomicOr(ctrl_err, bits); }

__device__ __forceinline__ unsigned long long fmix64(unsigned long long k) {
  k ^= k >> 33;
  k *= 0xff51afd7ed558ccdull;
  k ^= k >> 33;
  k *= 0xc4ceb9fe1a85ec53ull;
  k ^= k >> 33;
  return k;
}

// n / d for any 32-bit n via multiply-high (round-up multiplier, Granlund-Montgomery; d >= 1).
struct FastDiv {
  unsigned d, mul, shift;
  __host__ __device__ FastDiv() : d(1), mul(0), shift(0) {}
  __host__ explicit FastDiv(unsigned d_) : d(d_) {
    shift = 0;
    while ((1u << shift) < d) ++shift;
    unsigned long long m = ((1ull << (32 + shift)) + d - 1) / d;
    mul = (unsigned)m;  // the implicit bit 2^32 is added back in div()
    if (d == 1) { mul = 0; shift = 0; }
  }
  __device__ __forceinline__ unsigned div(unsigned n) const {
    if (d == 1) return n;
    // q = floor((n * (2^32 + mul)) / 2^(32+shift)) computed without overflow
    const unsigned t = __umulhi(n, mul);
    return (unsigned)(((unsigned long long)t + n) >> shift);
  }
};

// ---------------------------------------------------------------- diagnostics (WG_KTIMING=1 builds only)
// Per-block globaltimer marks of the hot kernels; the last block of a large launch prints when its blocks
// started and ended (10-bin histograms over the launch's span).  profiles/probes/ktiming.py.
#ifndef WG_KTIMING
#define WG_KTIMING 0
#endif
#if WG_KTIMING
static __device__ unsigned long long g_kt[4][16384][2];
static __device__ unsigned g_kt_done[4];
static __device__ __forceinline__ unsigned long long kt_now() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
static __device__ __forceinline__ void kt_begin(int k) {
  if (threadIdx.x == 0 && blockIdx.x < 16384) g_kt[k][blockIdx.x][0] = kt_now();
}
static __device__ __noinline__ void kt_end(int k, const char* name, int64_t work) {
  __syncthreads();
  if (threadIdx.x != 0 || blockIdx.x >= 16384) return;
  g_kt[k][blockIdx.x][1] = kt_now();
  __threadfence();
  if (atomicAdd(&g_kt_done[k], 1u) != gridDim.x - 1) return;
  g_kt_done[k] = 0;
  const unsigned nb = gridDim.x < 16384 ? gridDim.x : 16384;
  if (nb < 256) return;
  unsigned long long t0 = ~0ull, t1 = 0;
  for (unsigned b = 0; b < nb; ++b) {
    t0 = min(t0, g_kt[k][b][0]);
    t1 = max(t1, g_kt[k][b][1]);
  }
  const unsigned long long span = t1 - t0 + 1;
  unsigned hs[10] = {0}, he[10] = {0};
  unsigned long long dsum = 0, dmax = 0;
  for (unsigned b = 0; b < nb; ++b) {
    hs[min(9ull, (g_kt[k][b][0] - t0) * 10 / span)]++;
    he[min(9ull, (g_kt[k][b][1] - t0) * 10 / span)]++;
    const unsigned long long d = g_kt[k][b][1] - g_kt[k][b][0];
    dsum += d;
    dmax = max(dmax, d);
  }
  printf("KT %s blocks %u work %lld span %llu ns | block mean %llu max %llu | start %u %u %u %u %u %u %u %u %u %u | end %u %u %u %u %u %u %u %u %u %u\n",
         name, nb, (long long)work, span, dsum / nb, dmax, hs[0], hs[1], hs[2], hs[3], hs[4], hs[5], hs[6], hs[7], hs[8],
         hs[9], he[0], he[1], he[2], he[3], he[4], he[5], he[6], he[7], he[8], he[9]);
}
#define KT_BEGIN(k) kt_begin(k)
#define KT_END(k, name, work) kt_end(k, name, work)
#else
#define KT_BEGIN(k)
#define KT_END(k, name, work)
#endif

}  // namespace wg
