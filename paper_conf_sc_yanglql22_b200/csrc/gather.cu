// gather.cu -- global gather over the DSM: "a single gather
// kernel in each GPU"; NVLink/NVSwitch carry the remote reads.
//
// The output X[R][pitch] is treated as a flat stream of 32- or 16-byte chunks; thread
// t copies chunk c -> (row c / cpr, column c % cpr), cpr = pitch / chunk.  Adjacent
// threads therefore read adjacent 16 B pieces of the same source row (full 32 B
// sectors, one row = one contiguous burst from local HBM or a peer) and write fully
// coalesced 128 B lines.  Each thread keeps UNROLL independent 16 B loads in flight
// (ld.global.nc.L1::no_allocate: every byte is read exactly once), so a grid of
// ~8 x 256 threads per SM keeps ~0.5 MB in flight chip-wide -- enough to cover
// local-HBM and NVLink latency.  Rows whose size is not a multiple of 16 use the
// same scheme with 4- or 2-byte chunks.  For the split row layout (dsm.cu feat_geometry) a
// chunk at byte offset >= body_bytes comes from the owner's tail region (L2 evict_last).
#include <algorithm>
#include <cstdlib>

#include "device_util.cuh"
#include "wg_internal.cuh"

namespace wg {

constexpr int GATHER_THREADS = 256;
#ifndef GATHER_MINB
#define GATHER_MINB 5  // resident gather blocks per SM the register allocation must allow
#endif
#ifndef LEAN_UNROLL
#define LEAN_UNROLL 2  // loads in flight per thread of the lean throughput-mode gather
#endif
#ifndef GATHER_LEAN_MINB
#define GATHER_LEAN_MINB 8
#endif
#ifndef V32_UNROLL
#define V32_UNROLL 3  // 32 B loads in flight per thread (A/B on B200: 3 -> 48 registers, no spills: 0.86 vs 0.83 with 4)
#endif

// 32 B vectors (sm_100 LDG/STG.256) for rows that are multiples of 32 B
struct __align__(32) u32x8 {
  unsigned v[8];
};

template <typename V>
__device__ __forceinline__ V ld_feat(const void* p);
template <>
__device__ __forceinline__ u32x8 ld_feat<u32x8>(const void* p) {
  u32x8 r;
  asm("ld.global.nc.L1::no_allocate.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
      : "=r"(r.v[0]), "=r"(r.v[1]), "=r"(r.v[2]), "=r"(r.v[3]), "=r"(r.v[4]), "=r"(r.v[5]), "=r"(r.v[6]),
        "=r"(r.v[7])
      : "l"(p));
  return r;
}
template <>
__device__ __forceinline__ uint4 ld_feat<uint4>(const void* p) { return ld_nc_na_v4(p); }


template <>
__device__ __forceinline__ unsigned ld_feat<unsigned>(const void* p) { return ld_nc_na_u32(p); }
template <>
__device__ __forceinline__ unsigned short ld_feat<unsigned short>(const void* p) { return ld_nc_na_u16(p); }

// L2 policy for tail loads: the split layout's tail region is small and re-read by every batch,
// so it is kept in L2 with evict_last (createpolicy, the sm_80+ L2 cache-hint mechanism).
__device__ __forceinline__ unsigned long long l2_evict_last_policy() {
  unsigned long long p;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint4 ld_tail_v4(const void* p, unsigned long long pol) {
  uint4 r;
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v4.u32 {%0,%1,%2,%3}, [%4], %5;"
      : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
      : "l"(p), "l"(pol));
  return r;
}
__device__ __forceinline__ u32x8 ld_tail_v8(const void* p, unsigned long long pol) {
  u32x8 r;
  asm("ld.global.nc.L1::no_allocate.L2::cache_hint.v8.u32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8], %9;"
      : "=r"(r.v[0]), "=r"(r.v[1]), "=r"(r.v[2]), "=r"(r.v[3]), "=r"(r.v[4]), "=r"(r.v[5]), "=r"(r.v[6]),
        "=r"(r.v[7])
      : "l"(p), "l"(pol));
  return r;
}

// Chunk of `avail` (>= 16, a multiple of 16) tail bytes starting at t, as one vector V; bytes past
// the row (a pitched output's padding) read as zero.
template <typename V>
__device__ __forceinline__ V ld_tail(const uint8_t* t, unsigned avail, unsigned long long pol) {
  return ld_feat<V>(t);
}
template <>
__device__ __forceinline__ uint4 ld_tail<uint4>(const uint8_t* t, unsigned avail, unsigned long long pol) {
  return ld_tail_v4(t, pol);
}
template <>
__device__ __forceinline__ u32x8 ld_tail<u32x8>(const uint8_t* t, unsigned avail, unsigned long long pol) {
  if (avail >= 32 && ((uintptr_t)t & 31u) == 0) return ld_tail_v8(t, pol);
  const uint4 a = ld_tail_v4(t, pol);
  const uint4 b = avail >= 32 ? ld_tail_v4(t + 16, pol) : make_uint4(0, 0, 0, 0);
  u32x8 r;
  r.v[0] = a.x, r.v[1] = a.y, r.v[2] = a.z, r.v[3] = a.w, r.v[4] = b.x, r.v[5] = b.y, r.v[6] = b.z, r.v[7] = b.w;
  return r;
}

// Chunk at byte offset boff of row l on rank o: from the body (feature shard) or, for the split
// layout, from the tail region (boundaries are multiples of 128 B, so no chunk straddles them).
template <typename V>
__device__ __forceinline__ V ld_row_chunk(const ShardView& s, int o, int64_t l, unsigned boff,
                                          unsigned long long pol) {
  if (s.tail_pitch == 0 || boff < (unsigned)s.body_bytes) return ld_feat<V>(s.feat[o] + l * s.feat_stride + boff);
  const unsigned toff = boff - (unsigned)s.body_bytes;
  return ld_tail<V>(s.tail[o] + l * s.tail_pitch + toff, (unsigned)s.tail_pitch - toff, pol);
}

struct GatherArgs {
  ShardView s;
  const int64_t* ids;
  int64_t cap;
  const int64_t* d_n;
  const int64_t* d_begin;  // nullable: first row (rows [begin, n) of ids / out are processed)
  uint8_t* out;
  unsigned* ctrl;
  FastDiv cpr;  // chunks per row
};

template <typename V>
__device__ __forceinline__ void st_out(V* p, const V& v) {
  *p = v;
}
template <>
__device__ __forceinline__ void st_out<u32x8>(u32x8* p, const u32x8& r) {
  asm volatile("st.global.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(r.v[0]), "r"(r.v[1]), "r"(r.v[2]),
               "r"(r.v[3]), "r"(r.v[4]), "r"(r.v[5]), "r"(r.v[6]), "r"(r.v[7])
               : "memory");
}

// DENSE16 (V = u32x8 only): rows of R bytes with R % 32 == 16 (products: 400 B) written DENSELY (pitch R):
// chunk c of a row is still the 32 B source piece [32c, 32c + 32) -- one 32 B load from the body, 16 B
// for the last chunk -- but its destination row * R + 32c is only 16 B aligned, so it is stored as two
// 16 B vectors (one for the last chunk).  Consecutive threads still cover consecutive output bytes, so
// L2 merges the halves into whole sectors: no 16 B pitch padding reaches DRAM.
template <typename V>
__device__ __forceinline__ void st_out_dense16(uint8_t* p, const V& r, bool half);
template <>
__device__ __forceinline__ void st_out_dense16<u32x8>(uint8_t* p, const u32x8& r, bool half) {
  asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p), "r"(r.v[0]), "r"(r.v[1]), "r"(r.v[2]), "r"(r.v[3])
               : "memory");
  if (!half)
    asm volatile("st.global.v4.u32 [%0], {%1,%2,%3,%4};" ::"l"(p + 16), "r"(r.v[4]), "r"(r.v[5]), "r"(r.v[6]),
                 "r"(r.v[7])
                 : "memory");
}

// MINB: resident blocks per SM the register allocation must allow -- GATHER_MINB for a gather that
// fills the GPU alone; GATHER_LEAN_MINB (fewer registers, a few spills) for throughput-mode gathers
// capped at a block or two per SM, whose register file the other streams' hop kernels then use.
template <typename V, int GATHER_UNROLL, int MINB = GATHER_MINB, bool DENSE16 = false>
__global__ void __launch_bounds__(GATHER_THREADS, MINB) gather_kernel(const GatherArgs a) {
  pdl_enter();
  KT_BEGIN(3);
  int64_t n = a.cap;
  if (a.d_n) {
    n = *a.d_n;
    if (n > a.cap || n < 0) {
      if (threadIdx.x == 0 && blockIdx.x == 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
      n = n < 0 ? 0 : a.cap;
    }
  }
  int64_t begin = a.d_begin ? *a.d_begin : 0;
  begin = begin < 0 ? 0 : (begin > n ? n : begin);
  const int64_t* __restrict__ ids = a.ids + begin;
  n -= begin;
  const unsigned cpr = a.cpr.d;
  const unsigned total = (unsigned)(n * cpr);  // < 2^31 (checked on the host)
  const unsigned stride = gridDim.x * GATHER_THREADS;
  // DENSE16: rows of (cpr - 1) * 32 + 16 bytes
  const int64_t out_row = DENSE16 ? (int64_t)cpr * (int64_t)sizeof(V) - 16 : (int64_t)cpr * (int64_t)sizeof(V);
  V* __restrict__ out = reinterpret_cast<V*>(a.out + begin * out_row);
  uint8_t* __restrict__ out8 = a.out + begin * out_row;
  const unsigned long long pol = l2_evict_last_policy();
  for (unsigned c0 = blockIdx.x * GATHER_THREADS + threadIdx.x; c0 < total; c0 += stride * GATHER_UNROLL) {
    V val[GATHER_UNROLL];
    unsigned dst[GATHER_UNROLL];
#pragma unroll
    for (int j = 0; j < GATHER_UNROLL; ++j) {
      const unsigned c = c0 + (unsigned)j * stride;
      dst[j] = c;
      if (c < total) {
        const unsigned row = a.cpr.div(c);
        const unsigned colc = c - row * cpr;
        const int64_t v = ids[row];
        if (v >= 0 && v < a.s.n) {
          int o;
          int64_t l;
          owner_local(a.s, v, o, l);
          val[j] = ld_row_chunk<V>(a.s, o, l, colc * (unsigned)sizeof(V), pol);
        } else {
          if (colc == 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
          val[j] = V{};
        }
      }
    }
#pragma unroll
    for (int j = 0; j < GATHER_UNROLL; ++j) {
      if (dst[j] < total) {
        if (DENSE16) {
          const unsigned row = a.cpr.div(dst[j]);
          const unsigned colc = dst[j] - row * cpr;
          st_out_dense16<V>(out8 + (int64_t)row * out_row + colc * 32u, val[j], colc == cpr - 1);
        } else {
          st_out<V>(&out[dst[j]], val[j]);
        }
      }
    }
  }
  KT_END(3, "gather", n);
}

cudaError_t launch_gather(wg_dsm* h, const int64_t* ids, int64_t cap, const int64_t* d_n, const int64_t* d_begin,
                          void* out, int64_t out_pitch, cudaStream_t st) {
  const int64_t rb = h->row_bytes;
  const uintptr_t oa = (uintptr_t)out;
  // copy width per row: the row, or -- for a pitched output (out_pitch > row_bytes, <= the shard's
  // row pitch) -- the whole output pitch including padding, so 400 B rows can move as 13 x 32 B
  const int64_t cw = out_pitch > rb ? out_pitch : rb;
  // dense rows of 32k + 16 bytes (k >= 1) whose stored body is whole 32 B pieces: 32 B loads, 16 B stores
  const bool dense16 = cw == rb && rb % 32 == 16 && rb >= 48 && oa % 16 == 0 &&
                       (h->tail_pitch == 0 || h->body_bytes % 32 == 0) && (h->feat_stride % 32 == 0) &&
                       (h->tail_pitch == 0 || h->tail_pitch % 16 == 0);
  if (dense16) {
    GatherArgs a{h->view, ids, cap, d_n, d_begin, static_cast<uint8_t*>(out), h->ws.ctrl, FastDiv((unsigned)((rb + 16) / 32))};
    static int occ16 = 0;
    if (!occ16) {
      int nb = 0;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, gather_kernel<u32x8, V32_UNROLL, GATHER_MINB, true>, GATHER_THREADS, 0);
      occ16 = nb > 0 ? nb : 4;
    }
    const int want = h->gather_bps;
    const int per_sm = (want > 0 && want < occ16) ? want : occ16;
    const int64_t total = cap * ((rb + 16) / 32);
    int64_t blocks = (total + GATHER_THREADS * V32_UNROLL - 1) / (GATHER_THREADS * V32_UNROLL);
    const int64_t max_blocks = (int64_t)h->sm_count * per_sm;
    blocks = blocks < 1 ? 1 : (blocks > max_blocks ? max_blocks : blocks);
    if (per_sm <= 2)
      return launch_pdl(gather_kernel<u32x8, LEAN_UNROLL, GATHER_LEAN_MINB, true>, (unsigned)blocks, GATHER_THREADS, 0, st, a);
    return launch_pdl(gather_kernel<u32x8, V32_UNROLL, GATHER_MINB, true>, (unsigned)blocks, GATHER_THREADS, 0, st, a);
  }
  const int vb = (cw % 32 == 0 && oa % 32 == 0)   ? 32
                 : (cw % 16 == 0 && oa % 16 == 0) ? 16
                 : (cw % 4 == 0 && oa % 4 == 0)   ? 4
                                                  : 2;
  GatherArgs a{h->view, ids, cap, d_n, d_begin, static_cast<uint8_t*>(out), h->ws.ctrl, FastDiv((unsigned)(cw / vb))};
  // one full wave: resident blocks per SM (occupancy calculator, cached per vector width) x SMs
  static int occ[4] = {0, 0, 0, 0};
  const int which = vb == 32 ? 0 : vb == 16 ? 1 : vb == 4 ? 2 : 3;
  if (!occ[which]) {
    int nb = 0;
    if (vb == 32) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, gather_kernel<u32x8, V32_UNROLL>, GATHER_THREADS, 0);
    else if (vb == 16) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, gather_kernel<uint4, 4>, GATHER_THREADS, 0);
    else if (vb == 4) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, gather_kernel<unsigned, 4>, GATHER_THREADS, 0);
    else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, gather_kernel<unsigned short, 4>, GATHER_THREADS, 0);
    occ[which] = nb > 0 ? nb : 4;  // same value from every thread: a benign race
  }
  const int want = h->gather_bps;  // wg_dsm_set_gather_occupancy (0 = occupancy maximum)
  const int per_sm = (want > 0 && want < occ[which]) ? want : occ[which];
  const int64_t total = cap * (cw / vb);
  const int unr = vb == 32 ? V32_UNROLL : 4;
  int64_t blocks = (total + GATHER_THREADS * unr - 1) / (GATHER_THREADS * unr);
  const int64_t max_blocks = (int64_t)h->sm_count * per_sm;
  blocks = blocks < 1 ? 1 : (blocks > max_blocks ? max_blocks : blocks);
  const unsigned gb = (unsigned)blocks;
  // gathers capped at <= 2 blocks/SM (several batches in flight per GPU) use the register-lean
  // instantiation: the bytes in flight then come from the concurrent kernels, and the register file
  // stays free for the latency-bound hop kernels of the other streams
  if (vb == 32 && per_sm <= 2) return launch_pdl(gather_kernel<u32x8, LEAN_UNROLL, GATHER_LEAN_MINB>, gb, GATHER_THREADS, 0, st, a);
  if (vb == 32) return launch_pdl(gather_kernel<u32x8, V32_UNROLL>, gb, GATHER_THREADS, 0, st, a);
  if (vb == 16) return launch_pdl(gather_kernel<uint4, 4>, gb, GATHER_THREADS, 0, st, a);
  if (vb == 4) return launch_pdl(gather_kernel<unsigned, 4>, gb, GATHER_THREADS, 0, st, a);
  return launch_pdl(gather_kernel<unsigned short, 4>, gb, GATHER_THREADS, 0, st, a);
}

}  // namespace wg
