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
#define V32_UNROLL 4  // 32 B loads in flight per thread (A/B: 2 was slower, 0.88 vs 0.93 for 512 B rows)
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
  int st_hint;  // X stores: 0 default, 1 L2 evict_first policy, 2 .cs (streaming) (WG_GATHER_ST_HINT)
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

__device__ __forceinline__ void st_out_hint(u32x8* p, const u32x8& r, int hint, unsigned long long pol) {
  if (hint == 1)
    asm volatile("st.global.L2::cache_hint.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8}, %9;" ::"l"(p), "r"(r.v[0]),
                 "r"(r.v[1]), "r"(r.v[2]), "r"(r.v[3]), "r"(r.v[4]), "r"(r.v[5]), "r"(r.v[6]), "r"(r.v[7]), "l"(pol)
                 : "memory");
  else
    asm volatile("st.global.cs.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(p), "r"(r.v[0]), "r"(r.v[1]),
                 "r"(r.v[2]), "r"(r.v[3]), "r"(r.v[4]), "r"(r.v[5]), "r"(r.v[6]), "r"(r.v[7])
                 : "memory");
}

// MINB: resident blocks per SM the register allocation must allow -- GATHER_MINB for a gather that
// fills the GPU alone; GATHER_LEAN_MINB (fewer registers, a few spills) for throughput-mode gathers
// capped at a block or two per SM, whose register file the other streams' hop kernels then use.
template <typename V, int GATHER_UNROLL, int MINB = GATHER_MINB>
__global__ void __launch_bounds__(GATHER_THREADS, MINB) gather_kernel(const GatherArgs a) {
  pdl_enter();
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
  V* __restrict__ out = reinterpret_cast<V*>(a.out + begin * (int64_t)cpr * (int64_t)sizeof(V));
  const unsigned long long pol = l2_evict_last_policy();
  unsigned long long stp;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(stp));
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
    for (int j = 0; j < GATHER_UNROLL; ++j)
      if (dst[j] < total) {
        if constexpr (sizeof(V) == 32) {
          if (a.st_hint) {
            st_out_hint(reinterpret_cast<u32x8*>(&out[dst[j]]), *reinterpret_cast<const u32x8*>(&val[j]), a.st_hint, stp);
            continue;
          }
        }
        st_out<V>(&out[dst[j]], val[j]);
      }
  }
}

// ---------------------------------------------------------------------------- cp.async variant
// The same flat 16 B chunk stream as gather_kernel<uint4>, but every thread's loads are
// cp.async (LDGSTS) copies into shared memory: ASYNC_STAGES stages of ASYNC_K chunks per thread
// are in flight, and a thread stores a stage (ld.shared -> st.global, coalesced) once its own
// copies have landed (cp.async.wait_group; each thread reads back only what it copied, so no
// block barrier is needed).  The bytes in flight live in shared memory instead of registers
// (64 KB per 256-thread block), so the kernel needs few registers and leaves the register file
// to the hop kernels of concurrent batches.  Chunks past a row (pitched output) or of an
// invalid id are zero-filled by the copy itself (src-size 0).
constexpr int ASYNC_THREADS = 256;
constexpr int ASYNC_STAGES = 4;
constexpr int ASYNC_K = 4;
constexpr int ASYNC_SMEM = ASYNC_STAGES * ASYNC_K * ASYNC_THREADS * 16;

__device__ __forceinline__ void cp_async16(void* sdst, const void* gsrc, unsigned src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"((unsigned)__cvta_generic_to_shared(sdst)),
               "l"(gsrc), "r"(src_bytes)
               : "memory");
}
__device__ __forceinline__ void cp_async_wait(int pending) {
  switch (pending) {  // wait_group takes an immediate
    case 0: asm volatile("cp.async.wait_group 0;" ::: "memory"); break;
    case 1: asm volatile("cp.async.wait_group 1;" ::: "memory"); break;
    case 2: asm volatile("cp.async.wait_group 2;" ::: "memory"); break;
    default: asm volatile("cp.async.wait_group 3;" ::: "memory"); break;
  }
}

__global__ void __launch_bounds__(ASYNC_THREADS) gather_async_kernel(const GatherArgs a) {
  pdl_enter();
  extern __shared__ __align__(16) uint4 sbuf[];  // [ASYNC_STAGES][ASYNC_K][ASYNC_THREADS]
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
  const unsigned total = (unsigned)(n * cpr);
  uint4* __restrict__ out = reinterpret_cast<uint4*>(a.out + begin * (int64_t)cpr * 16);
  const unsigned per_stage = ASYNC_THREADS * ASYNC_K;
  const unsigned gstride = gridDim.x * per_stage;
  const unsigned first = blockIdx.x * per_stage;
  const unsigned tid = threadIdx.x;
  const unsigned row_bytes = (unsigned)(a.s.tail_pitch ? a.s.body_bytes + a.s.tail_pitch : a.s.body_bytes);

  auto issue = [&](unsigned base, int slot) {
#pragma unroll
    for (int k = 0; k < ASYNC_K; ++k) {
      const unsigned c = base + (unsigned)k * ASYNC_THREADS + tid;
      if (c < total) {
        const unsigned row = a.cpr.div(c);
        const unsigned boff = (c - row * cpr) * 16u;
        const int64_t v = ids[row];
        const void* src = a.s.feat[0];
        unsigned bytes = 0;
        if (v >= 0 && v < a.s.n) {
          int o;
          int64_t l;
          owner_local(a.s, v, o, l);
          if (a.s.tail_pitch == 0 || boff < (unsigned)a.s.body_bytes) {
            src = a.s.feat[o] + l * a.s.feat_stride + boff;
            bytes = 16;  // whole layout: a pitched chunk may cover the shard row's padding
          } else if (boff < row_bytes) {
            src = a.s.tail[o] + l * a.s.tail_pitch + (boff - (unsigned)a.s.body_bytes);
            bytes = 16;
          }  // else: output padding past a split row -> zeros
        } else if (boff == 0) {
          latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
        }
        cp_async16(&sbuf[((size_t)slot * ASYNC_K + k) * ASYNC_THREADS + tid], src, bytes);
      }
    }
    asm volatile("cp.async.commit_group;" ::: "memory");
  };

  unsigned next = first;
  int issued = 0, done = 0;
  while (issued < ASYNC_STAGES && next < total) {
    issue(next, issued % ASYNC_STAGES);
    next += gstride;
    ++issued;
  }
  while (done < issued) {
    cp_async_wait(issued - done - 1);  // this thread's copies of stage `done` have landed
    const int slot = done % ASYNC_STAGES;
    const unsigned base = first + (unsigned)done * gstride;
#pragma unroll
    for (int k = 0; k < ASYNC_K; ++k) {
      const unsigned c = base + (unsigned)k * ASYNC_THREADS + tid;
      if (c < total) out[c] = sbuf[((size_t)slot * ASYNC_K + k) * ASYNC_THREADS + tid];
    }
    ++done;
    if (next < total) {  // refill the slot just drained
      issue(next, slot);
      next += gstride;
      ++issued;
    }
  }
}

// ---------------------------------------------------------------------------- TMA variant
// One warp per block; the warp owns TMA_STAGES shared-memory stages of R rows at the output pitch.
// For each tile of R consecutive output rows, lane r issues the bulk copies (cp.async.bulk, the TMA
// engine: no registers hold the bytes in flight) of row r from the owner shard into the stage -- one
// copy for a whole row, or body + tail for the split layout -- all signalling one mbarrier with
// complete_tx; when the stage is full, lane 0 writes the whole tile (R * pitch contiguous bytes of X)
// with ONE bulk smem->global store.  TMA_STAGES tiles are in flight per warp.  The bytes in flight
// live in shared memory, so the kernel leaves the register file and the warp slots to kernels of other
// streams (concurrent batches).  Requires row_bytes, body/tail sizes and the pitch to be multiples of 16.
constexpr int TMA_STAGES = 4;
constexpr int TMA_STAGE_BYTES = 16 * 1024;

__device__ __forceinline__ unsigned smem_u32(const void* p) {
  return (unsigned)__cvta_generic_to_shared(p);
}

__device__ __forceinline__ void bulk_g2s(uint8_t* dst, const uint8_t* src, unsigned bytes, unsigned long long* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

__global__ void __launch_bounds__(32) gather_tma_kernel(const GatherArgs a, int rows_per_tile, int row_bytes,
                                                        int pitch) {
  pdl_enter();
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ __align__(8) unsigned long long mbar[TMA_STAGES];
  const int lane = threadIdx.x;
  int64_t n = a.cap;
  if (a.d_n) {
    n = *a.d_n;
    if (n > a.cap || n < 0) {
      if (lane == 0 && blockIdx.x == 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
      n = n < 0 ? 0 : a.cap;
    }
  }
  int64_t begin = a.d_begin ? *a.d_begin : 0;
  begin = begin < 0 ? 0 : (begin > n ? n : begin);
  const int64_t* ids = a.ids + begin;
  uint8_t* outp = a.out + begin * (int64_t)pitch;
  n -= begin;
  const int R = rows_per_tile;
  const int64_t ntiles = (n + R - 1) / R;
  const bool split = a.s.tail_pitch != 0;
  const unsigned body = split ? (unsigned)a.s.body_bytes : (unsigned)row_bytes;
  const unsigned tail = (unsigned)row_bytes - body;
  if (lane == 0) {
    for (int s = 0; s < TMA_STAGES; ++s)
      asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(smem_u32(&mbar[s])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (pitch > row_bytes)  // the bulk copies never write a row's padding: zero it once per stage
    for (int s = 0; s < TMA_STAGES; ++s)
      for (int r = lane; r < R; r += 32)
        for (int c = row_bytes; c < pitch; c += 16)
          *reinterpret_cast<uint4*>(smem + ((size_t)s * R + r) * pitch + c) = make_uint4(0, 0, 0, 0);
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  __syncwarp();

  auto issue = [&](int64_t tile, int s) {
    const int64_t r0 = tile * R;
    const int rows = (int)min((int64_t)R, n - r0);
    uint8_t* stage = smem + (size_t)s * R * pitch;
    bool ok = false;
    int o = 0;
    int64_t l = 0;
    if (lane < rows) {
      const int64_t v = ids[r0 + lane];
      if (v >= 0 && v < a.s.n) {
        owner_local(a.s, v, o, l);
        ok = true;
      } else {
        latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
        uint4* z = reinterpret_cast<uint4*>(stage + (size_t)lane * pitch);
        for (int c = 0; c < row_bytes / 16; ++c) z[c] = make_uint4(0, 0, 0, 0);
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // zero row visible to the bulk store
      }
    }
    const unsigned nvalid = __popc(__ballot_sync(FULL_MASK, ok));
    if (lane == 0)
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(&mbar[s])),
                   "r"(nvalid * (unsigned)row_bytes)
                   : "memory");
    __syncwarp();
    if (ok) {
      uint8_t* dst = stage + (size_t)lane * pitch;
      bulk_g2s(dst, a.s.feat[o] + l * a.s.feat_stride, body, &mbar[s]);
      if (split) bulk_g2s(dst + body, a.s.tail[o] + l * a.s.tail_pitch, tail, &mbar[s]);
    }
  };

  int64_t k = 0;
  for (int s = 0; s < TMA_STAGES; ++s) {
    const int64_t t = blockIdx.x + (int64_t)s * gridDim.x;
    if (t < ntiles) issue(t, s);
  }
  for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x, ++k) {
    const int s = (int)(k % TMA_STAGES);
    const unsigned phase = (unsigned)((k / TMA_STAGES) & 1);
    asm volatile(
        "{\n .reg .pred p;\n WAIT_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra WAIT_%=;\n }" ::
            "r"(smem_u32(&mbar[s])),
        "r"(phase)
        : "memory");
    const int64_t r0 = t * R;
    const int rows = (int)min((int64_t)R, n - r0);
    uint8_t* stage = smem + (size_t)s * R * pitch;
    if (lane == 0) {
      asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(outp + r0 * pitch),
                   "r"(smem_u32(stage)), "r"((unsigned)(rows * pitch))
                   : "memory");
      asm volatile("cp.async.bulk.commit_group;" ::: "memory");
      asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");  // stage may be refilled
    }
    __syncwarp();
    const int64_t tn = t + (int64_t)TMA_STAGES * gridDim.x;
    if (tn < ntiles) issue(tn, s);
  }
  if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

cudaError_t launch_gather(wg_dsm* h, const int64_t* ids, int64_t cap, const int64_t* d_n, const int64_t* d_begin,
                          void* out, int64_t out_pitch, cudaStream_t st) {
  const int64_t rb = h->row_bytes;
  static int knobs = 0, bps = 0, use_tma = 0, allow32 = 1, use_async = 0, use_g4 = 0;
  if (!knobs) {  // A/B knobs, read once: WG_GATHER_BPS (blocks per SM), WG_GATHER_TMA=1, WG_GATHER_V32=0,
                 // WG_GATHER_ASYNC=1 (cp.async variant)
    const char* g4 = getenv("WG_GATHER_G4");
    use_g4 = (g4 && g4[0] == '1') ? 1 : 0;
    const char* ca = getenv("WG_GATHER_ASYNC");
    use_async = (ca && ca[0] == '1') ? 1 : 0;
    const char* b = getenv("WG_GATHER_BPS");
    bps = b ? atoi(b) : 0;
    const char* t = getenv("WG_GATHER_TMA");
    use_tma = (t && t[0] == '1') ? 1 : 0;
    const char* v = getenv("WG_GATHER_V32");
    allow32 = (v && v[0] == '0') ? 0 : 1;
    knobs = 1;
  }
  const uintptr_t oa = (uintptr_t)out;
  // copy width per row: the row, or -- for a pitched output (out_pitch > row_bytes, <= the shard's
  // row pitch) -- the whole output pitch including padding, so 400 B rows can move as 13 x 32 B
  const int64_t cw = out_pitch > rb ? out_pitch : rb;
  const int vb = (allow32 && cw % 32 == 0 && oa % 32 == 0) ? 32
                 : (cw % 16 == 0 && oa % 16 == 0)           ? 16
                 : (cw % 4 == 0 && oa % 4 == 0)             ? 4
                                                            : 2;
  static int st_hint = -1;
  if (st_hint < 0) {
    const char* e = getenv("WG_GATHER_ST_HINT");
    st_hint = e ? atoi(e) : 0;
  }
  GatherArgs a{h->view, ids, cap, d_n, d_begin, static_cast<uint8_t*>(out), h->ws.ctrl, FastDiv((unsigned)(cw / vb)),
               st_hint};
  if (use_g4) {
    const cudaError_t e = launch_gather_g4(h, ids, cap, d_n, d_begin, out, cw, st);
    if (e != cudaErrorNotSupported) return e;
  }
  if (use_async && cw % 16 == 0 && oa % 16 == 0) {
    static int async_bps = 0;
    if (!async_bps) {
      cudaFuncSetAttribute(gather_async_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, ASYNC_SMEM);
      int nb = 0;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, gather_async_kernel, ASYNC_THREADS, ASYNC_SMEM);
      async_bps = nb > 0 ? nb : 1;
    }
    GatherArgs a16 = a;
    a16.cpr = FastDiv((unsigned)(cw / 16));
    const int want = bps > 0 ? bps : h->gather_bps;
    const int per_sm = (want > 0 && want < async_bps) ? want : async_bps;
    const int64_t total = cap * (cw / 16);
    int64_t blocks = (total + ASYNC_THREADS * ASYNC_K - 1) / (ASYNC_THREADS * ASYNC_K);
    const int64_t max_blocks = (int64_t)h->sm_count * per_sm;
    blocks = blocks < 1 ? 1 : (blocks > max_blocks ? max_blocks : blocks);
    return launch_pdl_w(&h->tail_window, gather_async_kernel, (unsigned)blocks, ASYNC_THREADS, (size_t)ASYNC_SMEM,
                        st, a16);
  }
  const int64_t body = h->tail_pitch ? h->body_bytes : rb;
  if (use_tma && rb % 16 == 0 && cw % 16 == 0 && body % 16 == 0 && oa % 16 == 0 && cw <= TMA_STAGE_BYTES) {
    const int R = (int)std::min<int64_t>(32, TMA_STAGE_BYTES / cw);
    const int smem = TMA_STAGES * R * (int)cw;
    static int tma_bps = 0;
    if (!tma_bps) {
      cudaFuncSetAttribute(gather_tma_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, TMA_STAGES * TMA_STAGE_BYTES);
      int nb = 0;
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, gather_tma_kernel, 32, TMA_STAGES * TMA_STAGE_BYTES);
      tma_bps = nb > 0 ? nb : 2;
    }
    const int want = bps > 0 ? bps : h->gather_bps;
    const int per_sm = (want > 0 && want < tma_bps) ? want : tma_bps;
    const int64_t tiles = (cap + R - 1) / R;
    int64_t gbk = (int64_t)h->sm_count * per_sm;
    gbk = std::max<int64_t>(1, std::min(gbk, tiles));
    return launch_pdl(gather_tma_kernel, (unsigned)gbk, 32, (size_t)smem, st, a, R, (int)rb, (int)cw);
  }
  // one full wave: resident blocks per SM (occupancy calculator, cached per vector width) x SMs
  static int occ[4] = {0, 0, 0, 0};
  const int which = vb == 32 ? 0 : vb == 16 ? 1 : vb == 4 ? 2 : 3;
  if (!occ[which]) {
    int nb = 0;
    if (vb == 32) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, gather_kernel<u32x8, V32_UNROLL>, GATHER_THREADS, 0);
    else if (vb == 16) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, gather_kernel<uint4, 4>, GATHER_THREADS, 0);
    else if (vb == 4) cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, gather_kernel<unsigned, 4>, GATHER_THREADS, 0);
    else cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, gather_kernel<unsigned short, 4>, GATHER_THREADS, 0);
    occ[which] = nb > 0 ? nb : 4;
  }
  const int want = bps > 0 ? bps : h->gather_bps;  // env knob (A/B) overrides the handle's setting
  const int per_sm = (want > 0 && want < occ[which]) ? want : occ[which];
  const int64_t total = cap * (cw / vb);
  const int unr = vb == 32 ? V32_UNROLL : 4;
  int64_t blocks = (total + GATHER_THREADS * unr - 1) / (GATHER_THREADS * unr);
  const int64_t max_blocks = (int64_t)h->sm_count * per_sm;
  blocks = blocks < 1 ? 1 : (blocks > max_blocks ? max_blocks : blocks);
  const unsigned gb = (unsigned)blocks;
  const cudaAccessPolicyWindow* w = &h->tail_window;  // num_bytes == 0 unless WG_TAIL_PERSIST=2
  static int lean = -1;  // A/B knob WG_GATHER_LEAN=0: the full-occupancy kernel for capped launches too
  if (lean < 0) {
    const char* e = getenv("WG_GATHER_LEAN");
    lean = (e && e[0] == '0') ? 0 : 1;
  }
  if (vb == 32 && lean && per_sm <= 2)
    return launch_pdl_w(w, gather_kernel<u32x8, LEAN_UNROLL, GATHER_LEAN_MINB>, gb, GATHER_THREADS, 0, st, a);
  if (vb == 32) return launch_pdl_w(w, gather_kernel<u32x8, V32_UNROLL>, gb, GATHER_THREADS, 0, st, a);
  if (vb == 16) return launch_pdl_w(w, gather_kernel<uint4, 4>, gb, GATHER_THREADS, 0, st, a);
  if (vb == 4) return launch_pdl_w(w, gather_kernel<unsigned, 4>, gb, GATHER_THREADS, 0, st, a);
  return launch_pdl_w(w, gather_kernel<unsigned short, 4>, gb, GATHER_THREADS, 0, st, a);
}

}  // namespace wg
