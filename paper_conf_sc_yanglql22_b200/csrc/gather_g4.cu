// gather_g4.cu -- the global gather with Blackwell TMA row gathers.
//
// cp.async.bulk.tensor.2d...tile::gather4 (sm_100) loads the same column box from FOUR rows of
// a 2-D tensor, given by four row coordinates, into shared memory with one instruction.  Each
// rank's feature shard is described by a tensor map (u32 elements, [n_local][body_bytes/4] at
// row pitch feat_stride; for the split layout a second map covers the tail region), so one
// gather4 moves 4 rows' bodies and one more their tails.  Per tile of 32 output rows a warp
// groups its rows by owner rank (__match_any_sync), packs each group into gather4 ops (the
// last op of a group repeats a row), waits on one mbarrier per stage and copies the staged
// rows to X with coalesced 32 B stores.  The bytes in flight live in shared memory, not in
// registers (A/B switch WG_GATHER_G4=1; rows whose body is > 1 KB, or outputs not pitched to
// 32 B, take the LSU path).
#include <cuda.h>
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdlib>

#include "device_util.cuh"
#include "wg_internal.cuh"

namespace wg {

constexpr int G4_WARPS = 4;   // warps per block, each with its own stages
constexpr int G4_STAGES = 2;  // tiles in flight per warp
constexpr int G4_TILE = 32;   // output rows per tile (one per lane)

struct G4Maps {
  CUtensorMap body[WG_MAX_WORLD];
  CUtensorMap tail[WG_MAX_WORLD];
};

struct G4Args {
  ShardView s;
  const int64_t* ids;
  int64_t cap;
  const int64_t* d_n;
  const int64_t* d_begin;
  uint8_t* out;
  unsigned* ctrl;
  int pitch;       // output row pitch (multiple of 32)
  int body;        // bytes per row loaded through the body map (= one box)
  int tail;        // bytes per row through the tail map (0 = whole rows)
  int slots;       // staged row slots per tile (32 + padding of the owner groups)
};

__device__ __forceinline__ unsigned g4_smem(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }

__device__ __forceinline__ void g4_load(uint8_t* dst, const CUtensorMap* map, int col, int r0, int r1, int r2, int r3,
                                        unsigned long long* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cta.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, "
      "%4, %5, %6}], [%7];" ::"r"(g4_smem(dst)),
      "l"(map), "r"(col), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(g4_smem(bar))
      : "memory");
}

__global__ void __launch_bounds__(G4_WARPS * 32) gather_g4_kernel(const __grid_constant__ G4Args a,
                                                                   const __grid_constant__ G4Maps maps) {
  pdl_enter();
  extern __shared__ __align__(128) uint8_t g4_sm[];
  __shared__ __align__(8) unsigned long long bars[G4_WARPS][G4_STAGES];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
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
  const int64_t* ids = a.ids + begin;
  uint8_t* outp = a.out + begin * (int64_t)a.pitch;
  n -= begin;
  const int rowb = a.body + a.tail;
  // TMA destinations must be 128 B aligned: every op (4 rows) gets a 128 B-aligned region
  const int nops = a.slots / 4;
  const int ob = (4 * a.body + 127) & ~127, ot = (4 * a.tail + 127) & ~127;
  const int stage_bytes = nops * (ob + ot);
  uint8_t* sm_base = g4_sm + ((128u - (g4_smem(g4_sm) & 127u)) & 127u);
  uint8_t* wsm = sm_base + (size_t)warp * G4_STAGES * stage_bytes;
  if (lane == 0) {
    for (int s = 0; s < G4_STAGES; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(g4_smem(&bars[warp][s])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  const int64_t ntiles = (n + G4_TILE - 1) / G4_TILE;
  const int64_t wstride = (int64_t)gridDim.x * G4_WARPS;
  const int64_t w0 = (int64_t)blockIdx.x * G4_WARPS + warp;

  // issue the gather4 ops of tile t into stage s; returns this lane's staged slot (-1: zero row)
  auto issue = [&](int64_t t, int s) -> int {
    const int64_t r = t * G4_TILE + lane;
    int own = -2;  // -2: no row, -1: invalid id
    int64_t l = 0;
    if (r < n) {
      const int64_t v = ids[r];
      if (v >= 0 && v < a.s.n) {
        owner_local(a.s, v, own, l);
      } else {
        own = -1;
        latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
      }
    }
    const bool live = own >= 0;
    const unsigned grp = __match_any_sync(FULL_MASK, live ? own : -1 - lane);  // rows of one owner
    const int leader = __ffs(grp) - 1;
    const int size = __popc(grp);
    const int rank = __popc(grp & ((1u << lane) - 1u));
    // group bases: leaders contribute their size rounded up to 4, exclusive scan over lanes
    int contrib = (live && lane == leader) ? ((size + 3) & ~3) : 0;
    int incl = contrib;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const int y = __shfl_up_sync(FULL_MASK, incl, d);
      if (lane >= d) incl += y;
    }
    const int base = __shfl_sync(FULL_MASK, incl - contrib, leader);
    const int slot = live ? base + rank : -1;
    // lanes of rank 0, 4, 8, ... issue one op for their 4 consecutive group members
    const bool issuer = live && (rank & 3) == 0;
    int rr[4];
    rr[0] = (int)l;
#pragma unroll
    for (int k = 1; k < 4; ++k) {
      const int src = (live && rank + k < size) ? (int)__fns(grp, 0, rank + k + 1) : lane;
      rr[k] = __shfl_sync(FULL_MASK, (int)l, src);
    }
    const unsigned ops = __popc(__ballot_sync(FULL_MASK, issuer));
    unsigned long long* bar = &bars[warp][s];
    if (lane == 0)
      asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(g4_smem(bar)),
                   "r"(ops * 4u * (unsigned)rowb)
                   : "memory");
    __syncwarp();
    if (issuer) {
      uint8_t* st = wsm + (size_t)s * stage_bytes;
      const int op = slot >> 2;
      g4_load(st + (size_t)op * ob, &maps.body[own], 0, rr[0], rr[1], rr[2], rr[3], bar);
      if (a.tail) g4_load(st + (size_t)nops * ob + (size_t)op * ot, &maps.tail[own], 0, rr[0], rr[1], rr[2], rr[3], bar);
    }
    return slot;
  };

  int myslot[G4_STAGES];
  int64_t k = 0;
  for (int s = 0; s < G4_STAGES; ++s) {
    const int64_t t = w0 + (int64_t)s * wstride;
    myslot[s] = t < ntiles ? issue(t, s) : -1;
  }
  const int cpr = a.pitch / 32;
  for (int64_t t = w0; t < ntiles; t += wstride, ++k) {
    const int s = (int)(k % G4_STAGES);
    const unsigned phase = (unsigned)((k / G4_STAGES) & 1);
    unsigned done = 0;
    for (long spin = 0; !done; ++spin) {
      asm volatile(
          "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n }"
          : "=r"(done)
          : "r"(g4_smem(&bars[warp][s])), "r"(phase)
          : "memory");
      if (!done && spin > (1l << 24)) {  // never expected: report instead of hanging
        latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_TMA);
        return;
      }
    }
    const uint8_t* st = wsm + (size_t)s * stage_bytes;
    const int64_t r0 = t * G4_TILE;
    const int rows = (int)min((int64_t)G4_TILE, n - r0);
    uint8_t* orow = outp + r0 * a.pitch;
    // per chunk: the row's slot comes from the lane that owns the row
    const int nchunks = rows * cpr;
    for (int c0 = 0; c0 < nchunks; c0 += 32) {
      const int c = c0 + lane;
      const int row = c < nchunks ? c / cpr : 0;
      const int sl = __shfl_sync(FULL_MASK, myslot[s], row);
      if (c < nchunks) {
        const int col = (c - row * cpr) * 32;
        uint4 lo = make_uint4(0, 0, 0, 0), hi = make_uint4(0, 0, 0, 0);
        if (sl >= 0) {
          if (col < a.body) {
            const uint4* p = reinterpret_cast<const uint4*>(st + (size_t)(sl >> 2) * ob + (sl & 3) * a.body + col);
            lo = p[0];
            hi = p[1];
          } else if (col - a.body < a.tail) {
            const int toff = col - a.body;
            const uint4* p =
                reinterpret_cast<const uint4*>(st + (size_t)nops * ob + (size_t)(sl >> 2) * ot + (sl & 3) * a.tail + toff);
            lo = p[0];
            if (a.tail - toff >= 32) hi = p[1];
          }
        }
        asm volatile("st.global.v8.u32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(orow + (int64_t)row * a.pitch + col),
                     "r"(lo.x), "r"(lo.y), "r"(lo.z), "r"(lo.w), "r"(hi.x), "r"(hi.y), "r"(hi.z), "r"(hi.w)
                     : "memory");
      }
    }
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // our smem reads before the next TMA writes
    __syncwarp();
    const int64_t tn = t + (int64_t)G4_STAGES * wstride;
    if (tn < ntiles) myslot[s] = issue(tn, s);
  }
}

static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPointByVersion("cuTensorMapEncodeTiled", &p, 12000, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
  }
  return fn;
}

static bool encode_rows(CUtensorMap* m, const void* base, int64_t rows, int row_bytes, int64_t pitch) {
  auto fn = encode_fn();
  if (!fn || rows < 1) return false;
  cuuint64_t dims[2] = {(cuuint64_t)(row_bytes / 4), (cuuint64_t)rows};
  cuuint64_t strides[1] = {(cuuint64_t)pitch};
  cuuint32_t box[2] = {(cuuint32_t)(row_bytes / 4), 1};
  cuuint32_t estr[2] = {1, 1};
  return fn(m, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, const_cast<void*>(base), dims, strides, box, estr,
            CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE,
            CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

// Returns cudaErrorNotSupported when this gather does not fit the gather4 path (caller falls back).
cudaError_t launch_gather_g4(wg_dsm* h, const int64_t* ids, int64_t cap, const int64_t* d_n, const int64_t* d_begin,
                             void* out, int64_t cw, cudaStream_t st) {
  const int64_t body = h->tail_pitch ? h->body_bytes : h->row_bytes;
  const int64_t tail = h->tail_pitch ? h->row_bytes - h->body_bytes : 0;
  if (cw % 32 != 0 || ((uintptr_t)out & 31) || body % 16 || tail % 16 || body > 1024 || body < 16 ||
      h->feat_stride % 16 || (tail && h->tail_pitch != tail))
    return cudaErrorNotSupported;
  thread_local G4Maps maps;  // per host thread (virtual ranks), rebuilt when the shards change
  thread_local const void* built_for = nullptr;
  if (built_for != h->view.feat[0]) {
    for (int r = 0; r < h->world; ++r) {
      if (!encode_rows(&maps.body[r], h->view.feat[r], std::max<int64_t>(1, h->n_local_of[r]), (int)body,
                       h->feat_stride))
        return cudaErrorNotSupported;
      if (tail && !encode_rows(&maps.tail[r], h->view.tail[r], std::max<int64_t>(1, h->n_local_of[r]), (int)tail,
                               h->tail_pitch))
        return cudaErrorNotSupported;
    }
    built_for = h->view.feat[0];
  }
  G4Args a{h->view, ids, cap, d_n, d_begin, static_cast<uint8_t*>(out), h->ws.ctrl, (int)cw, (int)body, (int)tail, 0};
  a.slots = G4_TILE + (h->world > 1 ? 4 * h->world : 0);
  const size_t ob = (4 * body + 127) & ~127, ot = (4 * tail + 127) & ~127;
  const size_t smem = (size_t)G4_WARPS * G4_STAGES * (a.slots / 4) * (ob + ot) + 128;  // + alignment slack
  if (smem > 220 * 1024) return cudaErrorNotSupported;
  static size_t attr_set = 0;
  if (smem > attr_set) {
    cudaFuncSetAttribute(gather_g4_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    attr_set = smem;
  }
  int per_sm = 0;
  cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, gather_g4_kernel, G4_WARPS * 32, smem);
  if (per_sm < 1) return cudaErrorNotSupported;
  const int64_t tiles = (cap + G4_TILE - 1) / G4_TILE;
  int64_t blocks = std::min<int64_t>((int64_t)h->sm_count * per_sm, (tiles + G4_WARPS - 1) / G4_WARPS);
  blocks = std::max<int64_t>(blocks, 1);
  return launch_pdl(gather_g4_kernel, (unsigned)blocks, G4_WARPS * 32, smem, st, a, maps);
}

}  // namespace wg
