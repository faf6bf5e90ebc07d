// sample.cu -- multi-GPU sampling op (Algorithm 1).
//
// sample_kernel (no scan, no inter-block dependency): a group of G = max(M, 4) lanes
// (fanout M <= 32) handles one target; each warp handles SAMPLE_UNR rounds
// of floor(32/G) targets at once, so every lane keeps SAMPLE_UNR independent neighbour loads
// in flight (the op is latency-bound: random 16 B row_ptr and 8 B col reads, local or
// over NVLink).  Per target:
//   - lane u of the group loads the (row_ptr[l], row_ptr[l+1]) pair of round u's
//     target from its owner o(v) (local HBM or a peer);
//   - if M >= N every lane i < N takes position i (L118: "all of N neighbors are
//     sampled", CSR order, A5);
//   - otherwise lane i draws r_i (Philox4x32-10, reading A3) and computes Algorithm
//     1's res[i] WITHOUT the sort: __match_any_sync on r gives, per lane, the previous
//     draw with the same value (the p[q[i]-1] of Alg.1 line 8) and whether it is the
//     last one (the run-end test of line 4); the chain of line 5 lives in 32 words of
//     shared memory per warp, path doubling (line 12) is log2(M) __shfl_sync rounds
//     and last (line 7) a subtraction.  This computes the same function as Algorithm 1
//     for every draw vector (both equal sequential partial Fisher-Yates; DESIGN.md
//     "Sampler");
//   - lane i loads col[start + res_i] and writes it to the PADDED slot k*M + i of the
//     workspace (draw order, A5); lane 0 writes cnt[k] = min(M, N).
// The dense CSR output (row_ptr = exclusive scan of cnt, compact neighbours) is
// produced by one scan pass afterwards: sample_compact_kernel for wg_sample_neighbors,
// or the flag pass of Append Unique for the fused hop (unique.cu), which scans the
// valid slots and the first occurrences together.
#include "hash.cuh"
#include "sample_warp.cuh"
#include "scan.cuh"

namespace wg {

#ifndef WG_SAMPLE_THREADS
#define WG_SAMPLE_THREADS 256  // threads per sampler block (A/B knob via WG_NVCC_DEFS)
#endif
constexpr int SAMPLE_THREADS = WG_SAMPLE_THREADS;
#ifndef SAMPLE_MINB
#define SAMPLE_MINB 6  // resident sampler blocks per SM the register allocation must allow
#endif
// SAMPLE_UNR = rounds per warp, all in flight at once (1, 2 or 4; chosen per launch: small hops use
// fewer rounds per warp and therefore more blocks / SMs); sample_group / the per-warp body: sample_warp.cuh

struct SampleArgs {
  ShardView s;
  const int64_t* targets;
  int64_t cap;
  const int64_t* d_n;
  int M;
  int hop;
  unsigned long long seed;
  const unsigned long long* d_seed;
  int64_t* nbrs_pad;  // [nT * M] (uint32 elements when pad32)
  int32_t* pos_pad;   // [nT * M]
  int32_t* cnt;       // [nT]
  unsigned* ctrl;
  HashTable ht;                // fused hop, compact hash table (prefix size of this hop's key bound)
  int64_t hwords;              // its full capacity (the idle table is zeroed at a cycle's first op)
  int pad32;                   // padded neighbour slots hold uint32 ids (num_nodes < 2^32)
  // MODE_DIRECT (fused hop with the direct table): the Append Unique insert happens here -- targets
  // first (U[k] = T[k], their own position k, duplicate-target check), every sampled id a RED.MIN of
  // its padded position nT + k*M + i (same order as the dense positions); padding slots get PAD_ID
  DirectTable dt;
  int64_t* U;
  int32_t* dup;
};
// sampler modes: plain; plain + the compact table's clear-ahead (fused hop with the compact hash: the
// insert pass follows); fused hop with the direct table, inserting here (the hop then has no insert pass).
// (Inserting into the compact hash table here measured slower: profiles/r02/ab_log.md.)
enum { MODE_PLAIN = 0, MODE_CLEAR = 1, MODE_DIRECT = 2 };

// Padded slot without a sample (direct mode: the flag pass reads no per-target count)
__device__ __forceinline__ int64_t pad_id(int pad32) { return pad32 ? (int64_t)0xFFFFFFFFu : (int64_t)-1; }

// Target k of a fused direct hop: U[k] = v (targets first, in order, L160), its word takes position k.
// Issued as soon as the target id is loaded, so that a hub that is also a target already holds a
// position smaller than every neighbour's when the neighbours' filtered inserts read it; the returned
// old word is checked at the end (direct_target_check): an earlier TARGET record of v (position < nT)
// in this epoch is a duplicate target (A8) -- of two equal targets the later atomic sees the other.
__device__ __forceinline__ unsigned direct_insert_target(const SampleArgs& a, unsigned* t, unsigned tag, int64_t k,
                                                         int64_t v) {
  a.U[k] = v;
  if (a.dup) a.dup[k] = 0;
  if (v < 0 || v >= a.s.n) return ~0u;  // the sampler latches WG_DEVERR_ID_RANGE
  return atomicMin(&t[v], dword(tag, k));
}
__device__ __forceinline__ void direct_target_check(const SampleArgs& a, unsigned tag, int64_t nT, unsigned old) {
  if ((old >> DPOS_BITS) == tag && (int64_t)(old & DPOS_MASK) < nT) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_DUP_TARGET);
}
// Sampled id nb at padded position q: RED.MIN of its word, issued only when a plain load of the word shows
// a larger position (the filter: hubs meet their own target's or an earlier sample's smaller position and
// issue no atomic; unfiltered REDs serialise on hub words, profiles/r02/ab_log.md).  Batched over a lane's
// UNR rounds: every round's load is issued before any is resolved.
template <int UNR>
__device__ __forceinline__ void direct_insert_nbrs(const SampleArgs& a, unsigned* t, unsigned tag, int64_t nT, int M,
                                                   int i, const int64_t* nb, const int64_t* kk, const bool* ok) {
  unsigned cur[UNR];
  bool in[UNR];
#pragma unroll
  for (int u = 0; u < UNR; ++u) {
    in[u] = ok[u] && nb[u] >= 0 && nb[u] < a.s.n;
    if (ok[u] && !in[u]) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
    cur[u] = 0u;
    if (in[u]) asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(cur[u]) : "l"(&t[nb[u]]));
  }
#pragma unroll
  for (int u = 0; u < UNR; ++u) {
    const unsigned mine = dword(tag, nT + kk[u] * M + i);
    if (in[u] && cur[u] > mine) atomicMin(&t[nb[u]], mine);
  }
}
// Single-key form (block sampler).
__device__ __forceinline__ void direct_insert_nbr(const SampleArgs& a, unsigned* t, unsigned tag, int64_t q,
                                                  int64_t nb) {
  if (nb < 0 || nb >= a.s.n) {
    latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
    return;
  }
  const unsigned mine = dword(tag, q);
  unsigned cur;
  asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(cur) : "l"(&t[nb]));
  if (cur > mine) atomicMin(&t[nb], mine);
}

template <int SAMPLE_UNR, int MODE, bool COL32>
__global__ void __launch_bounds__(SAMPLE_THREADS, SAMPLE_MINB) sample_kernel(const SampleArgs a) {
  pdl_enter();
  KT_BEGIN(0);
  unsigned epoch = 0;
  if (MODE != MODE_PLAIN) epoch = a.ctrl[CTRL_EPOCH];
  if (MODE == MODE_CLEAR) chash_clear_ahead(a.ht, a.hwords, epoch);
  if (MODE == MODE_DIRECT) dtab_clear_ahead(a.dt, epoch);
  __shared__ unsigned sm_chain[SAMPLE_THREADS / 32][32];
  const int tid = threadIdx.x, warp = tid >> 5;
  int64_t nT = a.cap;
  if (a.d_n) {
    nT = *a.d_n;
    if (nT > a.cap || nT < 0) {
      if (tid == 0 && blockIdx.x == 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
      nT = nT < 0 ? 0 : a.cap;
    }
  }
  const int M = a.M;
  const int TPW = 32 / sample_group(M);
  const int64_t warp_base = ((int64_t)blockIdx.x * (SAMPLE_THREADS / 32) + warp) * (TPW * SAMPLE_UNR);
  const unsigned long long seed = a.d_seed ? *a.d_seed : a.seed;
  const uint2 key = make_uint2((unsigned)(seed & 0xffffffffu), (unsigned)(seed >> 32));
  // padded slots k*M + i of the workspace (the scan pass that follows compacts them)
  unsigned* const dt = MODE == MODE_DIRECT ? dtab_cur(a.dt, epoch) : nullptr;
  const unsigned tag = MODE == MODE_DIRECT ? dtag(epoch) : 0u;
  sample_warp<SAMPLE_UNR, COL32>(
      a.s, a.targets, nT, M, a.hop, key, warp_base, sm_chain[warp], &a.ctrl[CTRL_ERR],
      [&](int64_t k, int64_t v) -> unsigned {
        return MODE == MODE_DIRECT ? direct_insert_target(a, dt, tag, k, v) : 0u;
      },
      [&](int64_t k, unsigned tok) {
        if (MODE == MODE_DIRECT) direct_target_check(a, tag, nT, tok);
      },
      [&](int64_t k, int c) {
        if (MODE != MODE_DIRECT) a.cnt[k] = c;
      },
      [&](int64_t k, int i, int64_t nb, unsigned pos) {
        st_pad(a.nbrs_pad, a.pad32, k * M + i, nb);
        if (a.pos_pad) a.pos_pad[k * M + i] = (int32_t)pos;
      },
      [&](int64_t k, int i) {
        if (MODE == MODE_DIRECT) st_pad(a.nbrs_pad, a.pad32, k * M + i, pad_id(a.pad32));
      },
      [&](const int64_t* nb, const int64_t* kk, const bool* ok) {
        const int i = (threadIdx.x & 31) - ((threadIdx.x & 31) / sample_group(M)) * sample_group(M);
        if (MODE == MODE_DIRECT) direct_insert_nbrs<SAMPLE_UNR>(a, dt, tag, nT, M, i, nb, kk, ok);
      });
  KT_END(0, "sample", nT);
}

// ---------------------------------------------------------------- fanout > 32
// One block of BT = next_pow2(M) threads per target, "M threads in the thread block of
// CUDA are grouped together to generate the sampled neighbors for one target node"
// (L118): Algorithm 1 exactly as listed (L122-158), with parallel_sort = a block bitonic
// sort of the packed 64-bit keys (r << 32 | i) (L118-120) in shared memory, chain / q /
// last in shared memory and path doubling as ceil(log2 M) synchronous rounds.
template <int BT, int MODE, bool COL32>
__global__ void __launch_bounds__(BT) sample_block_kernel(const SampleArgs a) {
  pdl_enter();
  unsigned epoch = 0;
  if (MODE != MODE_PLAIN) epoch = a.ctrl[CTRL_EPOCH];
  if (MODE == MODE_CLEAR) chash_clear_ahead(a.ht, a.hwords, epoch);
  if (MODE == MODE_DIRECT) dtab_clear_ahead(a.dt, epoch);
  unsigned* const dt = MODE == MODE_DIRECT ? dtab_cur(a.dt, epoch) : nullptr;
  const unsigned tag = MODE == MODE_DIRECT ? dtag(epoch) : 0u;
  __shared__ unsigned long long s_key[BT];
  __shared__ unsigned s_r[BT], s_chain[BT], s_q[BT], s_last[BT];
  __shared__ int64_t s_v, s_start;
  __shared__ unsigned s_n;
  int64_t nT = a.cap;
  if (a.d_n) {
    nT = *a.d_n;
    nT = nT < 0 ? 0 : (nT > a.cap ? a.cap : nT);
  }
  const int64_t k = blockIdx.x;
  if (k >= nT) return;
  const int i = threadIdx.x;
  const int M = a.M;
  if (i == 0) {
    int64_t v = a.targets[k], start = 0;
    unsigned n = 0;
    if (MODE == MODE_DIRECT) direct_target_check(a, tag, nT, direct_insert_target(a, dt, tag, k, v));
    if (v < 0 || v >= a.s.n) {
      latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
      v = -1;
    } else {
      int o;
      int64_t l;
      csr_owner_local(a.s, v, o, l);
      const int64_t* rp = a.s.row_ptr[o] + l;
      start = rp[0];
      const int64_t d = rp[1] - start;
      if (d >= (int64_t(1) << 32) || d < 0)
        latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_DEGREE);
      else
        n = (unsigned)d;
    }
    s_v = v;
    s_start = start;
    s_n = n;
    if (MODE != MODE_DIRECT) a.cnt[k] = v >= 0 ? (int32_t)min(n, (unsigned)M) : 0;
  }
  __syncthreads();
  const int64_t v = s_v;
  const unsigned N = s_n;
  // direct mode: slots past min(M, N) (all M for an invalid target) are padding
  if (MODE == MODE_DIRECT && i < M && (v < 0 || (unsigned)i >= N))
    st_pad(a.nbrs_pad, a.pad32, k * M + i, pad_id(a.pad32));
  if (v < 0) return;
  int o;
  int64_t l;
  csr_owner_local(a.s, v, o, l);
  const int64_t cbase = s_start;
  if (N <= (unsigned)M) {  // L118: all of N neighbours, CSR order (A5)
    for (unsigned j = i; j < N; j += BT) {
      const int64_t nb = ld_col<COL32>(a.s, o, cbase + j);
      st_pad(a.nbrs_pad, a.pad32, k * M + j, nb);
      if (a.pos_pad) a.pos_pad[k * M + j] = (int32_t)j;
      if (MODE == MODE_DIRECT) direct_insert_nbr(a, dt, tag, nT + k * M + j, nb);
    }
    return;
  }
  // line 1-4: r[i] = random(N-1-i); chain[i] = i
  const unsigned long long seed = a.d_seed ? *a.d_seed : a.seed;
  unsigned r = 0;
  if (i < M) {
    const uint4 x = philox4x32_10(make_uint4((unsigned)(i >> 2), (unsigned)a.hop, (unsigned)((uint64_t)v & 0xffffffffu),
                                             (unsigned)((uint64_t)v >> 32)),
                                  make_uint2((unsigned)(seed & 0xffffffffu), (unsigned)(seed >> 32)));
    const unsigned xi = (i & 3) == 0 ? x.x : (i & 3) == 1 ? x.y : (i & 3) == 2 ? x.z : x.w;
    r = __umulhi(xi, N - (unsigned)i);
  }
  s_r[i] = r;
  s_chain[i] = (unsigned)i;
  s_key[i] = i < M ? (((unsigned long long)r << 32) | (unsigned)i) : ~0ull;
  __syncthreads();
  // line 5: s, p = parallel_sort(r) -- bitonic sort of the packed keys
  for (int size = 2; size <= BT; size <<= 1) {
    for (int stride = size >> 1; stride > 0; stride >>= 1) {
      const int partner = i ^ stride;
      if (partner > i) {
        const unsigned long long x = s_key[i], y = s_key[partner];
        const bool up = (i & size) == 0;
        if ((x > y) == up) {
          s_key[i] = y;
          s_key[partner] = x;
        }
      }
      __syncthreads();
    }
  }
  // lines 6-11
  unsigned si = 0, pi = 0;
  if (i < M) {
    si = (unsigned)(s_key[i] >> 32);
    pi = (unsigned)(s_key[i] & 0xffffffffu);
    s_q[pi] = (unsigned)i;
    const bool run_end = (i == M - 1) || si != (unsigned)(s_key[i + 1] >> 32);
    if (run_end && si >= N - (unsigned)M) s_chain[N - si - 1] = pi;
  }
  __syncthreads();
  // line 12: path doubling
  for (int step = 1; step < M; step <<= 1) {
    const unsigned c = i < M ? s_chain[s_chain[i]] : 0u;
    __syncthreads();
    if (i < M) s_chain[i] = c;
    __syncthreads();
  }
  // lines 13-15
  if (i < M) s_last[i] = N - s_chain[i] - 1;
  __syncthreads();
  // lines 16-22
  if (i < M) {
    const unsigned qi = s_q[i];
    unsigned res;
    if (i == 0 || qi == 0 || (unsigned)(s_key[qi] >> 32) != (unsigned)(s_key[qi - 1] >> 32))
      res = s_r[i];
    else
      res = s_last[(unsigned)(s_key[qi - 1] & 0xffffffffu)];
    const int64_t nb = ld_col<COL32>(a.s, o, cbase + res);
    st_pad(a.nbrs_pad, a.pad32, k * M + i, nb);
    if (a.pos_pad) a.pos_pad[k * M + i] = (int32_t)res;
    if (MODE == MODE_DIRECT) direct_insert_nbr(a, dt, tag, nT + k * M + i, nb);
  }
}

// ---------------------------------------------------------------- compaction
// out_row_ptr = exclusive scan of cnt; out_nbrs / out_pos = the valid padded slots in
// order.  Single pass, decoupled look-back over tiles of COMPACT_TILE targets.
constexpr int COMPACT_THREADS = 256;
constexpr int COMPACT_TILE = COMPACT_THREADS;

struct CompactArgs {
  int64_t cap;
  const int64_t* d_n;
  int M;
  const int64_t* nbrs_pad;
  const int32_t* pos_pad;
  const int32_t* cnt;
  int64_t* out_row_ptr;
  int64_t* out_nbrs;
  int32_t* out_pos;
  int64_t* d_num_edges;
  unsigned long long* status;
  unsigned* ctrl;
  int pad32;
};

__global__ void __launch_bounds__(COMPACT_THREADS) sample_compact_kernel(const CompactArgs a) {
  pdl_enter();
  __shared__ LookbackSmem<COMPACT_THREADS> lb;
  __shared__ int sm_wtot[COMPACT_THREADS / 32 + 1];
  __shared__ int sm_flag;
  int64_t nT = a.cap;
  if (a.d_n) {
    nT = *a.d_n;
    nT = nT < 0 ? 0 : (nT > a.cap ? a.cap : nT);
  }
  const int tid = threadIdx.x;
  const int64_t tile_start = (int64_t)blockIdx.x * COMPACT_TILE;
  if (nT == 0) {
    if (blockIdx.x == 0 && tid == 0) {
      a.out_row_ptr[0] = 0;
      if (a.d_num_edges) *a.d_num_edges = 0;
    }
  } else if (tile_start < nT) {
    const int64_t k = tile_start + tid;
    const int c = k < nT ? a.cnt[k] : 0;
    int agg;
    const int ex = block_exclusive_sum<COMPACT_THREADS>(c, sm_wtot, &agg);
    const unsigned long long pre =
        gridDim.x <= WG_LB_DIRECT_MAX
            ? block_prefix_direct<COMPACT_THREADS>(a.status, (long)blockIdx.x, (unsigned long long)agg, lb)
            : block_lookback<COMPACT_THREADS>(a.status, (long)blockIdx.x, (unsigned long long)agg, lb);
    const int64_t off = (int64_t)pre + ex;
    if (k < nT) {
      a.out_row_ptr[k] = off;
      for (int i = 0; i < c; ++i) {
        a.out_nbrs[off + i] = ld_pad(a.nbrs_pad, a.pad32, k * a.M + i);
        if (a.out_pos) a.out_pos[off + i] = a.pos_pad[k * a.M + i];
      }
      if (k == nT - 1) {
        a.out_row_ptr[nT] = off + c;
        if (a.d_num_edges) *a.d_num_edges = off + c;
      }
    }
  }
  if (finish_block(&a.ctrl[CTRL_DONE_SAMPLE], &sm_flag)) {
    for (int t = tid; t < (int)gridDim.x; t += COMPACT_THREADS) a.status[t] = 0ull;
    if (tid == 0) a.ctrl[CTRL_DONE_SAMPLE] = 0u;
  }
}

template <int MODE, bool COL32>
static cudaError_t launch_block_sampler(int fanout, unsigned blocks, const SampleArgs& a, cudaStream_t st) {
  if (fanout <= 64) return launch_pdl(sample_block_kernel<64, MODE, COL32>, blocks, 64, 0, st, a);
  if (fanout <= 128) return launch_pdl(sample_block_kernel<128, MODE, COL32>, blocks, 128, 0, st, a);
  if (fanout <= 256) return launch_pdl(sample_block_kernel<256, MODE, COL32>, blocks, 256, 0, st, a);
  if (fanout <= 512) return launch_pdl(sample_block_kernel<512, MODE, COL32>, blocks, 512, 0, st, a);
  return launch_pdl(sample_block_kernel<1024, MODE, COL32>, blocks, 1024, 0, st, a);
}

template <int MODE, bool COL32>
static cudaError_t launch_warp_sampler(int unr, unsigned blocks, const SampleArgs& a, cudaStream_t st) {
  if (unr == 4) return launch_pdl(sample_kernel<4, MODE, COL32>, blocks, SAMPLE_THREADS, 0, st, a);
  if (unr == 2) return launch_pdl(sample_kernel<2, MODE, COL32>, blocks, SAMPLE_THREADS, 0, st, a);
  return launch_pdl(sample_kernel<1, MODE, COL32>, blocks, SAMPLE_THREADS, 0, st, a);
}

template <int MODE>
static cudaError_t launch_sampler_mode(bool block, bool col32, int fanout, int unr, unsigned blocks,
                                       const SampleArgs& a, cudaStream_t st) {
  if (block) return col32 ? launch_block_sampler<MODE, true>(fanout, blocks, a, st)
                          : launch_block_sampler<MODE, false>(fanout, blocks, a, st);
  return col32 ? launch_warp_sampler<MODE, true>(unr, blocks, a, st) : launch_warp_sampler<MODE, false>(unr, blocks, a, st);
}

cudaError_t launch_sample_padded(wg_dsm* h, const int64_t* targets, int64_t cap, const int64_t* d_n, int fanout,
                                 uint64_t seed, const uint64_t* d_seed, int hop, bool want_pos, cudaStream_t st,
                                 int64_t* U, int32_t* dup) {
  SampleArgs a;
  a.s = h->view;
  a.targets = targets;
  a.cap = cap;
  a.d_n = d_n;
  a.M = fanout;
  a.hop = hop;
  a.seed = seed;
  a.d_seed = reinterpret_cast<const unsigned long long*>(d_seed);
  a.nbrs_pad = h->ws.nbrs_pad;
  a.pad32 = h->ws.pad32;
  a.pos_pad = want_pos ? h->ws.pos_pad : nullptr;
  a.cnt = h->ws.cnt;
  a.ctrl = h->ws.ctrl;
  a.ht = HashTable{h->ws.hslots, (unsigned long long)table_prefix(h, cap + cap * fanout), h->ws.compact,
                   reinterpret_cast<HashSlot*>(h->ws.hslots2)};
  a.hwords = h->ws.hcap;
  a.dt = DirectTable{{h->ws.dtab[0], h->ws.dtab[1]}, h->n};
  a.U = U;
  a.dup = dup;
  // U != NULL: the fused hop (wg_sample_hop); with the direct key table its inserts happen here
  // (launch_hop skips the insert pass, hop_inserts_in_sampler)
  const int mode = !U ? MODE_PLAIN : h->ws.direct ? MODE_DIRECT : h->ws.compact ? MODE_CLEAR : MODE_PLAIN;
  const bool block = fanout > 32;  // block per target (Algorithm 1 with a block sort)
  int unr = 1;
  unsigned blocks = (unsigned)(cap > 0 ? cap : 1);
  if (!block) {
    const int G = sample_group(fanout);
    const int tpw = 32 / G;
    unr = SAMPLE_UNR_MAX;  // largest of 4/2/1 that still gives >= 2 blocks per SM
    while (unr > 1 && cap < (int64_t)(SAMPLE_THREADS / 32) * tpw * unr * 2 * h->sm_count) unr >>= 1;
    const int64_t tile = (int64_t)(SAMPLE_THREADS / 32) * tpw * unr;
    blocks = (unsigned)(cap > 0 ? (cap + tile - 1) / tile : 1);
  }
  const bool c32 = a.s.col32 != 0;
  if (mode == MODE_DIRECT) return launch_sampler_mode<MODE_DIRECT>(block, c32, fanout, unr, blocks, a, st);
  if (mode == MODE_CLEAR) return launch_sampler_mode<MODE_CLEAR>(block, c32, fanout, unr, blocks, a, st);
  return launch_sampler_mode<MODE_PLAIN>(block, c32, fanout, unr, blocks, a, st);
}

// Whether the fused hop's sampler inserts the keys itself (no insert pass), for launch_hop.
bool hop_inserts_in_sampler(const wg_dsm* h) { return h->ws.direct != 0; }

cudaError_t launch_sample(wg_dsm* h, const int64_t* targets, int64_t cap, const int64_t* d_n, int fanout,
                          uint64_t seed, const uint64_t* d_seed, int hop, int64_t* out_row_ptr,
                          int64_t* out_nbrs, int32_t* out_pos, int64_t* d_num_edges, cudaStream_t st) {
  cudaError_t e =
      launch_sample_padded(h, targets, cap, d_n, fanout, seed, d_seed, hop, out_pos != nullptr, st, nullptr, nullptr);
  if (e != cudaSuccess) return e;
  CompactArgs c{cap, d_n, fanout, h->ws.nbrs_pad, h->ws.pos_pad, h->ws.cnt, out_row_ptr, out_nbrs, out_pos,
                d_num_edges, h->ws.status_sample, h->ws.ctrl, h->ws.pad32};
  const unsigned blocks = (unsigned)(cap > 0 ? (cap + COMPACT_TILE - 1) / COMPACT_TILE : 1);
  return launch_pdl(sample_compact_kernel, blocks, COMPACT_THREADS, 0, st, c);
}

}  // namespace wg
