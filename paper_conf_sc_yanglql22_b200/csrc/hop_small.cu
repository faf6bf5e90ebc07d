// hop_small.cu -- one whole SMALL hop (sampling L116-158 + Append Unique L160-166 + the sub-graph CSR)
// in ONE kernel launch: a cluster of SH_CTAS thread blocks whose hash table lives in distributed shared
// memory (DSMEM).  Used by wg_sample_hop when n_targets * (1 + fanout) <= SH_MAX_KEYS and fanout <= 32
// (the first hop of a mini-batch: 1024 seeds x 15 = 16k keys), unless WG_DSM_NO_CLUSTER_HOP.
//
// Why: a small hop on the general path is four launch- and latency-bound kernels (sample, insert, flag
// scan with a decoupled look-back, relabel) over a global hash table, ~22 us for 1k targets on B200.
// Here every step after the sampler's DRAM loads runs on-chip, separated by cluster barriers:
//   1. block c samples targets [c*TPC, (c+1)*TPC) into its shared-memory padded slots (the warp
//      sampler of sample_warp.cuh: same draws, same positions);
//   2. every target and sampled neighbour is inserted into the DSMEM hash table (slot s lives in
//      block s / SH_SLOTS): 64-bit CAS claim of {id, position}, atomicMin of the position otherwise --
//      the table records each id's FIRST position in [targets ; padded neighbours] (A7, as unique.cu);
//   3. flags valid / first-occurrence per padded slot, a block scan, and the cluster prefix from the
//      lower blocks' aggregates (DSMEM reads, no look-back): dense CSR position p and new-node index f;
//   4. sub_col = the id of each neighbour's first occurrence, read from the owner block's new-id array
//      (so no separate relabel pass), and the duplicate counts (DSMEM counters per hash slot).
// Results are identical to the general path (same padded positions, same first-appearance rule).
#include <cooperative_groups.h>

#include <cstdio>
#include <mutex>

#include "device_util.cuh"

#include "sample_warp.cuh"

namespace cg = cooperative_groups;

namespace wg {

__device__ __forceinline__ void cluster_sync(cg::cluster_group& cl) { cl.sync(); }
#ifndef WG_SH_PRINT
#define WG_SH_PRINT 0
#endif
__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

constexpr int SH_CTAS = 16;        // cluster size (non-portable: needs 16 SMs of one GPC)
constexpr int SH_THREADS = 512;
constexpr int SH_WARPS = SH_THREADS / 32;
constexpr int SH_SLOTS = 4096;     // hash slots per block (8 B words): 64k slots per cluster
constexpr int SH_PAD = 2048;       // padded sampler slots per block (targets per block x fanout)
constexpr int SH_ITEMS = SH_PAD / SH_THREADS;
constexpr int64_t SH_MAX_KEYS = (int64_t)SH_CTAS * SH_SLOTS / 2;  // load factor <= 1/2
constexpr unsigned long long SH_EMPTY = ~0ull;

struct SmallHopArgs {
  ShardView s;
  const int64_t* T;
  int64_t capT;
  const int64_t* d_nT;
  int M;
  int hop;
  unsigned long long seed;
  const unsigned long long* d_seed;
  int64_t* out_row_ptr;
  int64_t* out_nbrs;
  int32_t* out_pos;
  int64_t* d_num_edges;
  int64_t* U;
  int64_t* d_nU;
  int32_t* sub_col;
  int32_t* dup;
  unsigned* ctrl;
};

struct SmallHopSmem {
  unsigned long long hash[SH_SLOTS];  // {id:32, first position:32}, SH_EMPTY when free
  unsigned dupc[SH_SLOTS];            // neighbour occurrences of the slot's id (duplicate counts)
  uint32_t pad_key[SH_PAD];           // sampled neighbour ids, padded slots (k - k0) * M + i
  int32_t pad_pos[SH_PAD];            // their adjacency positions (only when positions are wanted)
  int32_t newid[SH_PAD];              // new-node index f of a first-occurrence slot
  int32_t cnt[SH_PAD];                // per-target sample counts min(M, deg)
  unsigned chain[SH_WARPS][32];       // the warp sampler's chain words
  unsigned long long wtot[SH_WARPS + 1];
  unsigned long long agg;             // this block's (valid << 32 | first) totals, read by higher blocks
};

// Distributed shared memory, addressed with mapa + shared::cluster instructions.  Measured on B200
// (profiles/probes/small_hop_race.py): a 64-bit atomicMin on another block's shared memory is NOT atomic
// under contention -- ptxas lowers atom.shared::cluster.min.u64 (and the generic atomicMin) to a generic
// ATOM.E.MIN.64 whose fallback for non-global addresses is a plain load / min / store, and hub ids lost
// their first position in 23-34 of 40 runs.  The 64-bit CAS is atomic (profiles/probes/dsmem_atomics.cu),
// so positions are lowered with a CAS loop: 0 of 40.
__device__ __forceinline__ unsigned dsm_addr(const void* local, unsigned rank) {
  unsigned r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"((unsigned)__cvta_generic_to_shared(local)), "r"(rank));
  return r;
}
__device__ __forceinline__ unsigned long long dsm_cas64(unsigned a, unsigned long long cmp, unsigned long long v) {
  unsigned long long old;
  asm volatile("atom.shared::cluster.cas.b64 %0, [%1], %2, %3;" : "=l"(old) : "r"(a), "l"(cmp), "l"(v) : "memory");
  return old;
}
__device__ __forceinline__ void dsm_add32(unsigned a, unsigned v) {
  asm volatile("red.shared::cluster.add.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ unsigned long long dsm_ld64(unsigned a) {
  unsigned long long v;
  asm volatile("ld.shared::cluster.u64 %0, [%1];" : "=l"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ unsigned dsm_ld32(unsigned a) {
  unsigned v;
  asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(v) : "r"(a) : "memory");
  return v;
}
__device__ __forceinline__ unsigned hash_addr(SmallHopSmem& sm, int slot) {
  return dsm_addr(&sm.hash[slot % SH_SLOTS], (unsigned)(slot / SH_SLOTS));
}
__device__ __forceinline__ unsigned dupc_addr(SmallHopSmem& sm, int slot) {
  return dsm_addr(&sm.dupc[slot % SH_SLOTS], (unsigned)(slot / SH_SLOTS));
}

// Slot of `key` in the cluster table (claimed with word `mine` if new): returns the global slot and the
// word seen before (SH_EMPTY if this call claimed it, else the atomicMin's old value).
__device__ __forceinline__ int sh_insert(SmallHopSmem& sm, uint32_t key, uint32_t q, unsigned long long* old) {
  constexpr unsigned TOTAL = (unsigned)SH_CTAS * SH_SLOTS;
  const unsigned long long mine = ((unsigned long long)key << 32) | q;
  unsigned slot = (unsigned)__umul64hi(fmix64((unsigned long long)key), (unsigned long long)TOTAL);
  for (unsigned probe = 0; probe < TOTAL; ++probe) {
    const unsigned w = hash_addr(sm, (int)slot);
    unsigned long long cur = dsm_ld64(w);  // a read first: hub ids are found without any atomic
    for (;;) {
      if (cur == SH_EMPTY) {
        cur = dsm_cas64(w, SH_EMPTY, mine);
        if (cur == SH_EMPTY) {
          *old = SH_EMPTY;
          return (int)slot;
        }
        continue;  // claimed meanwhile: re-examine
      }
      if ((uint32_t)(cur >> 32) != key) break;  // another id: next slot
      while ((cur & 0xffffffffull) > q) {  // lower the position with a CAS loop (not atom.min.u64: see above)
        const unsigned long long o = dsm_cas64(w, cur, mine);
        if (o == cur) break;
        cur = o;
      }
      *old = cur;
      return (int)slot;
    }
    slot = slot + 1 == TOTAL ? 0 : slot + 1;
  }
  return -1;
}

template <int UNR, bool COL32>
__global__ void __launch_bounds__(SH_THREADS, 1) hop_small_kernel(const SmallHopArgs a) {
  unsigned long long T0 = WG_SH_PRINT ? gtime() : 0ull;
  pdl_enter();
  unsigned long long T1 = WG_SH_PRINT ? gtime() : 0ull;
  extern __shared__ __align__(16) unsigned char sh_raw[];
  SmallHopSmem& sm = *reinterpret_cast<SmallHopSmem*>(sh_raw);
  cg::cluster_group cl = cg::this_cluster();
  const int crank = (int)cl.block_rank();
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const unsigned lt = (1u << lane) - 1u;
  unsigned* err = &a.ctrl[CTRL_ERR];

  for (int i = tid; i < SH_SLOTS; i += SH_THREADS) {
    sm.hash[i] = SH_EMPTY;
    sm.dupc[i] = 0u;
  }
  int64_t nT = a.d_nT ? *a.d_nT : a.capT;
  if (nT > a.capT || nT < 0) {
    if (tid == 0 && crank == 0) latch_error(err, WG_DEVERR_CAPACITY);
    nT = nT < 0 ? 0 : a.capT;
  }
  const int M = a.M;
  const int64_t TPC = (nT + SH_CTAS - 1) / SH_CTAS;  // targets per block (<= SH_PAD / M, host-checked)
  const int64_t k0 = (int64_t)crank * TPC;
  const int64_t k1 = k0 + TPC < nT ? k0 + TPC : nT;
  const int nloc = k1 > k0 ? (int)(k1 - k0) : 0;
  const int L = nloc * M;  // this block's padded slots

  // ---- 1. sample this block's targets into the shared padded slots
  {
    const unsigned long long seed = a.d_seed ? *a.d_seed : a.seed;
    const uint2 key = make_uint2((unsigned)(seed & 0xffffffffu), (unsigned)(seed >> 32));
    const int TPW = 32 / sample_group(M);
    const int64_t step = (int64_t)SH_WARPS * TPW * UNR;
    for (int64_t base = k0 + (int64_t)warp * TPW * UNR; base < k1; base += step)
      sample_warp<UNR, COL32>(
          a.s, a.T, k1, M, a.hop, key, base, sm.chain[warp], err, [&](int64_t k, int c) { sm.cnt[k - k0] = c; },
          [&](int64_t k, int i, int64_t nb, unsigned pos) {
            sm.pad_key[(k - k0) * M + i] = (uint32_t)nb;
            if (a.out_pos) sm.pad_pos[(k - k0) * M + i] = (int32_t)pos;
          });
  }
  unsigned long long P0a = WG_SH_PRINT ? gtime() : 0ull;
  cluster_sync(cl);  // every block's table is initialised and every block's samples are in place
  unsigned long long P0b = WG_SH_PRINT ? gtime() : 0ull;

  // ---- 2. insert targets (positions k) and sampled neighbours (positions nT + global padded index)
  const int64_t pbase = nT + k0 * M;  // position of this block's padded slot 0
  int tslot[SH_ITEMS];
#pragma unroll
  for (int t = 0; t < SH_ITEMS; ++t) {
    const int kl = tid + t * SH_THREADS;
    tslot[t] = -2;
    if (kl < nloc) {
      const int64_t k = k0 + kl;
      const int64_t v = a.T[k];
      a.U[k] = v;  // targets first, input order (L160)
      if (v >= 0 && v < a.s.n) {
        unsigned long long old;
        tslot[t] = sh_insert(sm, (uint32_t)v, (uint32_t)k, &old);
        if (tslot[t] < 0) latch_error(err, WG_DEVERR_CAPACITY);
        else if (old != SH_EMPTY && (int64_t)(old & 0xffffffffull) < nT)
          latch_error(err, WG_DEVERR_DUP_TARGET);  // an earlier target with this id (A8)
      }  // an invalid target id was latched by the sampler (degree 0, no record)
    }
  }
  // warp-striped padded items: warp w covers local slots [w * 32 * SH_ITEMS, ...), lane l slots l + 32 t
  int slot[SH_ITEMS];
  uint32_t key[SH_ITEMS];
  bool valid[SH_ITEMS];
#pragma unroll
  for (int t = 0; t < SH_ITEMS; ++t) {
    const int j = warp * 32 * SH_ITEMS + 32 * t + lane;
    const int kl = j / M;
    valid[t] = j < L && (j - kl * M) < sm.cnt[kl];
    key[t] = valid[t] ? sm.pad_key[j] : 0u;
    slot[t] = -1;
    const bool good = valid[t] && (int64_t)key[t] < a.s.n;
    if (valid[t] && !good) {
      latch_error(err, WG_DEVERR_ID_RANGE);
      slot[t] = -2;  // a sample without a key to number (sub_col -1)
    }
    // one insert per distinct id in the warp: the lowest lane holds the smallest position
    const unsigned same = __match_any_sync(FULL_MASK, good ? (unsigned long long)key[t] : (1ull << 63) | lane);
    const int leader = __ffs(same) - 1;
    int sl = -1;
    if (good && leader == lane) {
      unsigned long long old;
      sl = sh_insert(sm, key[t], (uint32_t)(pbase + j), &old);
      if (sl < 0) latch_error(err, WG_DEVERR_CAPACITY);
    }
    sl = __shfl_sync(FULL_MASK, sl, leader);
    if (good) slot[t] = sl;
  }
  unsigned long long P1a = WG_SH_PRINT ? gtime() : 0ull;
  cluster_sync(cl);  // every first position is final
  unsigned long long P1b = WG_SH_PRINT ? gtime() : 0ull;

  // ---- 3. valid / first flags, block scan, cluster prefix
  int64_t mp[SH_ITEMS];
  unsigned vm[SH_ITEMS], fm[SH_ITEMS];
  unsigned long long wv = 0, wf = 0;
#pragma unroll
  for (int t = 0; t < SH_ITEMS; ++t) {
    const int j = warp * 32 * SH_ITEMS + 32 * t + lane;
    mp[t] = -1;
    if (slot[t] >= 0)
      mp[t] = (int64_t)(dsm_ld64(hash_addr(sm, slot[t])) & 0xffffffffull);
    vm[t] = __ballot_sync(FULL_MASK, valid[t]);
    fm[t] = __ballot_sync(FULL_MASK, valid[t] && mp[t] == pbase + j);
    wv += __popc(vm[t]);
    wf += __popc(fm[t]);
  }
  unsigned long long btot;
  const unsigned long long wex =
      __shfl_sync(FULL_MASK, block_exclusive_sum<SH_THREADS>(lane == 0 ? ((wv << 32) | wf) : 0ull, sm.wtot, &btot), 0);
  if (tid == 0) sm.agg = btot;
  unsigned long long P2a = WG_SH_PRINT ? gtime() : 0ull;
  cluster_sync(cl);  // block aggregates visible
  unsigned long long P2b = WG_SH_PRINT ? gtime() : 0ull;
  unsigned long long pre = 0;
  if (warp == 0) {
    unsigned long long v = lane < crank ? dsm_ld64(dsm_addr(&sm.agg, (unsigned)lane)) : 0ull;
    pre = warp_sum(v);
  }
  if (tid == 0) sm.wtot[SH_WARPS] = pre;  // (block_exclusive_sum is done with wtot)
  __syncthreads();
  pre = sm.wtot[SH_WARPS];
  int64_t ev = (int64_t)((pre + wex) >> 32);
  int64_t ef = (int64_t)((pre + wex) & 0xffffffffull);
  int64_t pos_p[SH_ITEMS];
#pragma unroll
  for (int t = 0; t < SH_ITEMS; ++t) {
    const int j = warp * 32 * SH_ITEMS + 32 * t + lane;
    const int64_t p = ev + __popc(vm[t] & lt);
    const int64_t f = ef + __popc(fm[t] & lt);
    pos_p[t] = p;
    if (j < L && j % M == 0) a.out_row_ptr[k0 + j / M] = p;
    if (valid[t]) {
      a.out_nbrs[p] = (int64_t)key[t];
      if (a.out_pos) a.out_pos[p] = sm.pad_pos[j];
    }
    if ((fm[t] >> lane) & 1u) {
      a.U[nT + f] = (int64_t)key[t];
      sm.newid[j] = (int32_t)f;
    }
    ev += __popc(vm[t]);
    ef += __popc(fm[t]);
  }
  if (crank == SH_CTAS - 1 && tid == 0) {  // totals = this (last) block's prefix + aggregate
    const int64_t tv = (int64_t)((pre + btot) >> 32), tf = (int64_t)((pre + btot) & 0xffffffffull);
    a.out_row_ptr[nT] = tv;
    *a.d_num_edges = tv;
    if (a.d_nU) *a.d_nU = nT + tf;
  }
  unsigned long long P3a = WG_SH_PRINT ? gtime() : 0ull;
  cluster_sync(cl);  // new-node indices visible
  unsigned long long P3b = WG_SH_PRINT ? gtime() : 0ull;

  // ---- 4. sub-graph ids of the neighbours, duplicate counts
#pragma unroll
  for (int t = 0; t < SH_ITEMS; ++t) {
    if (!valid[t]) continue;
    int32_t id = -1;
    if (mp[t] >= 0) {
      if (mp[t] < nT) {
        id = (int32_t)mp[t];
      } else {
        const int64_t jg = mp[t] - nT;  // global padded index of the first occurrence
        const int64_t c = (jg / M) / TPC;
        id = (int32_t)nT + (int32_t)dsm_ld32(dsm_addr(&sm.newid[jg - c * TPC * M], (unsigned)c));
      }
      if (a.dup) dsm_add32(dupc_addr(sm, slot[t]), 1u);
    }
    a.sub_col[pos_p[t]] = id;
  }
  if (a.dup) {
    cluster_sync(cl);  // counts complete
#pragma unroll
    for (int t = 0; t < SH_ITEMS; ++t) {
      const int kl = tid + t * SH_THREADS;
      if (kl < nloc)
        a.dup[k0 + kl] = tslot[t] >= 0 ? (int32_t)dsm_ld32(dupc_addr(sm, tslot[t])) : 0;
      const int j = warp * 32 * SH_ITEMS + 32 * t + lane;
      if ((fm[t] >> lane) & 1u)
        a.dup[nT + sm.newid[j]] = (int32_t)dsm_ld32(dupc_addr(sm, slot[t]));
    }
  }
  cluster_sync(cl);  // no block leaves while another may still read its shared memory
  if (WG_SH_PRINT && tid == 0 && (crank == 0 || crank == 15)) {
    const unsigned long long T9 = gtime();
    printf("SH cta %d: pdl %llu | sample %llu sync %llu | insert %llu sync %llu | flag %llu sync %llu | out %llu sync %llu | sub %llu  total %llu ns\n",
           crank, T1 - T0, P0a - T1, P0b - P0a, P1a - P0b, P1b - P1a, P2a - P1b, P2b - P2a, P3a - P2b, P3b - P3a,
           T9 - P3b, T9 - T0);
  }
}

bool small_hop_eligible(const wg_dsm* h, int64_t capT, int fanout) {
  if (h->flags & WG_DSM_NO_CLUSTER_HOP) return false;
  if (fanout > 32 || capT < 1 || h->n >= (int64_t(1) << 32)) return false;
  if (capT * (int64_t)(fanout + 1) > SH_MAX_KEYS) return false;
  if ((capT + SH_CTAS - 1) / SH_CTAS * fanout > SH_PAD) return false;
  return true;
}

template <int UNR, bool COL32>
static cudaError_t launch_small(int device, const SmallHopArgs& a, cudaStream_t st, bool* unsupported) {
  static std::mutex mu;
  static signed char state[256];  // per device: 0 unknown, 1 the cluster fits, -1 it does not
  auto kern = hop_small_kernel<UNR, COL32>;
  const size_t smem = sizeof(SmallHopSmem);
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(SH_CTAS);
  cfg.blockDim = dim3(SH_THREADS);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = SH_CTAS;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  const int d = device & 255;
  {
    std::lock_guard<std::mutex> g(mu);
    if (state[d] == 0) {
      int clusters = 0;
      const bool ok = cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) == cudaSuccess &&
                      cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem) == cudaSuccess &&
                      cudaOccupancyMaxActiveClusters(&clusters, kern, &cfg) == cudaSuccess && clusters > 0;
      cudaGetLastError();
      state[d] = ok ? 1 : -1;
    }
    if (state[d] < 0) {
      *unsupported = true;
      return cudaSuccess;
    }
  }
  cfg.numAttrs = 2;
  return cudaLaunchKernelEx(&cfg, kern, a);
}

// Returns cudaSuccess with *launched = false when the device cannot run the cluster (the caller then
// takes the general path).
cudaError_t launch_small_hop(wg_dsm* h, const int64_t* T, int64_t capT, const int64_t* d_nT, int fanout, uint64_t seed,
                             const uint64_t* d_seed, int hop, int64_t* out_row_ptr, int64_t* out_nbrs,
                             int32_t* out_pos, int64_t* d_num_edges, int64_t* U, int64_t* d_nU, int32_t* sub_col,
                             int32_t* dup, cudaStream_t st, bool* launched) {
  SmallHopArgs a;
  a.s = h->view;
  a.T = T;
  a.capT = capT;
  a.d_nT = d_nT;
  a.M = fanout;
  a.hop = hop;
  a.seed = seed;
  a.d_seed = reinterpret_cast<const unsigned long long*>(d_seed);
  a.out_row_ptr = out_row_ptr;
  a.out_nbrs = out_nbrs;
  a.out_pos = out_pos;
  a.d_num_edges = d_num_edges;
  a.U = U;
  a.d_nU = d_nU;
  a.sub_col = sub_col;
  a.dup = dup;
  a.ctrl = h->ws.ctrl;
  bool unsupported = false;
  cudaError_t e = a.s.col32 ? launch_small<2, true>(h->device, a, st, &unsupported)
                            : launch_small<2, false>(h->device, a, st, &unsupported);
  *launched = e == cudaSuccess && !unsupported;
  return e;
}

}  // namespace wg
