// unique.cu -- Append Unique op with first-appearance numbering (A7),
// and its fusion with the sampling op for one whole hop (wg_sample_hop).
//
// Keys live in the open-addressing hash table of hash.cuh, which stays in L2.
// Instead of the paper's per-bucket count of -1 values (whose order depends on the
// insertion race), every key records the MINIMUM position at which it occurs in
// the concatenated list [targets ; neighbours]; a neighbour position is a "first
// occurrence" iff that minimum is its own position, and the new ids are nT +
// exclusive scan of the first-occurrence flags.  The result is deterministic and
// equals the sequential definition.  Kernels:
//   insert   every key; __match_any_sync elects one lane per distinct key in a warp;
//            CAS claims a slot, atomicMin records the first position; every position
//            remembers its slot (slot_of).
//            It also copies the targets to U (targets first, L160) and detects
//            duplicate targets from the atomicMin's old value (A8).
//   flag     single-pass scan (block-wide decoupled look-back) over the neighbour
//            positions: reads the min position through slot_of (one dependent L2
//            read, no probing), writes U for first occurrences and the scan.  Its last
//            block advances the table epoch.
//   relabel  sub_col[p] = id of nbrs[p]; optional duplicate counts (L186).  Nothing
//            else in the batch reads it, so the fused hop runs it on a side stream.
// PADDED = true is the fused hop: neighbours come from the sampler's padded slots
// k*M + i (valid iff i < cnt[k]), positions are padded positions (same order as the
// dense ones), and the flag pass scans "valid" and "first" together -- it also emits
// the sampler's dense CSR (row_ptr, neighbours, positions), so no separate compaction
// pass is needed.
#include <climits>
#include <cstdlib>

#include <algorithm>

#include "hash.cuh"
#include "scan.cuh"

#ifndef WG_UQ_THREADS
#define WG_UQ_THREADS 256  // threads per append-unique block (A/B knob via WG_NVCC_DEFS)
#endif

namespace wg {

constexpr int UQ_THREADS = WG_UQ_THREADS;
// neighbour positions per thread of the flag scan: 1..8, chosen per launch so that small hops
// spread over many SMs (latency-bound) and large hops keep several loads in flight per thread
constexpr int CNT_BITS = 31;                    // packed scan value: (valid << 31) | first
#ifndef WG_PREP_BPS
#define WG_PREP_BPS 8
#endif
constexpr int PREP_BPS = WG_PREP_BPS;           // insert / relabel blocks per SM (full occupancy; A/B via WG_NVCC_DEFS)
constexpr int FLAG_ITEMS_MAX = 8;               // most positions per thread of the flag scan
constexpr int32_t SLOT_EMPTY = -1;              // slot_of: padded slot without a sample
constexpr int32_t SLOT_BADID = -2;              // slot_of: sample whose id is out of range

struct UniqueArgs {
  const int64_t* T;
  int64_t capT;
  const int64_t* d_nT;
  const int64_t* nbrs;     // dense neighbours (standalone) or padded slots (PADDED)
  int64_t capE;            // dense capacity (standalone) or capT * M (PADDED)
  const int64_t* d_nE;     // dense count (standalone) or NULL (PADDED)
  int M;                   // PADDED: fanout
  FastDiv Mdiv;            // PADDED: division by M
  const int32_t* cnt;      // PADDED: per-target sample counts
  const int32_t* pos_pad;  // PADDED: adjacency positions of the padded slots (nullable)
  int64_t* out_row_ptr;    // PADDED: dense CSR row pointer [nT+1]
  int64_t* out_nbrs;       // PADDED: dense neighbours
  int32_t* out_pos;        // PADDED: dense positions (nullable)
  int64_t* d_num_edges;    // PADDED: dense neighbour count
  int64_t* U;
  int64_t* d_nU;
  int32_t* sub_col;
  int32_t* dup;
  int32_t* excl;
  int32_t* slot_of;
  HashTable ht;
  DirectTable dt;          // FMT_DIRECT
  int pad32;               // PADDED: nbrs holds uint32 ids
  unsigned long long* status;
  unsigned* ctrl;
  int64_t n;
};

__device__ __forceinline__ int64_t clamp_count(const int64_t* d, int64_t cap, unsigned* ctrl) {
  if (!d) return cap;
  int64_t v = *d;
  if (v > cap || v < 0) {
    if (threadIdx.x == 0 && blockIdx.x == 0) latch_error(&ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
    v = v < 0 ? 0 : cap;
  }
  return v;
}

// key-table formats (hash.cuh): 16 B hashed slots, 8 B hashed slots, a direct word per node
enum { FMT_WIDE = 0, FMT_COMPACT = 1, FMT_DIRECT = 2 };

template <bool PADDED>
__device__ __forceinline__ void load_counts(const UniqueArgs& a, int64_t& nT, int64_t& nE) {
  nT = clamp_count(a.d_nT, a.capT, a.ctrl);
  nE = PADDED ? nT * a.M : clamp_count(a.d_nE, a.capE, a.ctrl);
}

template <bool PADDED, int FMT>
__global__ void __launch_bounds__(UQ_THREADS) unique_insert_kernel(const UniqueArgs a) {
  pdl_enter();
  int64_t nT, nE;
  load_counts<PADDED>(a, nT, nE);
  const unsigned epoch = a.ctrl[CTRL_EPOCH];
  constexpr bool COMPACT = FMT == FMT_COMPACT;
  if (FMT == FMT_DIRECT) dtab_clear_ahead(a.dt, epoch);  // the idle table (standalone: the op's first kernel)
  const HashTable ht = ht_for_epoch(a.ht, epoch);
  unsigned* const dt = FMT == FMT_DIRECT ? dtab_cur(a.dt, epoch) : nullptr;
  const unsigned tag = FMT == FMT_DIRECT ? dtag(epoch) : 0u;
  const int64_t total = nT + nE;
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (UQ_THREADS / 32);
  for (int64_t base = ((int64_t)blockIdx.x * (UQ_THREADS / 32) + (threadIdx.x >> 5)) * 32; base < total;
       base += warps * 32) {
    const int64_t q = base + lane;
    bool valid = q < total;
    int64_t key = 0;
    if (valid) {
      if (q < nT) {
        key = a.T[q];
      } else if (PADDED) {
        const int64_t j = q - nT;
        const unsigned k = a.Mdiv.div((unsigned)j);
        key = ld_pad(a.nbrs, a.pad32, j);  // loaded together with the count (ignored for a padding slot)
        valid = (int)((unsigned)j - k * (unsigned)a.M) < a.cnt[k];
        if (!valid && FMT != FMT_DIRECT) a.slot_of[q] = SLOT_EMPTY;  // padding slot: no sample here
      } else {
        key = a.nbrs[q - nT];
      }
      if (valid && (key < 0 || key >= a.n)) {
        latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
        if (FMT != FMT_DIRECT) a.slot_of[q] = SLOT_BADID;  // a sample, but no key to number
        valid = false;
      }
    }
    const unsigned long long mk = valid ? (unsigned long long)key : (0x8000000000000000ull | (unsigned)lane);
    const unsigned same = __match_any_sync(FULL_MASK, mk);
    const int leader = __ffs(same) - 1;  // lowest lane = smallest position among equal keys
    const bool is_target = q < nT;
    if (is_target) {  // targets first, original order (L160)
      a.U[q] = key;
      if (a.dup) a.dup[q] = 0;
    }
    // two equal targets in this warp: duplicate target (A8)
    const unsigned tmask = __ballot_sync(FULL_MASK, valid && is_target);
    if (valid && is_target && leader == lane && __popc(same & tmask) > 1)
      latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_DUP_TARGET);
    if (FMT == FMT_DIRECT) {  // no slots: the node's own word; targets check for an earlier target record
      if (valid && leader == lane) {
        if (is_target) {
          const unsigned old = atomicMin(&dt[key], dword(tag, q));
          if ((old >> DPOS_BITS) == tag && (int64_t)(old & DPOS_MASK) < nT)
            latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_DUP_TARGET);
        } else {
          atomicMin(&dt[key], dword(tag, q));
        }
      }
      continue;
    }
    long long slot = -1;
    if (valid && leader == lane) {
      if (COMPACT) {
        unsigned long long old;
        slot = chash_insert(ht, key, q, compact_epoch(epoch), is_target, &old);
        // a target meeting an earlier TARGET record of its key: duplicate target (A8)
        if (is_target && slot >= 0 && old != 0 && (int64_t)(old & CPOS_MASK) < nT)
          latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_DUP_TARGET);
      } else if (is_target) {
        bool dup = false;
        slot = hash_insert_target(ht, key, q, nT, epoch, &dup);
        if (dup) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_DUP_TARGET);
      } else {
        slot = hash_insert_min(ht, key, q, epoch);
      }
      if (slot < 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
    }
    slot = __shfl_sync(FULL_MASK, slot, leader);
    if (valid) a.slot_of[q] = (int32_t)slot;
  }
}

template <int FMT>
__device__ __forceinline__ int64_t min_pos_at(const HashTable& ht, int32_t slot) {
  if (slot < 0) return -1;
  if (FMT == FMT_COMPACT) return chash_min_pos(ht, slot);
  return (int64_t)(ht.slots[slot].val & KEY_MASK);
}

template <bool PADDED, int UQ_ITEMS, int FMT>
__global__ void __launch_bounds__(UQ_THREADS) unique_flag_kernel(const UniqueArgs a) {
  pdl_enter();
  // warp-striped: warp w of the tile covers 32 * UQ_ITEMS consecutive positions, lane l the
  // positions l, l+32, ...; every load and store instruction touches 32 consecutive elements,
  // and the in-warp scans are ballots + popc.
  constexpr int UQ_TILE = UQ_THREADS * UQ_ITEMS;
  __shared__ LookbackSmem<UQ_THREADS> lb;
  __shared__ unsigned long long sm_wtot[UQ_THREADS / 32 + 1];
  __shared__ int sm_flag;
  int64_t nT, nE;
  load_counts<PADDED>(a, nT, nE);
  const unsigned epoch = a.ctrl[CTRL_EPOCH];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const unsigned lt = (1u << lane) - 1u;

  const unsigned* const dt = FMT == FMT_DIRECT ? dtab_cur(a.dt, epoch) : nullptr;
  const unsigned tag = FMT == FMT_DIRECT ? dtag(epoch) : 0u;
  const HashTable ht = ht_for_epoch(a.ht, epoch);
  const int64_t pad_key = a.pad32 ? (int64_t)0xFFFFFFFFu : (int64_t)-1;  // direct: sampler's padding slots
  const int64_t tile_start = (int64_t)blockIdx.x * UQ_TILE;
  if (nE == 0) {
    if (blockIdx.x == 0 && tid == 0) {
      if (a.d_nU) *a.d_nU = nT;
      if (PADDED) {
        a.out_row_ptr[0] = 0;  // nT == 0 here (M >= 1)
        if (a.d_num_edges) *a.d_num_edges = 0;
      }
    }
  } else if (tile_start < nE) {
    const int64_t wbase = tile_start + (int64_t)warp * 32 * UQ_ITEMS + lane;
    int32_t slots[UQ_ITEMS];
    int64_t keys[UQ_ITEMS];
    int32_t poss[UQ_ITEMS];
    int64_t mps[UQ_ITEMS];
    unsigned vm[UQ_ITEMS], fm[UQ_ITEMS];
#pragma unroll
    for (int t = 0; t < UQ_ITEMS; ++t) {
      const int64_t j = wbase + 32 * t;
      const bool in = j < nE;
      // every position's slot (the insert pass wrote SLOT_EMPTY for padding): no count read needed
      if (FMT != FMT_DIRECT) slots[t] = in ? a.slot_of[nT + j] : SLOT_EMPTY;
      keys[t] = in ? (PADDED ? ld_pad(a.nbrs, a.pad32, j) : a.nbrs[j]) : -1;  // needed after the scan: issued now
    }
    unsigned long long wv = 0, wf = 0;
#pragma unroll
    for (int t = 0; t < UQ_ITEMS; ++t) {
      const int64_t j = wbase + 32 * t;
      bool valid;
      if (FMT == FMT_DIRECT) {  // padding slots hold pad_key; the key's own word holds its first position
        valid = j < nE && (!PADDED || keys[t] != pad_key);
        mps[t] = (valid && keys[t] >= 0 && keys[t] < a.n) ? dtab_min_pos(dt, tag, keys[t]) : -1;
      } else {
        valid = j < nE && (!PADDED || slots[t] != SLOT_EMPTY);
        mps[t] = min_pos_at<FMT>(ht, slots[t]);  // independent L2 reads
      }
      poss[t] = (PADDED && a.out_pos && valid) ? a.pos_pad[j] : 0;
      vm[t] = __ballot_sync(FULL_MASK, valid);
    }
#pragma unroll
    for (int t = 0; t < UQ_ITEMS; ++t) {
      const int64_t j = wbase + 32 * t;
      fm[t] = __ballot_sync(FULL_MASK, ((vm[t] >> lane) & 1u) && mps[t] == nT + j);
      wv += __popc(vm[t]);
      wf += __popc(fm[t]);
    }
    unsigned long long agg;
    unsigned long long ex =
        block_exclusive_sum<UQ_THREADS>(lane == 0 ? ((wv << CNT_BITS) | wf) : 0ull, sm_wtot, &agg);
    ex = __shfl_sync(FULL_MASK, ex, 0);  // this warp's offset inside the tile
    const unsigned long long pre = gridDim.x <= WG_LB_DIRECT_MAX
                                       ? block_prefix_direct<UQ_THREADS>(a.status, (long)blockIdx.x, agg, lb)
                                       : block_lookback<UQ_THREADS>(a.status, (long)blockIdx.x, agg, lb);
    const unsigned long long base = pre + ex;
    int64_t ev = (int64_t)(base >> CNT_BITS);                 // dense position of this warp's next valid slot
    int64_t ef = (int64_t)(base & ((1ull << CNT_BITS) - 1));  // next new-node index
#pragma unroll
    for (int t = 0; t < UQ_ITEMS; ++t) {
      const int64_t j = wbase + 32 * t;
      const bool valid = (vm[t] >> lane) & 1u;
      const bool first = (fm[t] >> lane) & 1u;
      const int64_t p = PADDED ? ev + __popc(vm[t] & lt) : j;
      const int64_t f = ef + __popc(fm[t] & lt);
      if (PADDED && j < nE) {
        const unsigned k = a.Mdiv.div((unsigned)j);
        if ((unsigned)j == k * (unsigned)a.M) a.out_row_ptr[k] = p;  // first slot of target k
      }
      if (valid) {
        if (PADDED) {
          a.out_nbrs[p] = keys[t];
          if (a.out_pos) a.out_pos[p] = poss[t];
        }
        a.sub_col[p] = (int32_t)mps[t];  // temporary: min position (relabel turns it into an id)
      }
      if (first) {
        a.U[nT + f] = keys[t];
        if (a.dup) a.dup[nT + f] = 0;
        a.excl[j] = (int32_t)f;
      }
      if (j == nE - 1) {
        if (a.d_nU) *a.d_nU = nT + f + first;
        if (PADDED) {
          a.out_row_ptr[nT] = p + valid;
          if (a.d_num_edges) *a.d_num_edges = p + valid;
        }
      }
      ev += __popc(vm[t]);
      ef += __popc(fm[t]);
    }
  }

  if (finish_block(&a.ctrl[CTRL_DONE_UNIQUE], &sm_flag)) {
    for (int t = tid; t < (int)gridDim.x; t += UQ_THREADS) a.status[t] = 0ull;
    if (tid == 0) {
      a.ctrl[CTRL_DONE_UNIQUE] = 0u;
      // the table is not read again in this call: advance its epoch (the compact table cycles
      // through 255 epochs and is cleared when a cycle restarts; the wide one has 2^23)
      // (the counter wraps modulo 2 * CEPOCHS: compact_epoch and the direct table's parity continue)
      if (FMT != FMT_WIDE)
        a.ctrl[CTRL_EPOCH] =
            epoch + 1u >= 2u * CEPOCHS * 2048u ? (epoch + 1u) % (2u * CEPOCHS) + 2u * CEPOCHS : epoch + 1u;
      else if (epoch + 1u >= EPOCH_MAX)
        latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_EPOCH);
      else
        a.ctrl[CTRL_EPOCH] = epoch + 1u;
    }
  }
}

// sub_col[p] = id of neighbour p; d_nE = the dense neighbour count.
__global__ void __launch_bounds__(UQ_THREADS) unique_relabel_kernel(const UniqueArgs a) {
  pdl_enter();
  const int64_t nT = clamp_count(a.d_nT, a.capT, a.ctrl);
  int64_t nE = a.d_nE ? *a.d_nE : a.capE;
  nE = nE < 0 ? 0 : (nE > a.capE ? a.capE : nE);
  for (int64_t p = (int64_t)blockIdx.x * UQ_THREADS + threadIdx.x; p < nE; p += (int64_t)gridDim.x * UQ_THREADS) {
    const int32_t mp = a.sub_col[p];
    int32_t id = -1;
    if (mp >= 0) id = mp < nT ? mp : (int32_t)nT + a.excl[mp - nT];
    a.sub_col[p] = id;
    if (a.dup && id >= 0) atomicAdd(&a.dup[id], 1);
  }
}

// Compact tables: at the first epoch of a cycle zero the idle one (chash_clear_ahead).  Launched before the
// insert pass of a standalone append-unique; the fused hop does the same inside its sampler.
__global__ void __launch_bounds__(256) hash_clear_kernel(const HashTable t, int64_t words, const unsigned* ctrl) {
  pdl_enter();
  chash_clear_ahead(t, words, ctrl[CTRL_EPOCH]);
}

cudaError_t launch_hash_clear(wg_dsm* h, cudaStream_t st) {
  const HashTable t{h->ws.hslots, 0ull, h->ws.compact, reinterpret_cast<HashSlot*>(h->ws.hslots2)};
  return launch_pdl(hash_clear_kernel, (unsigned)h->sm_count * 4, 256, 0, st, t, (int64_t)h->ws.hcap,
                    (const unsigned*)h->ws.ctrl);
}

template <int FMT>
static cudaError_t launch_insert_flag(wg_dsm* h, bool padded, int items, int64_t ib, unsigned fb, const UniqueArgs& a,
                                      cudaStream_t st) {
  // the fused hop with the direct or the compact table has no insert pass (its sampler inserted every key)
  if (!(padded && hop_inserts_in_sampler(h))) {
    cudaError_t e = padded ? launch_pdl(unique_insert_kernel<true, FMT>, (unsigned)ib, UQ_THREADS, 0, st, a)
                           : launch_pdl(unique_insert_kernel<false, FMT>, (unsigned)ib, UQ_THREADS, 0, st, a);
    if (e != cudaSuccess) return e;
    stage_mark(h, st);
  }
  if (padded) {
    switch (items) {
      case 8: return launch_pdl(unique_flag_kernel<true, 8, FMT>, fb, UQ_THREADS, 0, st, a);
      case 4: return launch_pdl(unique_flag_kernel<true, 4, FMT>, fb, UQ_THREADS, 0, st, a);
      case 2: return launch_pdl(unique_flag_kernel<true, 2, FMT>, fb, UQ_THREADS, 0, st, a);
      default: return launch_pdl(unique_flag_kernel<true, 1, FMT>, fb, UQ_THREADS, 0, st, a);
    }
  }
  switch (items) {
    case 8: return launch_pdl(unique_flag_kernel<false, 8, FMT>, fb, UQ_THREADS, 0, st, a);
    case 4: return launch_pdl(unique_flag_kernel<false, 4, FMT>, fb, UQ_THREADS, 0, st, a);
    case 2: return launch_pdl(unique_flag_kernel<false, 2, FMT>, fb, UQ_THREADS, 0, st, a);
    default: return launch_pdl(unique_flag_kernel<false, 1, FMT>, fb, UQ_THREADS, 0, st, a);
  }
}

static cudaError_t launch_unique_passes(wg_dsm* h, UniqueArgs& a, bool padded, cudaStream_t st, cudaStream_t side) {
  a.excl = h->ws.excl[h->excl_next];
  h->excl_next = (h->excl_next + 1) % EXCL_RING;
  a.slot_of = h->ws.slot_of;
  // Each call uses only a prefix of the table sized for ITS key bound (capT + capE): HASH_FACTOR x bound
  // slots (any size, a multiple of 8 = one 128 B line; at least HASH_MIN_SLOTS), so a hop touches
  // about as many lines as it has keys instead of random lines all over the table sized for the
  // largest hop.  Slots outside the prefix, or left by earlier calls, carry older epochs and read as
  // empty.
  a.ht = HashTable{h->ws.hslots, (unsigned long long)table_prefix(h, a.capT + a.capE), h->ws.compact,
                   reinterpret_cast<HashSlot*>(h->ws.hslots2)};
  a.dt = DirectTable{{h->ws.dtab[0], h->ws.dtab[1]}, h->n};
  a.status = h->ws.status_unique;
  a.ctrl = h->ws.ctrl;
  a.n = h->n;
  const int64_t total = a.capT + a.capE;
  const int64_t max_blocks = (int64_t)h->sm_count * PREP_BPS;
  int64_t ib = (total + UQ_THREADS - 1) / UQ_THREADS;
  ib = ib < 1 ? 1 : (ib > max_blocks ? max_blocks : ib);
  // items per thread: the largest of 8/4/2/1 that still gives >= 2 tiles per SM
  int items = FLAG_ITEMS_MAX;
  while (items > 1 && a.capE < (int64_t)items * UQ_THREADS * 2 * h->sm_count) items >>= 1;
  const int64_t tile = (int64_t)items * UQ_THREADS;
  const unsigned fb = (unsigned)(a.capE > 0 ? (a.capE + tile - 1) / tile : 1);
  cudaError_t e;
  if (!padded && h->ws.compact && !h->ws.direct) {
    e = launch_hash_clear(h, st);
    if (e != cudaSuccess) return e;
  }
  if (h->ws.direct)
    e = launch_insert_flag<FMT_DIRECT>(h, padded, items, ib, fb, a, st);
  else if (h->ws.compact)
    e = launch_insert_flag<FMT_COMPACT>(h, padded, items, ib, fb, a, st);
  else
    e = launch_insert_flag<FMT_WIDE>(h, padded, items, ib, fb, a, st);
  if (e != cudaSuccess) return e;
  stage_mark(h, st);
  if (a.capE > 0) {
    // relabel runs over the DENSE neighbours: count = num_edges (padded) or d_nE
    UniqueArgs r = a;
    if (padded) r.d_nE = a.d_num_edges;
    int64_t rb = (a.capE + UQ_THREADS - 1) / UQ_THREADS;
    rb = rb > max_blocks ? max_blocks : rb;
    cudaStream_t rs = st;
    if (side && side != st) {
      cudaError_t e = cudaEventRecord(h->fork_event, st);
      if (e != cudaSuccess) return e;
      e = cudaStreamWaitEvent(side, h->fork_event, 0);
      if (e != cudaSuccess) return e;
      rs = side;
    }
    unique_relabel_kernel<<<(unsigned)rb, UQ_THREADS, 0, rs>>>(r);
    stage_mark(h, rs);
  }
  return cudaGetLastError();
}

cudaError_t launch_append_unique(wg_dsm* h, const int64_t* T, int64_t capT, const int64_t* d_nT,
                                 const int64_t* nbrs, int64_t capE, const int64_t* d_nE, int64_t* U,
                                 int64_t* d_nU, int32_t* sub_col, int32_t* dup, cudaStream_t st) {
  UniqueArgs a{};
  a.T = T;
  a.capT = capT;
  a.d_nT = d_nT;
  a.nbrs = nbrs;
  a.capE = capE;
  a.d_nE = d_nE;
  a.M = 1;
  a.Mdiv = FastDiv(1u);
  a.U = U;
  a.d_nU = d_nU;
  a.sub_col = sub_col;
  a.dup = dup;
  h->stage_i = 0;
  return launch_unique_passes(h, a, false, st, nullptr);
}

cudaError_t launch_sample_padded(wg_dsm* h, const int64_t* targets, int64_t cap, const int64_t* d_n, int fanout,
                                 uint64_t seed, const uint64_t* d_seed, int hop, bool want_pos, cudaStream_t st,
                                 int64_t* U, int32_t* dup);

cudaError_t launch_hop(wg_dsm* h, const int64_t* T, int64_t capT, const int64_t* d_nT, int fanout, uint64_t seed,
                       const uint64_t* d_seed, int hop, int64_t* out_row_ptr, int64_t* out_nbrs, int32_t* out_pos,
                       int64_t* d_num_edges, int64_t* U, int64_t* d_nU, int32_t* sub_col, int32_t* dup,
                       cudaStream_t st, cudaStream_t side) {
  h->stage_i = 0;
  cudaError_t e = launch_sample_padded(h, T, capT, d_nT, fanout, seed, d_seed, hop, out_pos != nullptr, st, U, dup);
  if (e != cudaSuccess) return e;
  stage_mark(h, st);
  UniqueArgs a{};
  a.T = T;
  a.capT = capT;
  a.d_nT = d_nT;
  a.nbrs = h->ws.nbrs_pad;
  a.pad32 = h->ws.pad32;
  a.capE = capT * fanout;
  a.d_nE = nullptr;
  a.M = fanout;
  a.Mdiv = FastDiv((unsigned)fanout);
  a.cnt = h->ws.cnt;
  a.pos_pad = h->ws.pos_pad;
  a.out_row_ptr = out_row_ptr;
  a.out_nbrs = out_nbrs;
  a.out_pos = out_pos;
  a.d_num_edges = d_num_edges;
  a.U = U;
  a.d_nU = d_nU;
  a.sub_col = sub_col;
  a.dup = dup;
  return launch_unique_passes(h, a, true, st, side);
}

}  // namespace wg
