// unique.cu -- Append Unique op with first-appearance numbering (A7).
//
// Keys live in an open-addressing hash table (the paper's "GPU hash table ... key
// is nodeID", L160-166; Warpcore-style insertion [33]) that stays in L2.  Instead
// of the paper's per-bucket count of -1 values (whose order depends on the
// insertion race), every key records the MINIMUM position at which it occurs in
// the concatenated list [targets ; neighbours]; a neighbour position p is a "first
// occurrence" iff that minimum equals nT + p, and the new ids are nT + exclusive
// scan of the first-occurrence flags.  The result is deterministic and equals the
// sequential definition.  Three kernels:
//   insert   all nT+nE keys; __match_any_sync elects one lane per distinct key in a
//            warp; CAS claims a slot, atomicMin records the first position.
//   flag     single-pass scan over neighbour positions (decoupled look-back): looks
//            up the min position, writes U for first occurrences, the scan, and
//            handles the targets (U[k] = T[k], duplicate-target check).  Its last
//            block advances the table epoch.
//   relabel  sub_col[p] = id of nbrs[p]; optional duplicate counts (L186).
// The table is never cleared: keys carry an epoch tag (bits 40..62) and stale slots
// read as empty, so no per-call memset is needed.
#include "device_util.cuh"
#include "wg_internal.cuh"

namespace wg {

constexpr int UQ_THREADS = 256;
constexpr int UQ_ITEMS = 4;
constexpr int UQ_TILE = UQ_THREADS * UQ_ITEMS;  // neighbour positions per flag tile
constexpr unsigned long long KEY_MASK = (1ull << 40) - 1;

struct UniqueArgs {
  const int64_t* T;
  int64_t capT;
  const int64_t* d_nT;
  const int64_t* nbrs;
  int64_t capE;
  const int64_t* d_nE;
  int64_t* U;
  int64_t* d_nU;
  int32_t* sub_col;
  int32_t* dup;
  int32_t* excl;
  unsigned long long* hkeys;
  unsigned long long* hvals;
  unsigned long long hmask;
  unsigned long long* status;
  unsigned* ctrl;
  int64_t n;
};

__device__ __forceinline__ void load_counts(const UniqueArgs& a, int64_t& nT, int64_t& nE) {
  nT = a.capT;
  nE = a.capE;
  if (a.d_nT) {
    nT = *a.d_nT;
    if (nT > a.capT || nT < 0) {
      if (threadIdx.x == 0 && blockIdx.x == 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
      nT = nT < 0 ? 0 : a.capT;
    }
  }
  if (a.d_nE) {
    nE = *a.d_nE;
    if (nE > a.capE || nE < 0) {
      if (threadIdx.x == 0 && blockIdx.x == 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
      nE = nE < 0 ? 0 : a.capE;
    }
  }
}

// Returns the slot holding `stored` (claiming an empty one if needed), or -1 if full.
__device__ __forceinline__ long long hash_insert(const UniqueArgs& a, unsigned long long stored,
                                                 unsigned epoch) {
  unsigned long long slot = fmix64(stored & KEY_MASK) & a.hmask;
  for (unsigned long long probe = 0; probe <= a.hmask; ++probe) {
    unsigned long long cur = ld_volatile_u64(&a.hkeys[slot]);
    for (;;) {
      if (cur == stored) return (long long)slot;
      if ((unsigned)(cur >> 40) == epoch) break;  // occupied by another key this epoch
      const unsigned long long prev = atomicCAS(&a.hkeys[slot], cur, stored);
      if (prev == cur || prev == stored) return (long long)slot;
      cur = prev;
    }
    slot = (slot + 1) & a.hmask;
  }
  return -1;
}

__device__ __forceinline__ long long hash_find(const UniqueArgs& a, unsigned long long stored, unsigned epoch) {
  unsigned long long slot = fmix64(stored & KEY_MASK) & a.hmask;
  for (unsigned long long probe = 0; probe <= a.hmask; ++probe) {
    const unsigned long long cur = a.hkeys[slot];
    if (cur == stored) return (long long)slot;
    if ((unsigned)(cur >> 40) != epoch) return -1;  // empty: not present
    slot = (slot + 1) & a.hmask;
  }
  return -1;
}

__device__ __forceinline__ unsigned long long pack_pos(unsigned epoch, int64_t q) {
  return ((unsigned long long)(EPOCH_MAX - epoch) << 40) | (unsigned long long)q;
}

__global__ void __launch_bounds__(UQ_THREADS) unique_insert_kernel(const UniqueArgs a) {
  int64_t nT, nE;
  load_counts(a, nT, nE);
  const unsigned epoch = a.ctrl[CTRL_EPOCH];
  const int64_t total = nT + nE;
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (UQ_THREADS / 32);
  for (int64_t base = ((int64_t)blockIdx.x * (UQ_THREADS / 32) + (threadIdx.x >> 5)) * 32; base < total;
       base += warps * 32) {
    const int64_t q = base + lane;
    bool valid = q < total;
    int64_t key = 0;
    if (valid) {
      key = q < nT ? a.T[q] : a.nbrs[q - nT];
      if (key < 0 || key >= a.n) {
        latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
        valid = false;
      }
    }
    const unsigned long long mk = valid ? (unsigned long long)key : (0x8000000000000000ull | (unsigned)lane);
    const unsigned same = __match_any_sync(FULL_MASK, mk);
    // the lowest lane of each group of equal keys holds the smallest position
    if (valid && (same & ((1u << lane) - 1u)) == 0u) {
      const unsigned long long stored = ((unsigned long long)epoch << 40) | (unsigned long long)key;
      const long long slot = hash_insert(a, stored, epoch);
      if (slot < 0)
        latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
      else
        atomicMin(&a.hvals[slot], pack_pos(epoch, q));
    }
  }
}

__device__ __forceinline__ int64_t min_pos_of(const UniqueArgs& a, int64_t key, unsigned epoch) {
  const unsigned long long stored = ((unsigned long long)epoch << 40) | (unsigned long long)key;
  const long long slot = hash_find(a, stored, epoch);
  if (slot < 0) return -1;
  return (int64_t)(a.hvals[slot] & KEY_MASK);
}

__global__ void __launch_bounds__(UQ_THREADS) unique_flag_kernel(const UniqueArgs a) {
  __shared__ int sm_wtot[UQ_THREADS / 32 + 1];
  __shared__ unsigned long long sm_prefix;
  __shared__ int sm_flag;
  int64_t nT, nE;
  load_counts(a, nT, nE);
  const unsigned epoch = a.ctrl[CTRL_EPOCH];
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;

  // targets: U[k] = T[k] (targets first, original order, L160); duplicate check (A8)
  for (int64_t k = (int64_t)blockIdx.x * UQ_THREADS + tid; k < nT; k += (int64_t)gridDim.x * UQ_THREADS) {
    const int64_t key = a.T[k];
    a.U[k] = key;
    if (a.dup) a.dup[k] = 0;
    if (key >= 0 && key < a.n) {
      const int64_t mp = min_pos_of(a, key, epoch);
      if (mp != k) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_DUP_TARGET);
    }
  }

  const int64_t tile_start = (int64_t)blockIdx.x * UQ_TILE;
  if (nE == 0) {
    if (blockIdx.x == 0 && tid == 0 && a.d_nU) *a.d_nU = nT;
  } else if (tile_start < nE) {
    int64_t keys[UQ_ITEMS];
    int first[UQ_ITEMS];
    int cnt = 0;
#pragma unroll
    for (int j = 0; j < UQ_ITEMS; ++j) {
      const int64_t p = tile_start + (int64_t)tid * UQ_ITEMS + j;
      first[j] = 0;
      keys[j] = -1;
      if (p < nE) {
        const int64_t key = a.nbrs[p];
        keys[j] = key;
        int64_t mp = -1;
        if (key >= 0 && key < a.n) mp = min_pos_of(a, key, epoch);
        if (mp < 0 && key >= 0 && key < a.n) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
        first[j] = (mp == nT + p);
        a.sub_col[p] = (int32_t)mp;  // temporary: min position (relabel turns it into an id)
        if (a.dup) a.dup[nT + p] = 0;
        cnt += first[j];
      }
    }
    int agg;
    const int ex = block_exclusive_sum<UQ_THREADS>(cnt, sm_wtot, &agg);
    if (warp == 0) {
      const unsigned long long pre = tile_lookback(a.status, (long)blockIdx.x, (unsigned long long)agg);
      if (lane == 0) sm_prefix = pre;
    }
    __syncthreads();
    int64_t run = (int64_t)sm_prefix + ex;
#pragma unroll
    for (int j = 0; j < UQ_ITEMS; ++j) {
      const int64_t p = tile_start + (int64_t)tid * UQ_ITEMS + j;
      if (p < nE) {
        a.excl[p] = (int32_t)run;
        if (first[j]) a.U[nT + run] = keys[j];
        run += first[j];
        if (p == nE - 1 && a.d_nU) *a.d_nU = nT + run;
      }
    }
  }

  if (finish_block(&a.ctrl[CTRL_DONE_UNIQUE], &sm_flag)) {
    for (int t = tid; t < (int)gridDim.x; t += UQ_THREADS) a.status[t] = 0ull;
    if (tid == 0) {
      a.ctrl[CTRL_DONE_UNIQUE] = 0u;
      // the table is not read again in this call: advance its epoch
      if (epoch + 1u >= EPOCH_MAX)
        latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_EPOCH);
      else
        a.ctrl[CTRL_EPOCH] = epoch + 1u;
    }
  }
}

__global__ void __launch_bounds__(UQ_THREADS) unique_relabel_kernel(const UniqueArgs a) {
  int64_t nT, nE;
  load_counts(a, nT, nE);
  for (int64_t p = (int64_t)blockIdx.x * UQ_THREADS + threadIdx.x; p < nE; p += (int64_t)gridDim.x * UQ_THREADS) {
    const int32_t mp = a.sub_col[p];
    int32_t id = -1;
    if (mp >= 0) id = mp < nT ? mp : (int32_t)nT + a.excl[mp - nT];
    a.sub_col[p] = id;
    if (a.dup && id >= 0) atomicAdd(&a.dup[id], 1);
  }
}

cudaError_t launch_append_unique(wg_dsm* h, const int64_t* T, int64_t capT, const int64_t* d_nT,
                                 const int64_t* nbrs, int64_t capE, const int64_t* d_nE, int64_t* U,
                                 int64_t* d_nU, int32_t* sub_col, int32_t* dup, cudaStream_t st) {
  UniqueArgs a;
  a.T = T;
  a.capT = capT;
  a.d_nT = d_nT;
  a.nbrs = nbrs;
  a.capE = capE;
  a.d_nE = d_nE;
  a.U = U;
  a.d_nU = d_nU;
  a.sub_col = sub_col;
  a.dup = dup;
  a.excl = h->ws.excl;
  a.hkeys = h->ws.hkeys;
  a.hvals = h->ws.hvals;
  a.hmask = (unsigned long long)h->ws.hcap - 1;
  a.status = h->ws.status_unique;
  a.ctrl = h->ws.ctrl;
  a.n = h->n;
  const int64_t total = capT + capE;
  const int64_t max_blocks = (int64_t)h->sm_count * 8;
  int64_t ib = (total + UQ_THREADS - 1) / UQ_THREADS;
  ib = ib < 1 ? 1 : (ib > max_blocks ? max_blocks : ib);
  unique_insert_kernel<<<(unsigned)ib, UQ_THREADS, 0, st>>>(a);
  int64_t fb = capE > 0 ? (capE + UQ_TILE - 1) / UQ_TILE : 1;
  unique_flag_kernel<<<(unsigned)fb, UQ_THREADS, 0, st>>>(a);
  if (capE > 0) {
    int64_t rb = (capE + UQ_THREADS - 1) / UQ_THREADS;
    rb = rb > max_blocks ? max_blocks : rb;
    unique_relabel_kernel<<<(unsigned)rb, UQ_THREADS, 0, st>>>(a);
  }
  return cudaGetLastError();
}

}  // namespace wg
