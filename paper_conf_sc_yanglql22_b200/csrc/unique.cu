// unique.cu -- Append Unique op with first-appearance numbering (A7).
//
// Keys live in the open-addressing hash table of hash.cuh, which stays in L2.
// Instead of the paper's per-bucket count of -1 values (whose order depends on the
// insertion race), every key records the MINIMUM position at which it occurs in
// the concatenated list [targets ; neighbours]; a neighbour position p is a "first
// occurrence" iff that minimum equals nT + p, and the new ids are nT + exclusive
// scan of the first-occurrence flags.  The result is deterministic and equals the
// sequential definition.  Kernels:
//   insert   all nT+nE keys; __match_any_sync elects one lane per distinct key in a
//            warp; CAS claims a slot, atomicMin records the first position; every
//            position remembers its slot (slot_of).  (Fused into the sampler by
//            wg_sample_hop, sample.cu.)
//   flag     single-pass scan over neighbour positions (decoupled look-back): reads
//            the min position through slot_of (one dependent L2 read, no probing),
//            writes U for first occurrences and the scan, and handles the targets
//            (U[k] = T[k], duplicate-target check).  Its last block advances the
//            table epoch.
//   relabel  sub_col[p] = id of nbrs[p]; optional duplicate counts (L186).  Nothing
//            downstream in the batch needs it before the end, so it may run on a
//            side stream.
#include "hash.cuh"

namespace wg {

constexpr int UQ_THREADS = 256;
constexpr int UQ_ITEMS = 4;
constexpr int UQ_TILE = UQ_THREADS * UQ_ITEMS;  // neighbour positions per flag tile

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
  int32_t* slot_of;
  HashTable ht;
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
        a.slot_of[q] = -1;
        valid = false;
      }
    }
    const unsigned long long mk = valid ? (unsigned long long)key : (0x8000000000000000ull | (unsigned)lane);
    const unsigned same = __match_any_sync(FULL_MASK, mk);
    const int leader = __ffs(same) - 1;  // lowest lane = smallest position among equal keys
    long long slot = -1;
    if (valid && leader == lane) {
      slot = hash_insert_min(a.ht, key, q, epoch);
      if (slot < 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
    }
    slot = __shfl_sync(FULL_MASK, slot, leader);
    if (valid) a.slot_of[q] = (int32_t)slot;
  }
}

__device__ __forceinline__ int64_t min_pos_at(const UniqueArgs& a, int32_t slot) {
  if (slot < 0) return -1;
  return (int64_t)(a.ht.vals[slot] & KEY_MASK);
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
    a.U[k] = a.T[k];
    if (a.dup) a.dup[k] = 0;
    const int32_t slot = a.slot_of[k];
    if (slot >= 0 && min_pos_at(a, slot) != k) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_DUP_TARGET);
  }

  const int64_t tile_start = (int64_t)blockIdx.x * UQ_TILE;
  if (nE == 0) {
    if (blockIdx.x == 0 && tid == 0 && a.d_nU) *a.d_nU = nT;
  } else if (tile_start < nE) {
    int32_t slots[UQ_ITEMS];
    int64_t mps[UQ_ITEMS];
    const int64_t p0 = tile_start + (int64_t)tid * UQ_ITEMS;
    // coalesced 16-byte read of this thread's 4 slots when aligned (p0 is a multiple of 4)
    if (p0 + UQ_ITEMS <= nE && (nT & 3) == 0) {
      const int4 s4 = *reinterpret_cast<const int4*>(a.slot_of + nT + p0);
      slots[0] = s4.x; slots[1] = s4.y; slots[2] = s4.z; slots[3] = s4.w;
    } else {
#pragma unroll
      for (int j = 0; j < UQ_ITEMS; ++j) slots[j] = (p0 + j < nE) ? a.slot_of[nT + p0 + j] : -1;
    }
#pragma unroll
    for (int j = 0; j < UQ_ITEMS; ++j) mps[j] = min_pos_at(a, slots[j]);  // independent L2 reads
    int cnt = 0;
    int first[UQ_ITEMS];
#pragma unroll
    for (int j = 0; j < UQ_ITEMS; ++j) {
      const int64_t p = p0 + j;
      first[j] = (p < nE) && (mps[j] == nT + p);
      if (p < nE) {
        a.sub_col[p] = (int32_t)mps[j];  // temporary: min position (relabel turns it into an id)
        if (a.dup) a.dup[nT + p] = 0;
      }
      cnt += first[j];
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
      const int64_t p = p0 + j;
      if (p < nE) {
        a.excl[p] = (int32_t)run;
        if (first[j]) a.U[nT + run] = a.nbrs[p];
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
                                 int64_t* d_nU, int32_t* sub_col, int32_t* dup, bool inserted, cudaStream_t st,
                                 cudaStream_t side) {
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
  a.excl = h->ws.excl[h->excl_next];
  h->excl_next = (h->excl_next + 1) % EXCL_RING;
  a.slot_of = h->ws.slot_of;
  a.ht = HashTable{h->ws.hkeys, h->ws.hvals, (unsigned long long)h->ws.hcap - 1};
  a.status = h->ws.status_unique;
  a.ctrl = h->ws.ctrl;
  a.n = h->n;
  const int64_t total = capT + capE;
  const int64_t max_blocks = (int64_t)h->sm_count * 8;
  if (!inserted) {
    int64_t ib = (total + UQ_THREADS - 1) / UQ_THREADS;
    ib = ib < 1 ? 1 : (ib > max_blocks ? max_blocks : ib);
    unique_insert_kernel<<<(unsigned)ib, UQ_THREADS, 0, st>>>(a);
  }
  int64_t fb = capE > 0 ? (capE + UQ_TILE - 1) / UQ_TILE : 1;
  unique_flag_kernel<<<(unsigned)fb, UQ_THREADS, 0, st>>>(a);
  if (capE > 0) {
    int64_t rb = (capE + UQ_THREADS - 1) / UQ_THREADS;
    rb = rb > max_blocks ? max_blocks : rb;
    cudaStream_t rs = st;
    if (side && side != st) {
      cudaError_t e = cudaEventRecord(h->fork_event, st);
      if (e != cudaSuccess) return e;
      e = cudaStreamWaitEvent(side, h->fork_event, 0);
      if (e != cudaSuccess) return e;
      rs = side;
    }
    unique_relabel_kernel<<<(unsigned)rb, UQ_THREADS, 0, rs>>>(a);
  }
  return cudaGetLastError();
}

}  // namespace wg
