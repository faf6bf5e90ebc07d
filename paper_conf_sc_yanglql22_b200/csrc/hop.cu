// hop.cu -- one whole hop of mini-batch preparation (sampling, then Append Unique)
// as ONE single-pass kernel (fanout <= 32), for wg_sample_hop.
//
// Why.  Every step of the hop is a chain of dependent random accesses (row_ptr -> col_idx, key ->
// slot -> CAS, slot -> first position), and on B200 each step costs an L2 round trip (~185 ns) whether
// the line is in L2 or HBM (profiles/r02/ab_log.md).  Run as separate kernels (sample | insert | scan)
// the hop pays every kernel's ramp and drain and the SMs idle at each boundary; here the phases of
// different tiles overlap instead.
//
// How.  The key list of the hop is [targets ; padded neighbour slots k*M + i] (positions as in
// unique.cu).  It is cut into tiles processed in a single tile order, taken from an atomic counter
// (so every lower tile is already owned by a running block: no deadlock at any occupancy):
//   target tiles     (1024 targets each)  insert the targets (value = index, L160; duplicates latch
//                                         WG_DEVERR_DUP_TARGET, A8) and copy them to U;
//   neighbour tiles  (TB targets each)    sample their targets with the warp sampler (sample_warp.cuh,
//                                         Algorithm 1) into shared memory, insert every sampled id with its
//                                         position (atomicMin keeps the first, A7), then
//     wait until every LOWER tile has finished inserting (decoupled look-back on a done flag) -- from
//        then on the table holds, for each key of this tile, the minimum over ALL positions <= this
//        tile's, so "position p is the key's first occurrence" is final (later tiles only add larger
//        positions); then
//     scan the (valid, first) counts with a second decoupled look-back and write the dense CSR
//        (row_ptr, neighbours, positions), the new unique nodes U[nT + f] (first-appearance numbering)
//        and, per position, the first position of its key (relabelled into sub-graph ids by
//        unique_relabel_kernel, off the critical path).
// Results are those of sample_kernel + unique_insert_kernel + unique_flag_kernel<PADDED> (the same
// device code paths for the draws, the table and the numbering), bit for bit.
#include "hash.cuh"
#include "sample_warp.cuh"
#include "scan.cuh"

namespace wg {

constexpr int HOP_THREADS = 256;
constexpr int HOP_WARPS = HOP_THREADS / 32;
constexpr int HOP_TARGET_TILE = HOP_THREADS * 4;  // targets per target tile
constexpr int HOP_MAX_POS = 1024;                 // padded positions per neighbour tile (TB * M <= 8 * 32 * 4)
constexpr int HOP_ITEMS = HOP_MAX_POS / HOP_THREADS;  // positions per lane (warp-striped)
constexpr int HOP_CNT_BITS = 31;                  // packed scan value: (valid << 31) | first
#ifndef HOP_MINB
#define HOP_MINB 6
#endif

struct HopArgs {
  ShardView s;
  const int64_t* T;
  int64_t capT;
  const int64_t* d_nT;
  int M;
  int hop;
  int TB;                  // targets per neighbour tile (8 * TPW * UNR)
  unsigned long long seed;
  const unsigned long long* d_seed;
  int64_t* out_row_ptr;
  int64_t* out_nbrs;
  int32_t* out_pos;        // nullable
  int64_t* d_num_edges;
  int64_t* U;
  int64_t* d_nU;           // nullable
  int32_t* sub_col;        // first position of each edge's key (relabelled later)
  int32_t* dup;            // nullable: zeroed for every unique node
  int32_t* excl;           // [padded neighbour slot] new-node index of a first occurrence
  HashTable ht;
  unsigned long long* status_ins;
  unsigned long long* status_scan;
  unsigned* ctrl;
};

__device__ __forceinline__ unsigned long long ld_cg_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.global.cg.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}

// first position recorded for the key of `slot` (-1: no key), read past L1 (other blocks updated it)
template <bool COMPACT>
__device__ __forceinline__ int64_t min_pos_cg(const HashTable& t, long long slot) {
  if (slot < 0) return -1;
  if (COMPACT) return (int64_t)(ld_cg_u64(reinterpret_cast<const unsigned long long*>(t.slots) + slot) & CPOS_MASK);
  return (int64_t)(ld_cg_u64(&t.slots[slot].val) & KEY_MASK);
}

// Warp-collective insert of one key per lane (valid lanes only), as unique_insert_kernel: one leader per
// distinct key (__match_any_sync: the lowest lane = the smallest position), CAS claim / atomicMin.
// Returns the key's slot in every valid lane (-1 if the table is full).
template <bool COMPACT>
__device__ __forceinline__ long long insert_warp(const HopArgs& a, bool valid, bool is_target, int64_t key, int64_t q,
                                                 int64_t nT, unsigned epoch) {
  const int lane = threadIdx.x & 31;
  const unsigned long long mk = valid ? (unsigned long long)key : (0x8000000000000000ull | (unsigned)lane);
  const unsigned same = __match_any_sync(FULL_MASK, mk);
  const int leader = __ffs(same) - 1;
  const unsigned tmask = __ballot_sync(FULL_MASK, valid && is_target);
  if (valid && is_target && leader == lane && __popc(same & tmask) > 1)  // two equal targets in a warp (A8)
    latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_DUP_TARGET);
  long long slot = -1;
  if (valid && leader == lane) {
    if (COMPACT) {
      unsigned long long old;
      slot = chash_insert(a.ht, key, q, compact_epoch(epoch), is_target, &old);
      if (is_target && slot >= 0 && old != 0 && (int64_t)(old & CPOS_MASK) < nT)
        latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_DUP_TARGET);
    } else if (is_target) {
      bool dup = false;
      slot = hash_insert_target(a.ht, key, q, nT, epoch, &dup);
      if (dup) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_DUP_TARGET);
    } else {
      slot = hash_insert_min(a.ht, key, q, epoch);
    }
    if (slot < 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
  }
  return __shfl_sync(FULL_MASK, slot, leader);
}

template <int UNR, bool COMPACT>
__global__ void __launch_bounds__(HOP_THREADS, HOP_MINB) hop_fused_kernel(const HopArgs a) {
  pdl_enter();
  __shared__ int64_t s_key[HOP_MAX_POS];
  __shared__ int32_t s_pos[HOP_MAX_POS];
  __shared__ int32_t s_cnt[HOP_MAX_POS / 4];
  __shared__ unsigned s_chain[HOP_WARPS][32];
  __shared__ LookbackSmem<HOP_THREADS> lb;
  __shared__ unsigned long long s_wc[HOP_ITEMS * HOP_WARPS + 1];  // (round, warp) counts, then their scan
  __shared__ int s_tile, s_flag;
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  const unsigned lt = (1u << lane) - 1u;

  int64_t nT = a.capT;
  if (a.d_nT) {
    nT = *a.d_nT;
    if (nT > a.capT || nT < 0) {
      if (tid == 0 && blockIdx.x == 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
      nT = nT < 0 ? 0 : a.capT;
    }
  }
  const unsigned epoch = a.ctrl[CTRL_EPOCH];
  const int M = a.M;
  const int TB = a.TB;
  const int64_t ntt = (nT + HOP_TARGET_TILE - 1) / HOP_TARGET_TILE;  // target tiles
  const int64_t nbt = (nT + TB - 1) / TB;                            // neighbour tiles
  const int64_t nE = nT * M;                                         // padded neighbour slots
  if (tid == 0) s_tile = (int)atomicAdd(&a.ctrl[CTRL_TILE], 1u);
  __syncthreads();
  const int64_t t = s_tile;

  if (t == 0 && nT == 0 && tid == 0) {  // empty hop: counts only
    if (a.d_nU) *a.d_nU = 0;
    a.out_row_ptr[0] = 0;
    *a.d_num_edges = 0;
  }
  if (t < ntt) {
    // ---------------------------------------------------------------- target tile
#pragma unroll
    for (int it = 0; it < 4; ++it) {
      const int64_t q = t * HOP_TARGET_TILE + it * HOP_THREADS + tid;  // block-striped
      bool valid = q < nT;
      int64_t key = 0;
      if (valid) {
        key = a.T[q];
        a.U[q] = key;  // targets first, original order (L160)
        if (a.dup) a.dup[q] = 0;
        if (key < 0 || key >= a.s.n) {
          latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
          valid = false;
        }
      }
      insert_warp<COMPACT>(a, valid, true, key, q, nT, epoch);
    }
    __syncthreads();
    if (tid == 0) __threadfence();  // this tile's table updates are visible before it reports "inserted"
    block_lookback<HOP_THREADS>(a.status_ins, (long)t, 1ull, lb);
  } else if (t < ntt + nbt) {
    // ---------------------------------------------------------------- neighbour tile
    const int64_t j = t - ntt;
    const int64_t k0 = j * TB;                                  // first target of the tile
    const int tcount = (int)min((int64_t)TB, nT - k0);          // targets in the tile
    const int npos = tcount * M;                                // padded positions in the tile
    const int TPW = 32 / sample_group(M);
    const unsigned long long seed = a.d_seed ? *a.d_seed : a.seed;
    const uint2 key2 = make_uint2((unsigned)(seed & 0xffffffffu), (unsigned)(seed >> 32));
    // (1) sample the tile's targets into shared memory (padded slots (k - k0) * M + i)
    sample_warp<UNR>(
        a.s, a.T, k0 + tcount, M, a.hop, key2, k0 + (int64_t)warp * TPW * UNR, s_chain[warp], &a.ctrl[CTRL_ERR],
        [&](int64_t k, int c) { s_cnt[k - k0] = c; },
        [&](int64_t k, int i, int64_t nb, unsigned pos) {
          s_key[(k - k0) * M + i] = nb;
          s_pos[(k - k0) * M + i] = (int32_t)pos;
        });
    __syncthreads();
    // (2) insert every sampled id with its key-list position nT + padded slot; positions are block-striped
    //     (pl = it * 256 + tid), so every warp works even in a small tile
    long long slot[HOP_ITEMS];
    bool sampled[HOP_ITEMS];
#pragma unroll
    for (int it = 0; it < HOP_ITEMS; ++it) {
      const int pl = it * HOP_THREADS + tid;
      const bool in = pl < npos;
      const int kl = in ? pl / M : 0;
      sampled[it] = in && pl - kl * M < s_cnt[kl];
      const int64_t key = sampled[it] ? s_key[pl] : 0;
      bool valid = sampled[it];
      if (valid && (key < 0 || key >= a.s.n)) {
        latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
        valid = false;  // a sample, but no key to number (its edge keeps first position -1)
      }
      slot[it] = insert_warp<COMPACT>(a, valid, false, key, nT + k0 * M + pl, nT, epoch);
      if (!valid) slot[it] = -1;
    }
    __syncthreads();
    if (tid == 0) __threadfence();
    // (3) every lower tile has inserted: first occurrences of this tile's keys are final
    block_lookback<HOP_THREADS>(a.status_ins, (long)t, 1ull, lb);
    __threadfence();  // acquire: the lower tiles' table updates are visible to the reads below
    int64_t mps[HOP_ITEMS];
    unsigned vm[HOP_ITEMS], fm[HOP_ITEMS];
#pragma unroll
    for (int it = 0; it < HOP_ITEMS; ++it) mps[it] = min_pos_cg<COMPACT>(a.ht, slot[it]);  // independent L2 reads
#pragma unroll
    for (int it = 0; it < HOP_ITEMS; ++it) {
      const int pl = it * HOP_THREADS + tid;
      vm[it] = __ballot_sync(FULL_MASK, sampled[it]);
      fm[it] = __ballot_sync(FULL_MASK, sampled[it] && mps[it] == nT + k0 * M + pl);
      if (lane == 0) s_wc[it * HOP_WARPS + warp] = ((unsigned long long)__popc(vm[it]) << HOP_CNT_BITS) | __popc(fm[it]);
    }
    // (4) scan of the (valid, first) counts: within the tile over the 32 (round, warp) groups in position
    //     order, across the neighbour tiles with a decoupled look-back
    __syncthreads();
    if (warp == 0) {
      const unsigned long long v = s_wc[lane];
      const unsigned long long inc = warp_inclusive_sum(v, lane);
      s_wc[lane] = inc - v;
      if (lane == 31) s_wc[32] = inc;
    }
    __syncthreads();
    const unsigned long long pre = block_lookback<HOP_THREADS>(a.status_scan, (long)j, s_wc[32], lb);
#pragma unroll
    for (int it = 0; it < HOP_ITEMS; ++it) {
      const int pl = it * HOP_THREADS + tid;
      const int64_t jp = k0 * M + pl;  // padded neighbour slot (global)
      const bool valid = (vm[it] >> lane) & 1u;
      const bool first = (fm[it] >> lane) & 1u;
      const unsigned long long base = pre + s_wc[it * HOP_WARPS + warp];
      const int64_t p = (int64_t)(base >> HOP_CNT_BITS) + __popc(vm[it] & lt);
      const int64_t f = (int64_t)(base & ((1ull << HOP_CNT_BITS) - 1)) + __popc(fm[it] & lt);
      if (pl < npos && pl % M == 0) a.out_row_ptr[k0 + pl / M] = p;  // first slot of its target
      if (valid) {
        const int64_t key = s_key[pl];
        a.out_nbrs[p] = key;
        if (a.out_pos) a.out_pos[p] = s_pos[pl];
        a.sub_col[p] = (int32_t)mps[it];  // the key's first position (the relabel turns it into an id)
        if (first) {
          a.U[nT + f] = key;
          if (a.dup) a.dup[nT + f] = 0;
          a.excl[jp] = (int32_t)f;
        }
      }
      if (pl < npos && jp == nE - 1) {  // the hop's last padded slot: totals (lanes past npos alias the next tile)
        if (a.d_nU) *a.d_nU = nT + f + first;
        a.out_row_ptr[nT] = p + valid;
        *a.d_num_edges = p + valid;
      }
    }
  }

  if (finish_block(&a.ctrl[CTRL_DONE_HOP], &s_flag)) {
    for (int i = tid; i < (int)gridDim.x; i += HOP_THREADS) {
      a.status_ins[i] = 0ull;
      a.status_scan[i] = 0ull;
    }
    if (tid == 0) {
      a.ctrl[CTRL_TILE] = 0u;
      a.ctrl[CTRL_DONE_HOP] = 0u;
      // the table is not read again in this call: advance its epoch (as unique_flag_kernel)
      if (COMPACT)
        a.ctrl[CTRL_EPOCH] = epoch + 1u >= CEPOCHS * 4096u ? (epoch + 1u) % CEPOCHS + CEPOCHS : epoch + 1u;
      else if (epoch + 1u >= EPOCH_MAX)
        latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_EPOCH);
      else
        a.ctrl[CTRL_EPOCH] = epoch + 1u;
    }
  }
}

cudaError_t launch_hash_clear(wg_dsm* h, cudaStream_t st);
cudaError_t launch_relabel(wg_dsm* h, const int64_t* d_nT, int64_t capT, const int64_t* d_nE, int64_t capE,
                           int32_t* sub_col, int32_t* dup, const int32_t* excl, cudaStream_t st, cudaStream_t side);

template <bool COMPACT>
static cudaError_t launch_fused(int unr, unsigned grid, const HopArgs& a, cudaStream_t st) {
  if (unr == 4) return launch_pdl(hop_fused_kernel<4, COMPACT>, grid, HOP_THREADS, 0, st, a);
  if (unr == 2) return launch_pdl(hop_fused_kernel<2, COMPACT>, grid, HOP_THREADS, 0, st, a);
  return launch_pdl(hop_fused_kernel<1, COMPACT>, grid, HOP_THREADS, 0, st, a);
}

cudaError_t launch_hop_fused(wg_dsm* h, const int64_t* T, int64_t capT, const int64_t* d_nT, int fanout,
                             uint64_t seed, const uint64_t* d_seed, int hop, int64_t* out_row_ptr, int64_t* out_nbrs,
                             int32_t* out_pos, int64_t* d_num_edges, int64_t* U, int64_t* d_nU, int32_t* sub_col,
                             int32_t* dup, cudaStream_t st, cudaStream_t side) {
  h->stage_i = 0;
  HopArgs a{};
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
  a.excl = h->ws.excl[h->excl_next];
  h->excl_next = (h->excl_next + 1) % EXCL_RING;
  a.ht = HashTable{h->ws.hslots, (unsigned long long)table_prefix(h, capT + capT * (int64_t)fanout), h->ws.compact};
  a.status_ins = h->ws.status_sample;
  a.status_scan = h->ws.status_unique;
  a.ctrl = h->ws.ctrl;
  // rounds per warp: the largest of 4/2/1 that still gives >= 2 neighbour tiles per SM
  const int tpw = 32 / sample_group(fanout);
  int unr = SAMPLE_UNR_MAX;
  while (unr > 1 && capT < (int64_t)HOP_WARPS * tpw * unr * 2 * h->sm_count) unr >>= 1;
  a.TB = HOP_WARPS * tpw * unr;
  const int64_t tiles = (capT + HOP_TARGET_TILE - 1) / HOP_TARGET_TILE + (capT + a.TB - 1) / a.TB;
  const unsigned grid = (unsigned)(tiles > 0 ? tiles : 1);
  cudaError_t e = cudaSuccess;
  if (h->ws.compact) e = launch_hash_clear(h, st);  // zero the compact table when its epoch cycle restarts
  if (e != cudaSuccess) return e;
  stage_mark(h, st);
  e = h->ws.compact ? launch_fused<true>(unr, grid, a, st) : launch_fused<false>(unr, grid, a, st);
  if (e != cudaSuccess) return e;
  stage_mark(h, st);
  // sub-graph ids of the edges (and duplicate counts): nothing else in the batch waits for them
  return launch_relabel(h, d_nT, capT, d_num_edges, capT * fanout, sub_col, dup, a.excl, st, side);
}

}  // namespace wg
