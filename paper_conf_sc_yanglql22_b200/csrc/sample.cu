// sample.cu -- multi-GPU sampling op (Algorithm 1).
//
// One single-pass kernel per hop.  A block owns a tile of 32..128 targets (sample_tile):
//   count phase   one thread per target loads the (row_ptr[l], row_ptr[l+1]) pair
//                 from the owner's shard (local HBM or a peer over NVLink), computes
//                 cnt = min(M, deg), block-scans it and resolves the tile's global
//                 offset by decoupled look-back (no second pass, no host sync);
//   sample phase  a group of G lanes (G = next power of two >= M, 8..32) handles one
//                 target.  If M >= N every lane i < N copies col[start+i] (L118).
//                 Otherwise lane i draws r_i (Philox, reading A3) and computes
//                 Algorithm 1's res[i] WITHOUT the sort: __match_any_sync on r
//                 gives, per lane, the previous draw with the same value (the
//                 p[q[i]-1] of Alg.1 line 8) and whether it is the last one (the
//                 run-end test of line 4); the chain of line 5 lives in 32 words of
//                 shared memory per warp, path doubling (line 12) is log2(M)
//                 __shfl_sync rounds and last (line 7) a subtraction.  The result
//                 equals Algorithm 1 for every draw vector (it is the same
//                 sequential Fisher-Yates function).
//                 Lane i then loads col[start + res_i] (local or peer) and writes
//                 it at out_nbrs[offset + i], in draw order (A5).  Each warp works
//                 on UNR rounds at once so UNR independent neighbour loads are in
//                 flight per lane (the loads are latency-bound random 8 B reads).
// FUSED = true additionally performs the insert pass of Append Unique (unique.cu)
// in the same kernel: targets are inserted in the count phase (position k) and each
// sampled neighbour right after its load (position nT + p), so a whole hop needs
// only this kernel, the flag scan and the (off-critical-path) relabel.
#include "hash.cuh"

namespace wg {

constexpr int SAMPLE_THREADS = 256;
constexpr int SAMPLE_UNR = 4;  // rounds per warp, all in flight at once
// targets per block: (SAMPLE_THREADS / G) targets per round x SAMPLE_UNR rounds, i.e. 128 / 64 / 32 for
// G = 8 / 16 / 32.  Small tiles spread even a 1024-target hop over many SMs (the kernel is latency-bound)
// and leave each lane exactly one round of SAMPLE_UNR independent neighbour loads.
template <int G>
constexpr int sample_tile() { return (SAMPLE_THREADS / G) * SAMPLE_UNR; }

struct SampleArgs {
  ShardView s;
  const int64_t* targets;
  int64_t cap;
  const int64_t* d_n;
  int M;
  int hop;
  unsigned long long seed;
  const unsigned long long* d_seed;
  int64_t* out_row_ptr;
  int64_t* out_nbrs;
  int32_t* out_pos;
  int64_t* d_num_edges;
  unsigned long long* status;
  unsigned* ctrl;
  HashTable ht;      // FUSED only
  int32_t* slot_of;  // FUSED only: slot of every position [targets ; neighbours]
};

template <int G, bool FUSED>
__global__ void __launch_bounds__(SAMPLE_THREADS) sample_kernel(const SampleArgs a) {
  constexpr int SAMPLE_TILE = sample_tile<G>();
  __shared__ int64_t sm_v[SAMPLE_TILE];
  __shared__ int64_t sm_start[SAMPLE_TILE];
  __shared__ int64_t sm_off[SAMPLE_TILE];
  __shared__ unsigned sm_deg[SAMPLE_TILE];
  __shared__ unsigned sm_chain[SAMPLE_THREADS / 32][32];
  __shared__ int sm_wtot[SAMPLE_THREADS / 32 + 1];
  __shared__ unsigned long long sm_prefix;
  __shared__ int sm_flag;

  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  int64_t nT = a.cap;
  if (a.d_n) {
    nT = *a.d_n;
    if (nT > a.cap || nT < 0) {
      if (tid == 0 && blockIdx.x == 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
      nT = nT < 0 ? 0 : a.cap;
    }
  }
  const unsigned epoch = FUSED ? a.ctrl[CTRL_EPOCH] : 0u;
  const int64_t tile_start = (int64_t)blockIdx.x * SAMPLE_TILE;

  if (nT == 0) {
    if (blockIdx.x == 0 && tid == 0) {
      a.out_row_ptr[0] = 0;
      if (a.d_num_edges) *a.d_num_edges = 0;
    }
  } else if (tile_start < nT) {
    const int M = a.M;
    // ---------------- count phase
    const int64_t idx = tile_start + tid;
    unsigned deg = 0;
    int64_t v = -1, start = 0;
    if (tid < SAMPLE_TILE && idx < nT) {
      v = a.targets[idx];
      if (v < 0 || v >= a.s.n) {
        latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
        if (FUSED) a.slot_of[idx] = -1;
      } else {
        int o;
        int64_t l;
        owner_local(a.s, v, o, l);
        const int64_t* rp = a.s.row_ptr[o] + l;
        start = rp[0];
        const int64_t d = rp[1] - start;
        if (d >= (int64_t(1) << 32) || d < 0)
          latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_DEGREE);
        else
          deg = (unsigned)d;
        if (FUSED) {
          const long long slot = hash_insert_min(a.ht, v, idx, epoch);
          if (slot < 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
          a.slot_of[idx] = (int32_t)slot;
        }
      }
    }
    const int cnt = (int)min((unsigned)M, deg);
    int agg;
    const int excl = block_exclusive_sum<SAMPLE_THREADS>(cnt, sm_wtot, &agg);
    if (warp == 0) {
      const unsigned long long pre = tile_lookback(a.status, (long)blockIdx.x, (unsigned long long)agg);
      if (lane == 0) sm_prefix = pre;
    }
    __syncthreads();
    const int64_t off = (int64_t)sm_prefix + excl;
    if (tid < SAMPLE_TILE) {
      sm_v[tid] = v;
      sm_start[tid] = start;
      sm_deg[tid] = deg;
      sm_off[tid] = off;
    }
    if (tid < SAMPLE_TILE && idx < nT) a.out_row_ptr[idx] = off;
    if (tid < SAMPLE_TILE && idx == nT - 1) {
      a.out_row_ptr[nT] = off + cnt;
      if (a.d_num_edges) *a.d_num_edges = off + cnt;
    }
    __syncthreads();

    // ---------------- sample phase
    const unsigned long long seed = a.d_seed ? *a.d_seed : a.seed;
    const uint2 key = make_uint2((unsigned)(seed & 0xffffffffu), (unsigned)(seed >> 32));
    constexpr int TPW = 32 / G;                  // targets per warp per round
    constexpr int TPR = SAMPLE_THREADS / G;      // targets per block per round
    const int g = lane / G;                      // target slot within the warp
    const int i = lane % G;                      // draw index
    const int tile_n = (int)min((int64_t)SAMPLE_TILE, nT - tile_start);
    for (int r0 = 0; r0 < SAMPLE_UNR; r0 += SAMPLE_UNR) {  // one round-chunk per tile (see sample_tile)
      if (r0 * TPR >= tile_n) break;  // block-uniform
      const int64_t* src[SAMPLE_UNR];
      int64_t dst[SAMPLE_UNR];
      unsigned pos[SAMPLE_UNR];
      bool ok[SAMPLE_UNR];
#pragma unroll
      for (int u = 0; u < SAMPLE_UNR; ++u) {
        const int k = (r0 + u) * TPR + warp * TPW + g;
        const bool active = k < tile_n;
        int64_t tv = 0, tstart = 0, toff = 0;
        unsigned N = 0;
        if (active) {
          tv = sm_v[k];
          tstart = sm_start[k];
          N = sm_deg[k];
          toff = sm_off[k];
        }
        const bool full = N <= (unsigned)M;
        const bool draw = active && !full && i < M;
        unsigned r = 0;
        if (draw) {
          const uint4 x = philox4x32_10(
              make_uint4((unsigned)(i >> 2), (unsigned)a.hop, (unsigned)((uint64_t)tv & 0xffffffffu),
                         (unsigned)((uint64_t)tv >> 32)),
              key);
          const unsigned xi = (i & 3) == 0 ? x.x : (i & 3) == 1 ? x.y : (i & 3) == 2 ? x.z : x.w;
          r = __umulhi(xi, N - (unsigned)i);  // floor(x * (N-i) / 2^32), in [0, N-1-i]
        }
        const unsigned long long mkey =
            draw ? (((unsigned long long)g << 32) | r) : (0xffffffff00000000ull | (unsigned)lane);
        const unsigned same = __match_any_sync(FULL_MASK, mkey);
        const unsigned below = same & ((1u << lane) - 1u);
        const int prev = below ? 31 - __clz(below) : -1;  // previous draw with value r
        const bool is_last = (same >> lane) == 1u;        // no later draw with value r
        sm_chain[warp][lane] = (unsigned)i;
        __syncwarp();
        if (draw && is_last && r >= N - (unsigned)M) sm_chain[warp][g * G + (int)(N - 1u - r)] = (unsigned)i;
        __syncwarp();
        unsigned c = sm_chain[warp][lane];
        for (int s = 1; s < M; s <<= 1) c = __shfl_sync(FULL_MASK, c, g * G + (int)c);
        const unsigned last = N - c - 1u;
        const unsigned lastp = __shfl_sync(FULL_MASK, last, prev >= 0 ? prev : lane);
        __syncwarp();
        pos[u] = full ? (unsigned)i : (prev < 0 ? r : lastp);
        ok[u] = active && (full ? (unsigned)i < N : i < M);
        int o = 0;
        int64_t l;
        if (ok[u]) owner_local(a.s, tv, o, l);
        src[u] = a.s.col[o] + tstart + pos[u];
        dst[u] = toff + i;
      }
      int64_t nb[SAMPLE_UNR];
#pragma unroll
      for (int u = 0; u < SAMPLE_UNR; ++u) nb[u] = ok[u] ? *src[u] : -1;
#pragma unroll
      for (int u = 0; u < SAMPLE_UNR; ++u) {
        if (ok[u]) {
          a.out_nbrs[dst[u]] = nb[u];
          if (a.out_pos) a.out_pos[dst[u]] = (int32_t)pos[u];
        }
      }
      if (FUSED) {
#pragma unroll
        for (int u = 0; u < SAMPLE_UNR; ++u) {
          const bool valid = ok[u] && nb[u] >= 0 && nb[u] < a.s.n;
          if (ok[u] && !valid) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_ID_RANGE);
          const unsigned long long mk = valid ? (unsigned long long)nb[u] : (0x8000000000000000ull | (unsigned)lane);
          const unsigned same = __match_any_sync(FULL_MASK, mk);
          const int leader = __ffs(same) - 1;  // lowest lane = smallest position among equal keys
          long long slot = -1;
          if (valid && leader == lane) {
            slot = hash_insert_min(a.ht, nb[u], nT + dst[u], epoch);
            if (slot < 0) latch_error(&a.ctrl[CTRL_ERR], WG_DEVERR_CAPACITY);
          }
          slot = __shfl_sync(FULL_MASK, slot, leader);
          if (ok[u]) a.slot_of[nT + dst[u]] = valid ? (int32_t)slot : -1;
        }
      }
    }
  }

  // ---------------- reset the look-back status for the next launch
  if (finish_block(&a.ctrl[CTRL_DONE_SAMPLE], &sm_flag)) {
    for (int t = tid; t < (int)gridDim.x; t += SAMPLE_THREADS) a.status[t] = 0ull;
    if (tid == 0) a.ctrl[CTRL_DONE_SAMPLE] = 0u;
  }
}

template <bool FUSED>
static void launch_sample_t(const SampleArgs& a, int fanout, dim3 grid, cudaStream_t st) {
  if (fanout <= 8)
    sample_kernel<8, FUSED><<<grid, SAMPLE_THREADS, 0, st>>>(a);
  else if (fanout <= 16)
    sample_kernel<16, FUSED><<<grid, SAMPLE_THREADS, 0, st>>>(a);
  else
    sample_kernel<32, FUSED><<<grid, SAMPLE_THREADS, 0, st>>>(a);
}

cudaError_t launch_sample(wg_dsm* h, const int64_t* targets, int64_t cap, const int64_t* d_n, int fanout,
                          uint64_t seed, const uint64_t* d_seed, int hop, int64_t* out_row_ptr,
                          int64_t* out_nbrs, int32_t* out_pos, int64_t* d_num_edges, bool fused, cudaStream_t st) {
  SampleArgs a;
  a.s = h->view;
  a.targets = targets;
  a.cap = cap;
  a.d_n = d_n;
  a.M = fanout;
  a.hop = hop;
  a.seed = seed;
  a.d_seed = reinterpret_cast<const unsigned long long*>(d_seed);
  a.out_row_ptr = out_row_ptr;
  a.out_nbrs = out_nbrs;
  a.out_pos = out_pos;
  a.d_num_edges = d_num_edges;
  a.status = h->ws.status_sample;
  a.ctrl = h->ws.ctrl;
  a.ht = HashTable{h->ws.hkeys, h->ws.hvals, (unsigned long long)h->ws.hcap - 1};
  a.slot_of = h->ws.slot_of;
  const int tile = fanout <= 8 ? sample_tile<8>() : fanout <= 16 ? sample_tile<16>() : sample_tile<32>();
  const int64_t tiles = cap > 0 ? (cap + tile - 1) / tile : 1;
  dim3 grid((unsigned)tiles);
  if (fused)
    launch_sample_t<true>(a, fanout, grid, st);
  else
    launch_sample_t<false>(a, fanout, grid, st);
  return cudaGetLastError();
}

}  // namespace wg
