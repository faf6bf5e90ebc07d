// sample_warp.cuh -- the warp sampler's per-warp body (Algorithm 1 L122-158 in its
// sort-free form), shared by sample_kernel (sample.cu) and the single-pass hop kernel (hop.cu).
//
// A group of G = max(M, SAMPLE_UNR_MAX) lanes handles one target; a warp handles UNR rounds of
// TPW = floor(32 / G) targets, all in flight at once.  Per target (see sample.cu for the derivation):
//   - lane u of the group loads round u's (row_ptr[l], row_ptr[l+1]) pair from its owner;
//   - M >= N: lane i < N takes position i (L118, CSR order, A5);
//   - else lane i draws r_i (Philox4x32-10, A3) and computes Algorithm 1's res[i] with one
//     __match_any_sync (previous equal draw, run end), the chain in 32 words of shared memory and
//     path doubling by __shfl_sync -- the same function as Algorithm 1 / sequential Fisher-Yates;
//   - lane i loads col[start + res_i] (local HBM or a peer over NVLink).
#pragma once

#include "device_util.cuh"
#include "wg_internal.cuh"

namespace wg {

constexpr int SAMPLE_UNR_MAX = 4;
// Lane groups are G = max(M, SAMPLE_UNR_MAX) lanes (not a power of two), so a warp holds
// floor(32 / G) targets per round: e.g. 6 targets for M = 5, 3 for M = 10.
__host__ __device__ inline int sample_group(int M) { return M > SAMPLE_UNR_MAX ? M : SAMPLE_UNR_MAX; }

// One warp samples the targets k = warp_base + u * TPW + g (u < UNR, g < TPW, k < nT) of targets[].
// on_target(k, v) is called once per target k < nT with its id as loaded (before the range check),
// right after its row_ptr loads are issued; it returns a token handed to on_target_end(k, token) after every other callback
// of the warp (the direct table issues the target's atomic early and checks its result late); emit_cnt(k, c) once per target k < nT (c = min(M, deg), 0
// for an invalid id); emit(k, i, nb, pos) for every sampled slot i < c (draw order, A5); emit_pad(k, i)
// for the slots c <= i < M; then insert_all(nb, kk, ok) once with this lane's UNR rounds (sampled id,
// target, valid), so a key-table insert can issue all its first loads before resolving any.
// chain: this warp's 32 words of shared memory.
// All 32 lanes must call it (warp-collective); warps past nT return at once.
template <int UNR, bool COL32, typename OnTarget, typename OnTargetEnd, typename EmitCnt, typename Emit,
          typename EmitPad, typename InsertAll>
__device__ __forceinline__ void sample_warp(const ShardView& s, const int64_t* targets, int64_t nT, int M, int hop,
                                            uint2 key, int64_t warp_base, unsigned* chain, unsigned* ctrl_err,
                                            OnTarget on_target, OnTargetEnd on_target_end, EmitCnt emit_cnt, Emit emit,
                                            EmitPad emit_pad, InsertAll insert_all) {
  if (warp_base >= nT) return;  // warp-uniform
  const int lane = threadIdx.x & 31;
  const int G = sample_group(M);
  const int TPW = 32 / G;      // targets per warp per round
  const int g = lane / G;      // target slot within the warp (g == TPW: leftover lanes, idle)
  const int i = lane - g * G;  // draw index

  // ---- row_ptr pairs: lane u of each group fetches round u's target (all in flight)
  int64_t my_v = -1, my_start = 0;
  unsigned my_deg = 0, my_tok = 0;
  if (i < UNR && g < TPW) {
    const int64_t k = warp_base + (int64_t)i * TPW + g;
    if (k < nT) {
      my_v = targets[k];
      const int64_t raw = my_v;
      int64_t r1 = 0;
      if (my_v < 0 || my_v >= s.n) {
        latch_error(ctrl_err, WG_DEVERR_ID_RANGE);
        my_v = -1;
      } else {
        int o;
        int64_t l;
        csr_owner_local(s, my_v, o, l);
        const int64_t* rp = s.row_ptr[o] + l;
        my_start = rp[0];
        r1 = rp[1];
      }
      my_tok = on_target(k, raw);  // after the row_ptr loads are issued: their latency hides its work
      if (my_v >= 0) {
        const int64_t d = r1 - my_start;
        if (d >= (int64_t(1) << 32) || d < 0)
          latch_error(ctrl_err, WG_DEVERR_DEGREE);
        else
          my_deg = (unsigned)d;
      }
    }
  }

  int64_t src[UNR];  // col_idx entry of the draw
  int osrc[UNR];     // its owner rank
  int64_t kk[UNR];
  unsigned pos[UNR];
  bool ok[UNR], pad[UNR];
#pragma unroll
  for (int u = 0; u < UNR; ++u) {
    const int64_t k = warp_base + (int64_t)u * TPW + g;
    const int from = g * G + u;  // the lane that loaded this round's row_ptr pair
    const int64_t tv = __shfl_sync(FULL_MASK, my_v, from);
    const int64_t tstart = __shfl_sync(FULL_MASK, my_start, from);
    const unsigned N = __shfl_sync(FULL_MASK, my_deg, from);
    const bool active = g < TPW && k < nT && tv >= 0;
    const bool full = N <= (unsigned)M;
    const bool draw = active && !full && i < M;
    unsigned r = 0;
    if (draw) {
      const uint4 x = philox4x32_10(make_uint4((unsigned)(i >> 2), (unsigned)hop,
                                               (unsigned)((uint64_t)tv & 0xffffffffu), (unsigned)((uint64_t)tv >> 32)),
                                    key);
      const unsigned xi = (i & 3) == 0 ? x.x : (i & 3) == 1 ? x.y : (i & 3) == 2 ? x.z : x.w;
      r = __umulhi(xi, N - (unsigned)i);  // floor(x * (N-i) / 2^32), in [0, N-1-i]
    }
    const unsigned long long mkey =
        draw ? (((unsigned long long)g << 32) | r) : (0xffffffff00000000ull | (unsigned)lane);
    const unsigned same = __match_any_sync(FULL_MASK, mkey);
    const unsigned below = same & ((1u << lane) - 1u);
    const int prev = below ? 31 - __clz(below) : -1;  // previous draw with value r (Alg.1 p[q[i]-1])
    const bool is_last = (same >> lane) == 1u;        // no later draw with value r (Alg.1 line 4)
    chain[lane] = (unsigned)i;                        // Alg.1 line 1: chain[i] = i
    __syncwarp();
    if (draw && is_last && r >= N - (unsigned)M)      // Alg.1 lines 4-5
      chain[g * G + (int)(N - 1u - r)] = (unsigned)i;
    __syncwarp();
    unsigned c = chain[lane];
    for (int st = 1; st < M; st <<= 1) c = __shfl_sync(FULL_MASK, c, g * G + (int)c);  // line 12
    const unsigned last = N - c - 1u;                                                  // line 14
    const unsigned lastp = __shfl_sync(FULL_MASK, last, prev >= 0 ? prev : lane);
    __syncwarp();
    pos[u] = full ? (unsigned)i : (prev < 0 ? r : lastp);  // lines 16-22
    ok[u] = active && (full ? (unsigned)i < N : i < M);
    pad[u] = g < TPW && k < nT && i < M && !ok[u];
    int o = 0;
    int64_t l;
    if (ok[u]) csr_owner_local(s, tv, o, l);
    osrc[u] = o;
    src[u] = tstart + pos[u];
    kk[u] = k;
    if (i == 0 && g < TPW && k < nT) emit_cnt(k, active ? (int)min(N, (unsigned)M) : 0);
  }
  int64_t nb[UNR];
#pragma unroll
  for (int u = 0; u < UNR; ++u) nb[u] = ok[u] ? ld_col<COL32>(s, osrc[u], src[u]) : -1;
#pragma unroll
  for (int u = 0; u < UNR; ++u) {
    if (ok[u]) emit(kk[u], i, nb[u], pos[u]);
    else if (pad[u]) emit_pad(kk[u], i);
  }
  insert_all(nb, kk, ok);
  if (i < UNR && g < TPW) {
    const int64_t k = warp_base + (int64_t)i * TPW + g;
    if (k < nT) on_target_end(k, my_tok);
  }
}

}  // namespace wg
