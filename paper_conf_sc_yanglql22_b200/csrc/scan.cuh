// scan.cuh -- tile prefixes of the single-pass scans: a direct sum of the predecessors' aggregates for
// grids of at most WG_LB_DIRECT_MAX tiles, else a block-wide decoupled look-back.
//
// Look-back: the whole block (not one warp) inspects NT predecessor tiles per step, so the
// exclusive prefix of tile t resolves in ~t / NT dependent L2 round trips instead of
// ~t / 32: with ~1000 tiles in flight this is what keeps the scans from serialising.
#pragma once

#include "device_util.cuh"

// Back-off between polls of a predecessor tile that has published nothing yet (ns; 0 = spin).
#ifndef WG_LB_SLEEP_NS
#define WG_LB_SLEEP_NS 32
#endif

namespace wg {

__device__ __forceinline__ void lb_backoff() {
#if WG_LB_SLEEP_NS > 0
  __nanosleep(WG_LB_SLEEP_NS);
#endif
}

template <int NT>
struct LookbackSmem {
  unsigned pmask[NT / 32];
  unsigned long long part[NT / 32];
  int stop;
  int found;
};

// Called by ALL threads of the block.  Publishes `aggregate` for tile `tile`, resolves
// the tile's exclusive prefix (returned in every thread) and publishes the inclusive
// prefix.  Status word format as in device_util.cuh (LB_AGG / LB_PRE / LB_VAL).
template <int NT>
__device__ __forceinline__ unsigned long long block_lookback(unsigned long long* status, long tile,
                                                             unsigned long long aggregate, LookbackSmem<NT>& sm) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tile == 0) {
    if (tid == 0) st_volatile_u64(&status[0], LB_PRE | aggregate);
    return 0ull;
  }
  if (tid == 0) st_volatile_u64(&status[tile], LB_AGG | aggregate);
  // fast path: warp 0 inspects the 32 closest predecessors (usually enough: tiles finish roughly
  // in order); only if none of them holds an inclusive prefix does the whole block walk back
  if (warp == 0) {
    const long idx = tile - 1 - lane;
    unsigned long long s = idx >= 0 ? ld_volatile_u64(&status[idx]) : LB_PRE;
    while ((s >> 62) == 0) {
      lb_backoff();
      s = ld_volatile_u64(&status[idx]);
    }
    const unsigned pm = __ballot_sync(FULL_MASK, (s >> 62) == 2);
    const int stop = pm ? __ffs(pm) - 1 : 31;
    const unsigned long long v = warp_sum(lane <= stop ? (s & LB_VAL) : 0ull);
    if (lane == 0) {
      sm.part[0] = v;
      sm.found = pm != 0;
    }
  }
  __syncthreads();
  unsigned long long excl = sm.part[0];
  const bool fast = sm.found != 0;
  __syncthreads();  // sm is reused below
  long pred = tile - 33;
  for (; !fast;) {
    const long idx = pred - tid;
    unsigned long long s = idx >= 0 ? ld_volatile_u64(&status[idx]) : LB_PRE;
    while ((s >> 62) == 0) {
      lb_backoff();
      s = ld_volatile_u64(&status[idx]);
    }
    const unsigned pm = __ballot_sync(FULL_MASK, (s >> 62) == 2);
    if (lane == 0) sm.pmask[warp] = pm;
    __syncthreads();
    if (tid == 0) {
      int stop = NT - 1, found = 0;
      for (int w = 0; w < NT / 32; ++w)
        if (sm.pmask[w]) {
          stop = w * 32 + __ffs(sm.pmask[w]) - 1;  // closest predecessor holding an inclusive prefix
          found = 1;
          break;
        }
      sm.stop = stop;
      sm.found = found;
    }
    __syncthreads();
    const int stop = sm.stop;
    const bool found = sm.found != 0;
    unsigned long long v = tid <= stop ? (s & LB_VAL) : 0ull;
    v = warp_sum(v);
    if (lane == 0) sm.part[warp] = v;
    __syncthreads();
    unsigned long long tot = 0;
#pragma unroll
    for (int w = 0; w < NT / 32; ++w) tot += sm.part[w];
    excl += tot;
    __syncthreads();  // sm reused next step
    if (found) break;
    pred -= NT;
  }
  if (tid == 0) st_volatile_u64(&status[tile], LB_PRE | (excl + aggregate));
  return excl;
}

// Direct form for grids of at most WG_LB_DIRECT_MAX tiles: tile t publishes its
// aggregate, then its threads read the aggregates of ALL tiles < t (ceil(t / NT) loads each, spinning until
// published) and reduce them -- one round, no chain of inclusive prefixes.  Tiles never publish an
// inclusive prefix here, so every status word keeps its aggregate.  The aggregates of one wave are
// published within a few microseconds of each other, so the polls spin without back-off.  Measured on
// B200 (profiles/r02/ab_log.md): products hop 2 (440 tiles) single batch -2 %, throughput +2 %.
#ifndef WG_LB_DIRECT_MAX
#define WG_LB_DIRECT_MAX 1024
#endif
template <int NT>
__device__ __forceinline__ unsigned long long block_prefix_direct(unsigned long long* status, long tile,
                                                                  unsigned long long aggregate, LookbackSmem<NT>& sm) {
  const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
  if (tid == 0) st_volatile_u64(&status[tile], LB_AGG | aggregate);
  unsigned long long v = 0;
  for (long j = tid; j < tile; j += NT) {
    unsigned long long s = ld_volatile_u64(&status[j]);
    while ((s >> 62) == 0) s = ld_volatile_u64(&status[j]);
    v += s & LB_VAL;
  }
  v = warp_sum(v);
  if (lane == 0) sm.part[warp] = v;
  __syncthreads();
  unsigned long long tot = 0;
#pragma unroll
  for (int w = 0; w < NT / 32; ++w) tot += sm.part[w];
  __syncthreads();  // sm reused by the caller
  return tot;
}

}  // namespace wg
