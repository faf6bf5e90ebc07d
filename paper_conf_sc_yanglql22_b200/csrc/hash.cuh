// hash.cuh -- the append-unique hash table (PAPER.md: "The key of our GPU
// hash table is nodeID"; Warpcore-style open addressing [33]).
//
// Slot s (16 B, key and value in the same 32 B sector so an insert touches one
// sector): key = (epoch << 40) | node id, val = ((EPOCH_MAX - epoch) << 40) | first
// position.  A key from an older epoch reads as an empty slot and an older
// value always loses an atomicMin against the current epoch, so the table is never
// cleared between calls.  Linear probing, fmix64 hash mapped onto [0, size) by a multiply-high,
// load factor <= 1 / HASH_FACTOR (2) at the capacity bound.
#pragma once

#include "device_util.cuh"
#include "wg_internal.cuh"

namespace wg {

constexpr unsigned long long KEY_MASK = (1ull << 40) - 1;

struct HashTable {
  HashSlot* slots;
  unsigned long long size;  // slots in use (any size: slot = high half of hash * size)
  int compact;              // 8 B slots (below) instead of 16 B HashSlots
  HashSlot* slots2;         // compact: the table of odd 255-epoch cycles (slots serves the even ones)
};
// The table an op at this epoch uses: the compact format alternates between two tables per 255-epoch
// cycle like the direct one (below); the wide format has one table and 2^23 epochs.
__device__ __forceinline__ HashTable ht_for_epoch(HashTable t, unsigned epoch) {
  if (t.compact && ((epoch / CEPOCHS) & 1u)) t.slots = t.slots2;
  return t;
}
// Compact format, called by every thread of the FIRST kernel of an append-unique: at the first epoch of
// a cycle, zero the other (idle) table's `words` words (grid-strided) -- it served the previous cycle,
// whose ops have all finished, and serves the next one.
static __device__ __noinline__ void chash_clear_words(unsigned long long* w, int64_t words) {
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < words; i += stride) w[i] = 0ull;
}
__device__ __forceinline__ void chash_clear_ahead(const HashTable& t, int64_t words, unsigned epoch) {
  if (t.compact && compact_epoch(epoch) == 1u)
    chash_clear_words(reinterpret_cast<unsigned long long*>(((epoch / CEPOCHS) & 1u) ? t.slots : t.slots2), words);
}

// ---- compact table: one 64-bit word per slot, [63:56] epoch (1..255), [55:28] node id, [27:0]
// first position (nodes and positions < 2^28).  Claimed with one 64-bit CAS of the whole word;
// later occurrences of the key lower it with a 64-bit atomicMin (epoch and id bits are equal,
// so the minimum is taken over the position).  Stale words (another epoch, or 0 after a clear)
// read as empty; two tables alternate per 255-epoch cycle and the idle one is zeroed at a cycle's
// first op (chash_clear_ahead), so neither needs a per-call memset.
constexpr unsigned long long CPOS_MASK = (1ull << 28) - 1;
__device__ __forceinline__ unsigned long long cword(unsigned ce, int64_t key, int64_t q) {
  return ((unsigned long long)ce << 56) | ((unsigned long long)key << 28) | (unsigned long long)q;
}
// Home slot of `key` in a table of t.size slots.
__device__ __forceinline__ unsigned long long chash_home(const HashTable& t, int64_t key) {
  return __umul64hi(fmix64((unsigned long long)key), t.size);
}
__device__ __forceinline__ unsigned long long chash_load(const HashTable& t, unsigned long long slot) {
  unsigned long long cur;
  asm volatile("ld.volatile.global.u64 %0, [%1];" : "=l"(cur) : "l"(&reinterpret_cast<unsigned long long*>(t.slots)[slot]));
  return cur;
}
// Insert continuing from slot `slot` whose word was read as `cur` (chash_home / chash_load; issuing several
// keys' first loads before resolving any measured slower, profiles/r02/ab_log.md).  Returns the slot of `key` (claimed
// with position q if new), or -1 if full; *old = the word seen (0 if this call claimed the slot).
// Applies the atomicMin (with return if want_old; else only when the word holds a larger position).
__device__ __forceinline__ long long chash_insert_from(const HashTable& t, int64_t key, int64_t q, unsigned ce,
                                                       bool want_old, unsigned long long* old, unsigned long long slot,
                                                       unsigned long long cur) {
  unsigned long long* w = reinterpret_cast<unsigned long long*>(t.slots);
  const unsigned long long mine = cword(ce, key, q);
  for (unsigned long long probe = 0; probe < t.size; ++probe) {
    if (probe) cur = chash_load(t, slot);
    for (;;) {
      if ((cur >> 28) == (mine >> 28)) {  // our key, this epoch
        if (want_old) {
          *old = atomicMin(&w[slot], mine);
        } else {
          if ((cur & CPOS_MASK) > (unsigned long long)q) atomicMin(&w[slot], mine);
          *old = cur;
        }
        return (long long)slot;
      }
      if ((unsigned)(cur >> 56) == ce) break;  // another key this epoch
      const unsigned long long prev = atomicCAS(&w[slot], cur, mine);
      if (prev == cur) {
        *old = 0;
        return (long long)slot;
      }
      cur = prev;
    }
    slot = slot + 1 == t.size ? 0 : slot + 1;
  }
  return -1;
}
__device__ __forceinline__ long long chash_insert(const HashTable& t, int64_t key, int64_t q, unsigned ce,
                                                  bool want_old, unsigned long long* old) {
  const unsigned long long slot = chash_home(t, key);
  return chash_insert_from(t, key, q, ce, want_old, old, slot, chash_load(t, slot));
}
__device__ __forceinline__ int64_t chash_min_pos(const HashTable& t, long long slot) {
  return (int64_t)(reinterpret_cast<const unsigned long long*>(t.slots)[slot] & CPOS_MASK);
}

// ---- direct table: one 32-bit word per node v, [31:24] 255 - compact_epoch(e) (1..255), [23:0] the first
// position of v in the current call.  A newer epoch has a SMALLER tag, so one atomicMin of the whole word
// both overrides a stale word and keeps the minimum position; 0xFFFFFFFF is empty.  Epochs come in cycles
// of CEPOCHS; cycle c = e / CEPOCHS uses table c & 1 for all its epochs, so consecutive hops and batches of
// a workspace keep hitting the same (L2-resident) lines.  The first op of cycle c clears table (c+1) & 1
// -- idle: it served cycle c-1, whose ops have all finished -- so the next cycle starts on a clean table;
// the tables are never cleared per call.  No slot, no probe, no claim: a neighbour insert is one RED.MIN.
struct DirectTable {
  unsigned* t[2];
  int64_t n;  // words per table (num_nodes)
};
constexpr unsigned DPOS_MASK = (1u << DPOS_BITS) - 1u;
__device__ __forceinline__ unsigned dtag(unsigned epoch) { return 255u - compact_epoch(epoch); }
__device__ __forceinline__ unsigned dword(unsigned tag, int64_t q) { return (tag << DPOS_BITS) | (unsigned)q; }
__device__ __forceinline__ unsigned* dtab_cur(const DirectTable& d, unsigned epoch) {
  return ((epoch / CEPOCHS) & 1u) ? d.t[1] : d.t[0];
}
// First position recorded for v in this epoch, or -1 (not inserted in this epoch).
__device__ __forceinline__ int64_t dtab_min_pos(const unsigned* t, unsigned tag, int64_t v) {
  const unsigned w = t[v];
  return (w >> DPOS_BITS) == tag ? (int64_t)(w & DPOS_MASK) : -1;
}
static __device__ __noinline__ void dtab_clear_words(unsigned* t, int64_t n) {
  uint4* w = reinterpret_cast<uint4*>(t);
  const int64_t n4 = (n + 3) / 4;  // tables are allocated in whole 16 B units
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n4; i += stride)
    w[i] = make_uint4(~0u, ~0u, ~0u, ~0u);
}
// Called by every thread of the FIRST kernel of an append-unique (the fused hop's sampler, or the
// standalone insert pass): at the first epoch of a cycle, clear the other (idle) table (grid-strided).
__device__ __forceinline__ void dtab_clear_ahead(const DirectTable& d, unsigned epoch) {
  if (compact_epoch(epoch) == 1u) dtab_clear_words(((epoch / CEPOCHS) & 1u) ? d.t[0] : d.t[1], d.n);
}

__device__ __forceinline__ unsigned long long stored_key(unsigned epoch, int64_t key) {
  return ((unsigned long long)epoch << 40) | (unsigned long long)key;
}

__device__ __forceinline__ unsigned long long pack_pos(unsigned epoch, int64_t q) {
  return ((unsigned long long)(EPOCH_MAX - epoch) << 40) | (unsigned long long)q;
}

// 128-bit compare-and-swap (sm_90+): claims a slot by writing key AND value in one atomic.
__device__ __forceinline__ void cas128(HashSlot* p, unsigned long long& k, unsigned long long& v,
                                       unsigned long long nk, unsigned long long nv) {
  asm volatile(
      "{\n .reg .b128 c, n, d;\n mov.b128 c, {%0, %1};\n mov.b128 n, {%2, %3};\n"
      " atom.global.cas.b128 d, [%4], c, n;\n mov.b128 {%0, %1}, d;\n}"
      : "+l"(k), "+l"(v)
      : "l"(nk), "l"(nv), "l"(p)
      : "memory");
}

// Returns the slot holding `stored` (claiming an empty one if needed), or -1 if full.
// *seen receives the slot's value as read together with its key (one 16 B load) when the
// key was already present.  A claim writes the key together with the value `mine` in one
// 128-bit CAS, and *seen = 0 tells the caller nothing is left to do.
__device__ __forceinline__ long long hash_insert(const HashTable& t, unsigned long long stored, unsigned epoch,
                                                 unsigned long long mine, unsigned long long* seen) {
  unsigned long long slot = __umul64hi(fmix64(stored & KEY_MASK), t.size);  // uniform in [0, size)
  for (unsigned long long probe = 0; probe < t.size; ++probe) {
    unsigned long long cur, val;
    asm volatile("ld.volatile.global.v2.u64 {%0, %1}, [%2];" : "=l"(cur), "=l"(val) : "l"(&t.slots[slot]));
    for (;;) {
      if (cur == stored) {
        *seen = val;
        return (long long)slot;
      }
      if ((unsigned)(cur >> 40) == epoch) break;  // occupied by another key this epoch
      const unsigned long long ck = cur, cv = val;
      cas128(&t.slots[slot], cur, val, stored, mine);  // cur, val <- the slot's previous contents
      if (cur == ck && val == cv) {
        *seen = 0;  // claimed with our position already in place
        return (long long)slot;
      }
      // re-examine what is there now (our key, another key, or a newer stale pair)
    }
    slot = slot + 1 == t.size ? 0 : slot + 1;
  }
  return -1;
}

// The atomicMin is skipped when the value read with the key already holds a smaller
// position of this epoch: hub ids occur thousands of times per hop, and this removes
// most of the same-address atomics they would otherwise serialise on.
__device__ __forceinline__ long long hash_insert_min(const HashTable& t, int64_t key, int64_t q, unsigned epoch) {
  unsigned long long seen;
  const unsigned long long mine = pack_pos(epoch, q);
  const long long slot = hash_insert(t, stored_key(epoch, key), epoch, mine, &seen);
  if (slot >= 0 && seen > mine) atomicMin(&t.slots[slot].val, mine);
  return slot;
}

// Target insert (position q < nT): returns the slot and sets *dup if another TARGET
// with the same key was recorded first in this epoch (the returned old minimum is
// then a target position).  Of two equal targets the later atomic always sees the
// earlier one, so a duplicate target is always detected (reading A8).
__device__ __forceinline__ long long hash_insert_target(const HashTable& t, int64_t key, int64_t q, int64_t nT,
                                                        unsigned epoch, bool* dup) {
  unsigned long long seen;
  const unsigned long long mine = pack_pos(epoch, q);
  const long long slot = hash_insert(t, stored_key(epoch, key), epoch, mine, &seen);
  *dup = false;
  if (slot >= 0 && seen != 0) {  // seen == 0: claimed by our 128-bit CAS, no earlier record
    const unsigned long long old = atomicMin(&t.slots[slot].val, mine);
    *dup = (old >> 40) == (unsigned long long)(EPOCH_MAX - epoch) && (int64_t)(old & KEY_MASK) < nT;
  }
  return slot;
}

}  // namespace wg
