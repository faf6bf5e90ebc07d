// hash.cuh -- the append-unique hash table (PAPER.md: "The key of our GPU
// hash table is nodeID"; Warpcore-style open addressing [33]).
//
// Slot s (16 B, key and value in the same 32 B sector so an insert touches one
// sector): key = (epoch << 40) | node id, val = ((EPOCH_MAX - epoch) << 40) | first
// position.  A key from an older epoch reads as an empty slot and an older
// value always loses an atomicMin against the current epoch, so the table is never
// cleared between calls.  Linear probing, fmix64 hash mapped onto [0, size) by a multiply-high,
// load factor <= 1 / WG_HASH_FACTOR at the capacity bound.
#pragma once

#include "device_util.cuh"
#include "wg_internal.cuh"

namespace wg {

constexpr unsigned long long KEY_MASK = (1ull << 40) - 1;

struct HashTable {
  HashSlot* slots;
  unsigned long long size;  // slots in use (any size: slot = high half of hash * size)
};

__device__ __forceinline__ unsigned long long stored_key(unsigned epoch, int64_t key) {
  return ((unsigned long long)epoch << 40) | (unsigned long long)key;
}

__device__ __forceinline__ unsigned long long pack_pos(unsigned epoch, int64_t q) {
  return ((unsigned long long)(EPOCH_MAX - epoch) << 40) | (unsigned long long)q;
}

// Returns the slot holding `stored` (claiming an empty one if needed), or -1 if full.
// *seen receives the slot's value as read together with its key (one 16 B load) when the
// key was already present, or ~0 when this call claimed the slot.
__device__ __forceinline__ long long hash_insert(const HashTable& t, unsigned long long stored, unsigned epoch,
                                                 unsigned long long* seen) {
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
      const unsigned long long prev = atomicCAS(&t.slots[slot].key, cur, stored);
      if (prev == cur) {
        *seen = ~0ull;
        return (long long)slot;
      }
      if (prev == stored) {
        *seen = ~0ull;  // claimed by another thread a moment ago: its minimum may not be there yet
        return (long long)slot;
      }
      cur = prev;
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
  const long long slot = hash_insert(t, stored_key(epoch, key), epoch, &seen);
  const unsigned long long mine = pack_pos(epoch, q);
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
  const long long slot = hash_insert(t, stored_key(epoch, key), epoch, &seen);
  *dup = false;
  if (slot >= 0) {
    const unsigned long long old = atomicMin(&t.slots[slot].val, pack_pos(epoch, q));
    *dup = (old >> 40) == (unsigned long long)(EPOCH_MAX - epoch) && (int64_t)(old & KEY_MASK) < nT;
  }
  return slot;
}

}  // namespace wg
