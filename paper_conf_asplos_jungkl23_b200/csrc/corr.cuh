// Execution ID correlation table (PAPER.md; reading D5):
// open addressing over 32 B slots {key = (owner e, h1, h2, h3), last =
// max(k << 32 | succ), first = min(k)}.  The 16 B key is claimed with one
// 128-bit CAS; the successor is the last observed (atomicMax on the packed
// launch index), the record order is first seen (atomicMin) -- both
// independent of thread order.  New records are appended to a
// dense list (rec_slot) that the jump-table build iterates.
#pragma once
#include "device_util.cuh"

namespace dum {

__device__ __forceinline__ uint32_t corr_hash(uint32_t owner, uint32_t h1, uint32_t h2, uint32_t h3, uint32_t cap) {
  const unsigned long long k0 = (unsigned long long)owner | ((unsigned long long)h1 << 32);
  const unsigned long long k1 = (unsigned long long)h2 | ((unsigned long long)h3 << 32);
  return (uint32_t)fmix64(k0 * 0x9E3779B97F4A7C15ull ^ fmix64(k1)) & (cap - 1);
}

__device__ __forceinline__ void corr_upsert(CorrSlot *corr, uint32_t cap, uint32_t *rec_slot, uint32_t owner,
                                            uint32_t h1, uint32_t h2, uint32_t h3, uint32_t succ, uint32_t k,
                                            DevState *st) {
  const unsigned long long k0 = (unsigned long long)owner | ((unsigned long long)h1 << 32);
  const unsigned long long k1 = (unsigned long long)h2 | ((unsigned long long)h3 << 32);
  uint32_t s = corr_hash(owner, h1, h2, h3, cap);
  for (uint32_t p = 0; p < cap; ++p) {
    CorrSlot *sl = corr + s;
    const volatile uint32_t *kv = sl->key;
    const uint32_t c0 = kv[0];
    bool mine = false;
    if (c0 == NONE) {
      unsigned long long o0, o1;
      cas128(sl->key, EMPTY64, EMPTY64, k0, k1, o0, o1);
      if (o0 == EMPTY64 && o1 == EMPTY64) {
        const uint32_t r = atomicAdd(&st->corr_used, 1u);
        if (r < cap) rec_slot[r] = s;
        mine = true;
      } else {
        mine = (o0 == k0 && o1 == k1);
      }
    } else {
      mine = c0 == owner && kv[1] == h1 && kv[2] == h2 && kv[3] == h3;
    }
    if (mine) {
      atomicMax(&sl->last, ((unsigned long long)k << 32) | succ);
      atomicMin(&sl->first, (unsigned long long)k);
      return;
    }
    s = (s + 1) & (cap - 1);
  }
  set_err(st, ERR_ECAPACITY, 2ull * cap);
}

// Slot of record (owner; h1, h2, h3) or NONE.  The 32 B slot is read with two
// independent 16 B loads (one round trip per probe); *succ receives the
// record's successor.
__device__ __forceinline__ uint32_t corr_find(const CorrSlot *corr, uint32_t cap, uint32_t owner, uint32_t h1,
                                              uint32_t h2, uint32_t h3, uint32_t *succ) {
  uint32_t s = corr_hash(owner, h1, h2, h3, cap);
  for (uint32_t p = 0; p < cap; ++p) {
    const uint4 *sp = reinterpret_cast<const uint4 *>(corr + s);
    const uint4 kk = __ldcg(sp);
    const uint4 vv = __ldcg(sp + 1);
    if (kk.x == NONE) return NONE;
    if (kk.x == owner && kk.y == h1 && kk.z == h2 && kk.w == h3) {
      *succ = vv.x;  // low word of `last`
      return s;
    }
    s = (s + 1) & (cap - 1);
  }
  return NONE;
}

}  // namespace dum
