// Device helpers shared by the kernels of libdeepum_b200.so.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "engine.cuh"

namespace dum {

#ifdef DUM_CHECKS
#define DCHECK(cond, ...)                                                        \
  do {                                                                           \
    if (!(cond)) {                                                               \
      printf("DCHECK %s:%d block %d thread %d: %s\n", __FILE__, __LINE__,        \
             (int)blockIdx.x, (int)threadIdx.x, #cond);                          \
      printf(__VA_ARGS__);                                                       \
      __trap();                                                                  \
    }                                                                            \
  } while (0)
#else
#define DCHECK(cond, ...) \
  do {                    \
  } while (0)
#endif

// Internal consistency guard: records the first failure (line, value) in the
// device state; the caller clamps/skips the offending access.
#define GUARD(st, cond, val)                                          \
  ((cond) ? true : (atomicCAS(&(st)->dbg_line, 0u, (uint32_t)__LINE__) == 0u \
                        ? ((st)->dbg_val = (uint32_t)(val), false)    \
                        : false))

__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31; }
__device__ __forceinline__ uint32_t warp_id() { return threadIdx.x >> 5; }

__device__ __forceinline__ void set_err(DevState *st, uint32_t bit, unsigned long long need = 0) {
  atomicOr(&st->err, bit);
  if (need) atomicMax(&st->needed, need);
}

// Block-wide exclusive scan of one value per thread.  `ws` must hold
// blockDim.x/32 u32.  Returns the exclusive prefix; *total = block sum.
// All threads of the block must call it.
__device__ __forceinline__ uint32_t block_excl_scan(uint32_t v, uint32_t *ws, uint32_t *total) {
  const uint32_t lane = lane_id(), wid = warp_id(), nw = blockDim.x >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= (uint32_t)o) x += y;
  }
  if (lane == 31) ws[wid] = x;
  __syncthreads();
  if (wid == 0) {
    uint32_t w = lane < nw ? ws[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(0xffffffffu, w, o);
      if (lane >= (uint32_t)o) w += y;
    }
    if (lane < nw) ws[lane] = w;
  }
  __syncthreads();
  uint32_t pre = (wid ? ws[wid - 1] : 0) + x - v;
  *total = ws[nw - 1];
  __syncthreads();
  return pre;
}

// 128-bit compare-and-swap (sm_90+: atom.cas.b128).  Returns the old value in
// (o0, o1).
__device__ __forceinline__ void cas128(void *addr, unsigned long long c0, unsigned long long c1,
                                       unsigned long long n0, unsigned long long n1,
                                       unsigned long long &o0, unsigned long long &o1) {
  asm volatile(
      "{\n\t.reg .b128 dd, cc, nn;\n\t"
      "mov.b128 cc, {%2, %3};\n\t"
      "mov.b128 nn, {%4, %5};\n\t"
      "atom.global.cas.b128 dd, [%6], cc, nn;\n\t"
      "mov.b128 {%0, %1}, dd;\n\t}"
      : "=l"(o0), "=l"(o1)
      : "l"(c0), "l"(c1), "l"(n0), "l"(n1), "l"(addr)
      : "memory");
}

// ---------------------------------------------------------------------------
// Open-addressing u32 -> u32 "minimum" map over generic memory (shared or
// global).  keys == NONE marks an empty slot.  cap is a power of two.
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t hslot(uint32_t key, uint32_t cap) { return fmix32(key) & (cap - 1); }

// Insert key (if absent) and lower its value to min(value, v).  Returns false
// if the table is full.
__device__ __forceinline__ bool hmap_insert_min(uint32_t *keys, uint32_t *vals, uint32_t cap, uint32_t key,
                                                uint32_t v) {
  uint32_t s = hslot(key, cap);
  for (uint32_t probe = 0; probe < cap; ++probe) {
    uint32_t k = ((volatile uint32_t *)keys)[s];
    if (k == NONE) {
      uint32_t old = atomicCAS(&keys[s], NONE, key);
      if (old == NONE || old == key) {
        atomicMin(&vals[s], v);
        return true;
      }
    } else if (k == key) {
      atomicMin(&vals[s], v);
      return true;
    }
    s = (s + 1) & (cap - 1);
  }
  return false;
}

// Lookup; returns NONE when absent.
__device__ __forceinline__ uint32_t hmap_get(const uint32_t *keys, const uint32_t *vals, uint32_t cap,
                                             uint32_t key) {
  uint32_t s = hslot(key, cap);
  for (uint32_t probe = 0; probe < cap; ++probe) {
    uint32_t k = ((const volatile uint32_t *)keys)[s];
    if (k == key) return ((const volatile uint32_t *)vals)[s];
    if (k == NONE) return NONE;
    s = (s + 1) & (cap - 1);
  }
  return NONE;
}

// Single-writer set ops used by the sequential walker (one warp, lane-parallel
// probes of distinct keys are fine because keys within one step are distinct).
__device__ __forceinline__ bool hset_contains(const uint32_t *keys, uint32_t cap, uint32_t key) {
  uint32_t s = hslot(key, cap);
  for (uint32_t probe = 0; probe < cap; ++probe) {
    uint32_t k = ((const volatile uint32_t *)keys)[s];
    if (k == key) return true;
    if (k == NONE) return false;
    s = (s + 1) & (cap - 1);
  }
  return false;
}
// Insert; returns the slot the key occupies (new or existing) and sets *added
// when this call placed it; NONE when the table is full.
__device__ __forceinline__ uint32_t hset_insert(uint32_t *keys, uint32_t cap, uint32_t key, bool *added) {
  uint32_t s = hslot(key, cap);
  *added = false;
  for (uint32_t probe = 0; probe < cap; ++probe) {
    uint32_t old = atomicCAS(&keys[s], NONE, key);
    if (old == NONE) {
      *added = true;
      return s;
    }
    if (old == key) return s;
    s = (s + 1) & (cap - 1);
  }
  return NONE;
}

// Warp-aggregated test-and-set of bit b in a shared bitmap: lanes hitting the
// same 32-bit word combine into one atomicOr.  Returns true if the block was
// already present (set before, or by a lower lane of this warp step).
__device__ __forceinline__ bool warp_test_and_set(uint32_t *bitmap, uint32_t b, bool valid) {
  const uint32_t lane = threadIdx.x & 31;
  const uint32_t w = valid ? (b >> 5) : 0xFFFFFFFFu;
  const uint32_t bit = valid ? 1u << (b & 31) : 0u;
  // walk lists are mostly runs of consecutive blocks: when the warp's words
  // are lane 0's word and the next one, two ballots group the lanes (no MATCH)
  const uint32_t w0 = __shfl_sync(0xffffffffu, w, 0);
  const bool in0 = w == w0;
  uint32_t grp;
  if (__all_sync(0xffffffffu, in0 || w == w0 + 1 || w == 0xFFFFFFFFu)) {
    const uint32_t m0 = __ballot_sync(0xffffffffu, in0), m1 = __ballot_sync(0xffffffffu, w == w0 + 1);
    grp = in0 ? m0 : (w == w0 + 1 ? m1 : ~(m0 | m1));
  } else {
    grp = __match_any_sync(0xffffffffu, w);
  }
  const uint32_t comb = __reduce_or_sync(grp, bit);
  const uint32_t leader = __ffs(grp) - 1;
  uint32_t old = 0;
  if (lane == leader && valid) old = atomicOr(&bitmap[w], comb);
  old = __shfl_sync(0xffffffffu, old, leader);
  bool dup = valid && (old & bit);
  if (__popc(comb) < __popc(grp) && valid) {
    // two lanes carry the same block: all but the lowest are duplicates
    const uint32_t same = __match_any_sync(grp, b);
    dup |= lane != (uint32_t)(__ffs(same) - 1);
  }
  return dup;
}

__device__ __forceinline__ uint32_t pow2ceil(uint32_t x) {
  return x <= 1 ? 1u : 1u << (32 - __clz(x - 1));
}

}  // namespace dum
