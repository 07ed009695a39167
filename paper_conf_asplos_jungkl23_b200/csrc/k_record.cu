// a1 + a2: fault-trace ingest and the execution ID table.
//
//  k_ingest        one CTA per launch: first-occurrence dedupe of the launch's
//                  fault records (PAPER.md L124 step (2): the driver "removes the
//                  duplicate addresses and groups them according to their UM
//                  blocks"; reading D2) with an order-preserving block scan, and
//                  the launch's probe of the execution ID table (PAPER.md:
//                  "looks up the execution ID table to find the command of the
//                  same hash value").
//  k_exec_assign   one CTA: new hashes get dense IDs in first-seen order
//                  ("Otherwise, it assigns a new execution ID", PAPER.md L136;
//                  D3) = rank of each new hash by its minimum launch position
//                  (order-independent).
#include <algorithm>

#include "device_util.cuh"
#include "kernels.cuh"

namespace dum {

constexpr int INGEST_NT = 256;
constexpr uint32_t INGEST_HCAP = 2048;  // smem hash capacity (n <= 1024 in smem): 16 KB, 8 CTAs / SM
constexpr uint32_t IDCAP = 1024;        // repeated-block hash of the bitmap path
constexpr uint32_t INGEST_SMEM_MAX = 24 * 1024;  // bitmap (exact for small W, else hashed) + dup hash

// bit of block b in a hashed bitmap of 2^k bits: runs of consecutive blocks
// stay consecutive (the warp's word grouping), far regions land at
// pseudo-random offsets.  A shared bit is only a candidate repeat: the
// min-position hash then settles it exactly.
__device__ __forceinline__ uint32_t bm_bit(uint32_t b, uint32_t nbits) {
  return (b + (b / nbits) * 0x9E3779B1u) & (nbits - 1);
}

__global__ void __launch_bounds__(INGEST_NT) k_ingest(
    const uint64_t *__restrict__ hash, const uint64_t *__restrict__ off, const uint32_t *__restrict__ faults,
    uint32_t n_launch, uint32_t W, uint32_t l0, uint64_t f0, uint64_t *__restrict__ stage_hash,
    uint64_t *__restrict__ stage_off, uint32_t *__restrict__ stage_norm, uint32_t *__restrict__ stage_cnt,
    uint32_t *__restrict__ stage_slot, unsigned long long *exec_keys, uint32_t *exec_vals, uint32_t *exec_minpos,
    uint32_t exec_cap, uint32_t *big_pool, uint64_t big_entries, uint32_t bm_words, bool bm_hashed,
    uint32_t *__restrict__ stage_exec,
    uint32_t *__restrict__ out_exec, uint32_t *__restrict__ pend, uint32_t Emax, uint64_t n_fault, DevState *st) {
  extern __shared__ uint32_t dyn[];  // hash (2 x INGEST_HCAP) or bitmap + small dup hash
  __shared__ uint32_t ws[INGEST_NT / 32];
  __shared__ uint32_t s_dups, s_ovf;
  const uint32_t i = blockIdx.x;
  if (i >= n_launch) return;
  uint64_t a = off[i], b = off[i + 1];
  if (b < a || b > n_fault || (i == 0 && a != 0)) {
    // offsets not monotone / past the batch: the launch is dropped (sticky EINVAL)
    if (threadIdx.x == 0) set_err(st, ERR_EINVAL);
    a = b = 0;
  }
  const uint32_t n = (uint32_t)(b - a);
  if (threadIdx.x == 0) {
    stage_hash[l0 + i] = hash[i];
    stage_off[l0 + i] = f0 + a;
    ctr_add(st, DUM_CTR_LAUNCHES, 1);
    s_dups = 0;
  }
  if (threadIdx.x == 0) {
    // execution ID table probe (insert if absent), PAPER.md L136 -- issued
    // first so that its atomics overlap the record dedupe below.  A known hash
    // gets its ID here; a hash first seen in this batch is PENDING and queued
    // for k_exec_assign.
    const uint64_t h = hash[i];
    uint32_t slot = NONE;
    if (h == EMPTY64) {
      slot = exec_cap;  // sentinel-key slot; exec_keys[exec_cap] is a presence word
      atomicCAS(&exec_keys[exec_cap], 0ull, 1ull);
    } else {
      uint32_t s = (uint32_t)fmix64(h) & (exec_cap - 1);
      for (uint32_t p = 0; p < exec_cap; ++p) {
        const unsigned long long old = atomicCAS(&exec_keys[s], EMPTY64, (unsigned long long)h);
        if (old == EMPTY64 || old == h) {
          slot = s;
          break;
        }
        s = (s + 1) & (exec_cap - 1);
      }
    }
    uint32_t id = NONE;
    if (slot == NONE) {
      set_err(st, ERR_ECAPACITY, 2ull * exec_cap);
    } else if ((id = ((volatile uint32_t *)exec_vals)[slot]) == PENDING) {
      atomicMin(&exec_minpos[slot], i);
      pend[atomicAdd(&st->n_pend, 1u)] = i;
    }
    if (id != PENDING) {
      if (id != NONE && id >= Emax) id = NONE;
      stage_exec[l0 + i] = id;
      if (out_exec) out_exec[i] = id;
    }
    stage_slot[l0 + i] = slot;
  }
  // Big launches (> INGEST_HCAP/2 records) dedupe through a bitmap: over the
  // block-id space when it fits the shared-memory budget, else hashed
  // (bm_bit).  An order-free warp-aggregated test-and-set finds the records
  // whose bit was already set (normally none: the input is then copied);
  // only those blocks go through a small min-position hash, which keeps the
  // first occurrence of each.  A private global-pool hash takes launches
  // whose candidates overflow it.
  const bool use_bitmap = n > INGEST_HCAP / 2 && bm_words != 0;
  if (n > 0 && use_bitmap) {
    uint32_t *bm = dyn, *dk = dyn + ((bm_words + 3) & ~3u), *dv = dk + IDCAP;
    for (uint32_t t = threadIdx.x; t < bm_words; t += INGEST_NT) bm[t] = 0;
    for (uint32_t t = threadIdx.x; t < IDCAP; t += INGEST_NT) {
      dk[t] = NONE;
      dv[t] = NONE;
    }
    if (threadIdx.x == 0) s_ovf = 0;
    __syncthreads();
    uint32_t ndup = 0;
    for (uint32_t c = 0; c < n; c += INGEST_NT) {
      const uint32_t j = c + threadIdx.x;
      uint32_t blk = j < n ? faults[a + j] : NONE;
      const bool inr = j < n && blk < W;
      if (j < n && blk >= W) {
        set_err(st, ERR_EINVAL);
        ++ndup;  // dropped: take the compaction path
      }
      if (warp_test_and_set(bm, bm_hashed && inr ? bm_bit(blk, bm_words * 32) : blk, inr)) {
        ++ndup;
        if (!hmap_insert_min(dk, dv, IDCAP, blk, j)) s_ovf = 1;
      }
    }
    if (ndup) s_dups = 1;
    __syncthreads();
    uint32_t run = n;
    if (!s_dups) {
      for (uint32_t j = threadIdx.x; j < n; j += INGEST_NT) stage_norm[f0 + a + j] = faults[a + j];
    } else if (!s_ovf) {
      // every occurrence of a repeated block lowers that block's min position
      for (uint32_t j = threadIdx.x; j < n; j += INGEST_NT) {
        const uint32_t blk = faults[a + j];
        if (blk >= W) continue;
        for (uint32_t p = 0, sl = hslot(blk, IDCAP); p < IDCAP; ++p, sl = (sl + 1) & (IDCAP - 1)) {
          const uint32_t kk = dk[sl];
          if (kk == NONE) break;
          if (kk == blk) {
            atomicMin(&dv[sl], j);
            break;
          }
        }
      }
      __syncthreads();
      run = 0;
      for (uint32_t c = 0; c < n; c += INGEST_NT) {
        const uint32_t j = c + threadIdx.x;
        uint32_t blk = NONE, keep = 0;
        if (j < n) {
          blk = faults[a + j];
          if (blk < W) {
            const uint32_t m = hmap_get(dk, dv, IDCAP, blk);
            keep = m == NONE || m == j;
          }
        }
        uint32_t tot;
        const uint32_t pre = block_excl_scan(keep, ws, &tot);
        if (keep) stage_norm[f0 + a + run + pre] = blk;
        run += tot;
      }
    }
    if (!s_dups || !s_ovf) {
      if (threadIdx.x == 0) {
        if (run < n) ctr_add(st, DUM_CTR_INGEST_DUP, 1);
        stage_cnt[l0 + i] = run;
        ctr_add(st, DUM_CTR_RAW_RECORDS, n);
        ctr_add(st, DUM_CTR_NORM_RECORDS, run);
      }
    }
  }
  if (n > 0 && (!use_bitmap || (s_dups && s_ovf))) {
    // hash of (block -> first position) in shared memory, or in a private
    // region of the global pool for launches with > INGEST_HCAP/2 records
    uint32_t *keys = dyn, *vals = dyn + INGEST_HCAP;
    uint32_t cap = pow2ceil(2 * n);
    if (cap < 64) cap = 64;
    bool fits = true;
    if (n > INGEST_HCAP / 2) {
      const uint64_t pbase = 4ull * (f0 + a);  // region [4(f0+a), 4(f0+b)) holds >= cap entries
      if (pbase + cap > big_entries) {
        if (threadIdx.x == 0) set_err(st, ERR_ECAPACITY, pbase + cap);
        fits = false;
      }
      keys = big_pool + 2ull * pbase;
      vals = keys + cap;
    }
    __syncthreads();
    if (threadIdx.x == 0) s_dups = 0;
    if (fits) {
      for (uint32_t t = threadIdx.x; t < cap; t += INGEST_NT) {
        keys[t] = NONE;
        vals[t] = NONE;
      }
      __syncthreads();
      bool dup = false;
      for (uint32_t j = threadIdx.x; j < n; j += INGEST_NT) {
        const uint32_t blk = faults[a + j];
        if (blk >= W) {
          set_err(st, ERR_EINVAL);
          dup = true;  // dropped: take the compaction path
          continue;
        }
        // first-occurrence test: insert (block -> min position)
        uint32_t s = hslot(blk, cap);
        for (uint32_t p = 0; p < cap; ++p) {
          const uint32_t old = atomicCAS(&keys[s], NONE, blk);
          if (old == NONE || old == blk) {
            dup |= old == blk;
            atomicMin(&vals[s], j);
            break;
          }
          s = (s + 1) & (cap - 1);
        }
      }
      if (dup) s_dups = 1;
      __syncthreads();
      if (threadIdx.x == 0 && s_dups) ctr_add(st, DUM_CTR_INGEST_DUP, 1);
      uint32_t run = n;
      if (!s_dups) {
        // no duplicate record in this launch: the normalised list is the input
        for (uint32_t j = threadIdx.x; j < n; j += INGEST_NT) stage_norm[f0 + a + j] = faults[a + j];
      } else {
        // order-preserving compaction of first occurrences
        run = 0;
        for (uint32_t c = 0; c < n; c += INGEST_NT) {
          const uint32_t j = c + threadIdx.x;
          uint32_t blk = NONE, keep = 0;
          if (j < n) {
            blk = faults[a + j];
            keep = blk < W && hmap_get(keys, vals, cap, blk) == j;
          }
          uint32_t tot;
          const uint32_t pre = block_excl_scan(keep, ws, &tot);
          if (keep) stage_norm[f0 + a + run + pre] = blk;
          run += tot;
        }
      }
      if (threadIdx.x == 0) {
        stage_cnt[l0 + i] = run;
        ctr_add(st, DUM_CTR_RAW_RECORDS, n);
        ctr_add(st, DUM_CTR_NORM_RECORDS, run);
      }
    } else if (threadIdx.x == 0) {
      stage_cnt[l0 + i] = 0;
    }
  } else if (n == 0 && threadIdx.x == 0) {
    stage_cnt[l0 + i] = 0;
  }
}

constexpr int ASSIGN_NT = 1024;

__global__ void __launch_bounds__(ASSIGN_NT) k_exec_assign(
    uint32_t n_launch, uint32_t l0, const uint32_t *__restrict__ stage_slot, const uint64_t *__restrict__ stage_hash,
    uint32_t *exec_vals, uint32_t *exec_minpos, uint64_t *exec_hash, uint32_t *__restrict__ stage_exec,
    uint32_t *__restrict__ out_exec, const uint32_t *__restrict__ pend, uint32_t Emax, DevState *st) {
  __shared__ uint32_t ws[ASSIGN_NT / 32];
  __shared__ uint32_t s_first[2 * ASSIGN_NT], s_nf;
  const uint32_t E0 = st->E;
  const uint32_t npend = *(volatile uint32_t *)&st->n_pend;
  if (npend <= 2 * ASSIGN_NT) {
    // Only the launches whose hash was first seen in this batch (k_ingest
    // queued them).  New IDs go to the first occurrences in launch order:
    // rank = first occurrences at an earlier position (the queue is short).
    if (threadIdx.x == 0) s_nf = 0;
    __syncthreads();
    uint32_t mine[2], nm = 0;
    for (uint32_t t = threadIdx.x; t < npend; t += ASSIGN_NT) {
      const uint32_t i = pend[t], slot = stage_slot[l0 + i];
      if (slot != NONE && ((volatile uint32_t *)exec_minpos)[slot] == i) {
        mine[nm++] = i;
        s_first[atomicAdd(&s_nf, 1u)] = i;
      }
    }
    __syncthreads();
    const uint32_t nf = s_nf;
    for (uint32_t k = 0; k < nm; ++k) {
      const uint32_t i = mine[k], slot = stage_slot[l0 + i];
      uint32_t r = 0;
      for (uint32_t q = 0; q < nf; ++q) r += s_first[q] < i;
      const uint32_t id = E0 + r;
      exec_vals[slot] = id;
      exec_minpos[slot] = NONE;
      if (id < Emax) exec_hash[id] = stage_hash[l0 + i];
    }
    __syncthreads();
    for (uint32_t t = threadIdx.x; t < npend; t += ASSIGN_NT) {
      const uint32_t i = pend[t], slot = stage_slot[l0 + i];
      uint32_t id = slot == NONE ? NONE : ((volatile uint32_t *)exec_vals)[slot];
      if (id != NONE && id >= Emax) id = NONE;
      stage_exec[l0 + i] = id;
      if (out_exec) out_exec[i] = id;
    }
    if (threadIdx.x == 0) {
      uint32_t E = E0 + nf;
      if (E > Emax) {
        set_err(st, ERR_ECAPACITY, E);
        E = Emax;
      }
      st->E = E;
      st->n_pend = 0;
    }
    return;
  }
  // long queue (a first batch): scan every launch of the batch
  uint32_t base = 0;
  for (uint32_t c = 0; c < n_launch; c += ASSIGN_NT) {
    const uint32_t i = c + threadIdx.x;
    uint32_t flag = 0, slot = NONE;
    if (i < n_launch) {
      slot = stage_slot[l0 + i];
      if (slot != NONE)
        flag = ((volatile uint32_t *)exec_vals)[slot] == PENDING &&
               ((volatile uint32_t *)exec_minpos)[slot] == i;
    }
    uint32_t tot;
    uint32_t pre = block_excl_scan(flag, ws, &tot);
    if (flag) {
      uint32_t id = E0 + base + pre;
      exec_vals[slot] = id;
      exec_minpos[slot] = NONE;
      if (id < Emax) exec_hash[id] = stage_hash[l0 + i];
    }
    base += tot;
  }
  __syncthreads();
  for (uint32_t i = threadIdx.x; i < n_launch; i += ASSIGN_NT) {
    uint32_t slot = stage_slot[l0 + i];
    uint32_t id = slot == NONE ? NONE : ((volatile uint32_t *)exec_vals)[slot];
    if (id != NONE && id >= Emax) id = NONE;
    stage_exec[l0 + i] = id;
    if (out_exec) out_exec[i] = id;
  }
  if (threadIdx.x == 0) {
    uint32_t E = E0 + base;
    if (E > Emax) {
      set_err(st, ERR_ECAPACITY, E);
      E = Emax;
    }
    st->E = E;
    st->n_pend = 0;
  }
}

cudaError_t launch_record(dum_engine *e, const uint64_t *hash, const uint64_t *off, uint32_t n_launch,
                          const uint32_t *faults, uint64_t n_fault, uint32_t *out_exec, cudaStream_t s) {
  if (n_launch == 0) return cudaSuccess;
  {
  TimerScope t(e, DUM_T_INGEST, s);
  // the bitmap: exact over [0, W) when it fits, else the largest power-of-two
  // word count that does (hashed)
  uint32_t bmw = (e->g.W + 31) / 32;
  const bool bm_hashed = (size_t)((bmw + 3) & ~3u) * 4 + 2 * IDCAP * 4 > INGEST_SMEM_MAX;
  if (bm_hashed) {
    bmw = 1;
    while ((size_t)(2 * bmw) * 4 + 2 * IDCAP * 4 <= INGEST_SMEM_MAX) bmw *= 2;
  }
  const size_t bm_bytes = (size_t)((bmw + 3) & ~3u) * 4 + 2 * IDCAP * 4;
  const size_t smem = std::max<size_t>(2 * INGEST_HCAP * 4, bm_bytes);
  // the attribute is per device and function: raised by every engine on its own device
  if ((int)smem > e->ingest_smem) {
    cudaFuncSetAttribute(k_ingest, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    e->ingest_smem = (int)smem;
  }
  k_ingest<<<n_launch, INGEST_NT, smem, s>>>(hash, off, faults, n_launch, e->g.W, e->n_staged, e->staged_faults,
                                             e->d_stage_hash, e->d_stage_off, e->d_stage_norm, e->d_stage_cnt,
                                             e->d_stage_slot, e->d_exec_keys, e->d_exec_vals, e->d_exec_minpos,
                                             e->exec_cap, e->d_ingest_pool, e->big_pool_entries, bmw, bm_hashed,
                                             e->d_stage_exec, out_exec, e->d_pend, e->g.Emax, n_fault, e->d_state);
  }
  TimerScope t(e, DUM_T_EXEC_ASSIGN, s);
  k_exec_assign<<<1, ASSIGN_NT, 0, s>>>(n_launch, e->n_staged, e->d_stage_slot, e->d_stage_hash, e->d_exec_vals,
                                        e->d_exec_minpos, e->d_exec_hash, e->d_stage_exec, out_exec, e->d_pend, e->g.Emax,
                                        e->d_state);
  e->kernel_launches += 2;
  return cudaGetLastError();
}

}  // namespace dum
