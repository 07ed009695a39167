// the closed loop on the GPU (dum_simulate).
//
// The paper's runtime interleaves demand migration, table updates, prediction
// and prefetch per kernel: the fault-handling thread
// hands faults to the migration thread with the highest priority (L158), the
// correlator updates the tables (L154), the prefetching thread chains ahead
// (L156, L218-L224) and pre-evicts when memory runs out (L236-L243),
// invalidating victims of inactive PT blocks (L285).  dum_simulate replays an
// access stream through exactly that loop, launch by launch, with every step
// in this library's kernels and no host round trip (all list sizes stay on
// the device):
//   1. faults = the launch's accesses without a frame (first occurrence, D2)
//   2. record_faults(launch)                                   (a1, a2)
//   3. demand: if the faults exceed the free frames, LRM victims that the
//      launch does not access (D22) -> write-back / invalidate; then H2D of
//      the faults                                              (a8 rule, a9)
//   4. build_tables                                            (a3 - a6)
//   5. transition query for the next launch (its exec ID if its hash is
//      known; the last three exec IDs as history)             (a7)
//   6. pre-eviction of the window (DUM_SIM_PREEVICT)          (a8)
//   7. H2D of the window's non-resident blocks: with pre-eviction the prefix
//      that fits the free frames; without it (prefetch only) all of them, the
//      driver evicting least-recently-migrated blocks for those beyond the
//      free frames, window or not (the driver's policy
//      "evicts pages that are least recently migrated", which is what
//      pre-eviction avoids)
// Without a data plane (B/G: 720 GB do not fit host memory) the migrations
// move the residency only; with one (T) the bytes move too.  Flags select the
// Fig. 10 ablation: no prefetch (naive UM), prefetch,
// + pre-eviction, + invalidation.
#include <algorithm>
#include <vector>

#include "device_util.cuh"
#include "kernels.cuh"
#include "predict.cuh"
#include "select_tail.cuh"

namespace dum {

constexpr int SIM_NT = 1024;
constexpr uint32_t SIM_HCAP = 16384;  // launch accesses <= SIM_HCAP / 2 (shared first-position hash, 128 KiB)

// 1. faults of one launch: its accesses without a frame, first occurrence,
// in access order; marks the launch's access set in acc_bits (demand rule D22).
__global__ void __launch_bounds__(SIM_NT) k_sim_faults(const uint32_t *__restrict__ acc, uint32_t n, uint32_t W,
                                                       const uint32_t *__restrict__ res_bits, uint32_t *acc_bits,
                                                       uint32_t *faults, uint64_t *foff, dum_sim_stats *stats,
                                                       DevState *st) {
  extern __shared__ uint32_t sh[];  // keys | min positions
  __shared__ uint32_t ws[SIM_NT / 32];
  uint32_t *hk = sh, *hv = sh + SIM_HCAP;
  const uint32_t tid = threadIdx.x;
  if (n > SIM_HCAP / 2) {
    if (tid == 0) {
      set_err(st, ERR_ECAPACITY, n);
      foff[0] = foff[1] = 0;
    }
    return;
  }
  uint32_t cap = pow2ceil(2 * n);
  if (cap < 64) cap = 64;
  for (uint32_t p = tid; p < cap; p += SIM_NT) {
    hk[p] = NONE;
    hv[p] = NONE;
  }
  __syncthreads();
  for (uint32_t j = tid; j < n; j += SIM_NT) {
    const uint32_t b = acc[j];
    if (b >= W) {
      set_err(st, ERR_EINVAL);
      continue;
    }
    hmap_insert_min(hk, hv, cap, b, j);
    atomicOr(&acc_bits[b >> 5], 1u << (b & 31));
  }
  __syncthreads();
  uint32_t run = 0;
  for (uint32_t c = 0; c < n; c += SIM_NT) {
    const uint32_t j = c + tid;
    uint32_t b = NONE, keep = 0;
    if (j < n) {
      b = acc[j];
      keep = b < W && hmap_get(hk, hv, cap, b) == j && !((res_bits[b >> 5] >> (b & 31)) & 1u);
    }
    uint32_t tot;
    const uint32_t pre = block_excl_scan(keep, ws, &tot);
    if (keep) faults[run + pre] = b;
    run += tot;
  }
  if (tid == 0) {
    foff[0] = 0;
    foff[1] = run;
    stats->faults = run;
  }
}

// 3. demand victims (D22): need = faults - free frames; the first `need`
// entries of the LRM log not accessed by the launch, split by PT-block
// inactivity (L285) -- the selection of select_tail.cuh with the launch's
// access set as the window.
constexpr int DEM_NT = 512;  // select_tail chunk = DEM_NT * 8 <= SEL_CHUNK

__global__ void __launch_bounds__(DEM_NT) k_sim_demand(SelectOut so, const uint32_t *acc_bits, const uint64_t *foff,
                                                       DevState *st) {
  __shared__ SelShared ss;
  __shared__ uint32_t stage[SEL_CHUNK];
  const uint32_t tid = threadIdx.x;
  if (tid == 0) {
    const uint32_t nf = (uint32_t)foff[1];
    const uint32_t nfree = *(volatile uint32_t *)&st->free_count;
    const uint32_t need = nf > nfree ? nf - nfree : 0;
    ss.need = need;
    ss.ok = need <= so.cap;
    ss.bwb = ss.binv = 0;
    ss.head = *(volatile uint32_t *)&st->lrm_head;
    ss.tail = *(volatile uint32_t *)&st->lrm_tail;
    ss.clean = *(volatile uint32_t *)&st->log_dirty == 0;
    if (!ss.ok) set_err(st, ERR_ECAPACITY, need);
  }
  __syncthreads();
  select_tail<DEM_NT, 0>(so, 0, ss, InBlockBitmap{acc_bits}, st, tid, stage);
}

// 5. the transition query for launch k+1: its exec ID if the hash is in the
// execution ID table (else no window), the last three exec IDs (build's
// history register) as history, no anchor (D14).
__global__ void k_sim_query(const uint64_t *hash_next, const unsigned long long *exec_keys,
                            const uint32_t *exec_vals, uint32_t exec_cap, uint32_t degree, dum_query *q,
                            const DevState *st) {
  if (threadIdx.x != 0) return;
  const uint64_t h = *hash_next;
  uint32_t id = NONE;
  if (h == EMPTY64) {
    if (exec_keys[exec_cap] != 0ull) id = exec_vals[exec_cap];
  } else {
    uint32_t s = (uint32_t)fmix64(h) & (exec_cap - 1);
    for (uint32_t p = 0; p < exec_cap; ++p) {
      const unsigned long long k = exec_keys[s];
      if (k == h) {
        id = exec_vals[s];
        break;
      }
      if (k == EMPTY64) break;
      s = (s + 1) & (exec_cap - 1);
    }
  }
  if (id == PENDING) id = NONE;
  dum_query Q;
  Q.exec = id;
  Q.hist[0] = st->hist[1];
  Q.hist[1] = st->hist[2];
  Q.hist[2] = st->hist[3];
  Q.anchor = NONE;
  Q.n = degree;
  *q = Q;
}

// 7. the window's blocks without a frame, in window order: as many as there
// are free frames, or (driver eviction) as there are frames.
__global__ void __launch_bounds__(SIM_NT) k_sim_prefetch(const uint32_t *__restrict__ pairs,
                                                         const uint64_t *__restrict__ prange,
                                                         const uint32_t *__restrict__ res_bits, uint32_t *pf,
                                                         uint64_t *pf_range, uint32_t driver_evict, DevState *st) {
  __shared__ uint32_t ws[SIM_NT / 32];
  const uint32_t tid = threadIdx.x;
  const uint64_t a = prange[0], b = prange[1];
  const uint32_t nfree = __ldcg(&st->free_count) + (driver_evict ? __ldcg(&st->n_resident) : 0u);
  uint32_t run = 0;
  for (uint64_t c = a; c < b && run < nfree; c += SIM_NT) {
    const uint64_t i = c + tid;
    uint32_t blk = NONE, keep = 0;
    if (i < b) {
      blk = pairs[2 * i];
      keep = !((res_bits[blk >> 5] >> (blk & 31)) & 1u);
    }
    uint32_t tot;
    const uint32_t pre = block_excl_scan(keep, ws, &tot);
    if (keep && run + pre < nfree) pf[run + pre] = blk;
    run += tot;
  }
  if (tid == 0) {
    pf_range[0] = 0;
    pf_range[1] = min(run, nfree);
  }
}

// 7'. prefetch only: the driver's victims for the prefetched blocks beyond the
// free frames -- the first entries of the LRM log, no exclusion.
struct NoneExcluded {
  __device__ __forceinline__ uint32_t operator()(uint32_t, uint32_t) const { return 0u; }
};

__global__ void __launch_bounds__(DEM_NT) k_sim_driver_evict(SelectOut so, const uint64_t *pf_range, DevState *st) {
  __shared__ SelShared ss;
  __shared__ uint32_t stage[SEL_CHUNK];
  const uint32_t tid = threadIdx.x;
  if (tid == 0) {
    const uint32_t npf = (uint32_t)(pf_range[1] - pf_range[0]);
    const uint32_t nfree = __ldcg(&st->free_count);
    const uint32_t need = npf > nfree ? npf - nfree : 0;
    ss.need = need;
    ss.ok = need <= so.cap;
    ss.bwb = ss.binv = 0;
    ss.head = __ldcg(&st->lrm_head);
    ss.tail = __ldcg(&st->lrm_tail);
    ss.clean = __ldcg(&st->log_dirty) == 0;
    if (!ss.ok) set_err(st, ERR_ECAPACITY, need);
  }
  __syncthreads();
  select_tail<DEM_NT, 0>(so, 0, ss, NoneExcluded{}, st, tid, stage);
}

// launch statistics from the lists' ranges; clears the launch's access set
__global__ void k_sim_close(const uint32_t *__restrict__ acc, uint32_t n, uint32_t W, uint32_t *acc_bits,
                            const uint64_t *dem_rng, const uint64_t *pre_rng, const uint64_t *pf_range,
                            uint32_t evicted, uint32_t prefetch, uint32_t invalidate, dum_sim_stats *stats) {
  const uint32_t tid = blockIdx.x * blockDim.x + threadIdx.x;
  for (uint32_t j = tid; j < n; j += gridDim.x * blockDim.x) {
    const uint32_t b = acc[j];
    if (b < W) atomicAnd(&acc_bits[b >> 5], ~(1u << (b & 31)));
  }
  if (tid == 0) {
    // without DUM_SIM_INVALIDATE the inactive victims were written back too
    const uint32_t dw = (uint32_t)(dem_rng[1] - dem_rng[0]), di = (uint32_t)(dem_rng[3] - dem_rng[2]);
    // pre-eviction (or, prefetch only, the driver's evictions for the prefetch)
    const uint32_t pw = evicted ? (uint32_t)(pre_rng[1] - pre_rng[0]) : 0u;
    const uint32_t pi = evicted ? (uint32_t)(pre_rng[3] - pre_rng[2]) : 0u;
    stats->demand_wb = invalidate ? dw : dw + di;
    stats->demand_inv = invalidate ? di : 0u;
    stats->pre_wb = invalidate ? pw : pw + pi;
    stats->pre_inv = invalidate ? pi : 0u;
    stats->prefetched = prefetch ? (uint32_t)(pf_range[1] - pf_range[0]) : 0u;
  }
}

__global__ void k_sim_zero_ranges(uint64_t *r, uint32_t n) {
  if (threadIdx.x < n) r[threadIdx.x] = 0;
}

static cudaError_t ensure_sim(dum_engine *e, uint32_t max_acc) {
  if (e->sim_ready && max_acc <= e->sim_acc_cap) return cudaSuccess;
  const Geo &g = e->g;
  cudaError_t err = cudaSuccess;
  auto A = [&](cudaError_t x) {
    if (err == cudaSuccess) err = x;
  };
  cudaDeviceSynchronize();
  void *ptrs[] = {e->sim_acc_bits, e->sim_faults, e->sim_foff, e->sim_q, e->sim_pairs, e->sim_ranges, e->sim_wb,
                  e->sim_inv, e->sim_pf};
  for (void *p : ptrs)
    if (p) cudaFree(p);
  e->sim_acc_cap = std::max<uint32_t>(max_acc, 1024);
  e->sim_pair_cap = (uint64_t)(g.N + 1) * g.walk_cap + 64;
  A(cudaMalloc((void **)&e->sim_acc_bits, 4ull * ((g.W + 31) / 32)));
  A(cudaMalloc((void **)&e->sim_faults, 4ull * e->sim_acc_cap));
  A(cudaMalloc((void **)&e->sim_foff, 16));
  A(cudaMalloc((void **)&e->sim_q, sizeof(dum_query)));
  A(cudaMalloc((void **)&e->sim_pairs, 8ull * e->sim_pair_cap));
  A(cudaMalloc((void **)&e->sim_ranges, 8ull * 16));  // pairs(2) | demand(4) | pre(4) | prefetch(2) | kern scratch
  A(cudaMalloc((void **)&e->sim_wb, 4ull * g.C + 64));
  A(cudaMalloc((void **)&e->sim_inv, 4ull * g.C + 64));
  A(cudaMalloc((void **)&e->sim_pf, 4ull * g.C + 64));
  if (err == cudaSuccess) err = cudaMemset(e->sim_acc_bits, 0, 4ull * ((g.W + 31) / 32));
  if (err == cudaSuccess) err = cudaMemset(e->sim_ranges, 0, 8ull * 16);
  if (err == cudaSuccess) err = cudaFuncSetAttribute(k_sim_faults, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                                     (int)(2 * SIM_HCAP * 4));
  e->sim_ready = err == cudaSuccess;
  return err;
}

cudaError_t launch_simulate(dum_engine *e, const uint64_t *hash, uint32_t n_launch, const uint64_t *acc_off,
                            const uint32_t *acc_blk, uint32_t n_kernels, uint32_t degree, uint32_t flags,
                            dum_sim_stats *stats, cudaStream_t s) {
  uint32_t max_acc = 0;
  for (uint32_t j = 0; j < n_kernels; ++j) max_acc = std::max<uint32_t>(max_acc, (uint32_t)(acc_off[j + 1] - acc_off[j]));
  if (max_acc > SIM_HCAP / 2) return cudaErrorInvalidValue;
  cudaError_t err = ensure_sim(e, max_acc);
  if (err != cudaSuccess) return err;
  const Geo &g = e->g;
  const bool prefetch = flags & DUM_SIM_PREFETCH, preevict = prefetch && (flags & DUM_SIM_PREEVICT);
  const bool invalidate = flags & DUM_SIM_INVALIDATE;
  uint64_t *r_pairs = e->sim_ranges, *r_dem = e->sim_ranges + 2, *r_pre = e->sim_ranges + 6,
           *r_pf = e->sim_ranges + 10;
  SelectOut dem = make_select_out(e, e->sim_wb, e->sim_inv, g.C, r_dem);
  SelectOut pre = make_select_out(e, e->sim_wb, e->sim_inv, g.C, r_pre);
  for (uint32_t k = 0; k < n_launch; ++k) {
    const uint32_t j = k % n_kernels;
    const uint32_t n = (uint32_t)(acc_off[j + 1] - acc_off[j]);
    const uint32_t *acc = acc_blk + acc_off[j];
    // 1. faults of the launch
    k_sim_faults<<<1, SIM_NT, 2 * SIM_HCAP * 4, s>>>(acc, n, g.W, e->d_res_bits, e->sim_acc_bits, e->sim_faults,
                                                    e->sim_foff, stats + k, e->d_state);
    // 2. record (one launch; the fault count stays on the device)
    if ((uint64_t)e->n_staged + 1 > e->stage_launch_cap || e->staged_faults + n > e->stage_fault_cap)
      return cudaErrorInvalidValue;
    if ((err = launch_record(e, hash + k, e->sim_foff, 1, e->sim_faults, n, nullptr, s)) != cudaSuccess) return err;
    e->n_staged += 1;
    e->staged_faults += n;
    e->launches += 1;
    // 3. demand path: victims the launch does not touch, then the faults in
    k_sim_demand<<<1, DEM_NT, 0, s>>>(dem, e->sim_acc_bits, e->sim_foff, e->d_state);
    if ((err = launch_migrate(e, DUM_D2H, e->sim_wb, nullptr, g.C, 1, s, r_dem)) != cudaSuccess) return err;
    if ((err = launch_migrate(e, invalidate ? DUM_INVALIDATE : DUM_D2H, e->sim_inv, nullptr, g.C, 1, s,
                              r_dem + 2)) != cudaSuccess)
      return err;
    if ((err = launch_migrate(e, DUM_H2D, e->sim_faults, nullptr, g.C, 1, s, e->sim_foff)) != cudaSuccess)
      return err;
    // 4. tables
    if ((err = launch_build(e, s)) != cudaSuccess) return err;
    e->n_staged = 0;
    e->staged_faults = 0;
    e->built_launches = e->launches;
    // 5 - 7. the window of the next launch: pre-eviction, prefetch
    if (prefetch && k + 1 < n_launch) {
      k_sim_query<<<1, 32, 0, s>>>(hash + k + 1, e->d_exec_keys, e->d_exec_vals, e->exec_cap, degree, e->sim_q,
                                   e->d_state);
      if ((err = launch_predict(e, e->sim_q, 1, e->sim_pairs, e->sim_pair_cap, r_pairs, nullptr, nullptr, nullptr,
                                preevict ? &pre : nullptr, nullptr, s)) != cudaSuccess)
        return err;
      if (preevict) {
        if ((err = launch_migrate(e, DUM_D2H, e->sim_wb, nullptr, g.C, 1, s, r_pre)) != cudaSuccess) return err;
        if ((err = launch_migrate(e, invalidate ? DUM_INVALIDATE : DUM_D2H, e->sim_inv, nullptr, g.C, 1, s,
                                  r_pre + 2)) != cudaSuccess)
          return err;
      }
      k_sim_prefetch<<<1, SIM_NT, 0, s>>>(e->sim_pairs, r_pairs, e->d_res_bits, e->sim_pf, r_pf, preevict ? 0u : 1u,
                                          e->d_state);
      if (!preevict) {  // prefetch only: the driver evicts for the blocks beyond the free frames
        k_sim_driver_evict<<<1, DEM_NT, 0, s>>>(pre, r_pf, e->d_state);
        if ((err = launch_migrate(e, DUM_D2H, e->sim_wb, nullptr, g.C, 1, s, r_pre)) != cudaSuccess) return err;
        if ((err = launch_migrate(e, invalidate ? DUM_INVALIDATE : DUM_D2H, e->sim_inv, nullptr, g.C, 1, s,
                                  r_pre + 2)) != cudaSuccess)
          return err;
      }
      if ((err = launch_migrate(e, DUM_H2D, e->sim_pf, nullptr, g.C, 1, s, r_pf)) != cudaSuccess) return err;
    }
    k_sim_close<<<8, 256, 0, s>>>(acc, n, g.W, e->sim_acc_bits, r_dem, r_pre, r_pf,
                                  (prefetch && k + 1 < n_launch) ? 1u : 0u,
                                  (prefetch && k + 1 < n_launch) ? 1u : 0u, invalidate ? 1u : 0u, stats + k);
    e->kernel_launches += 8;
  }
  return cudaGetLastError();
}

}  // namespace dum
