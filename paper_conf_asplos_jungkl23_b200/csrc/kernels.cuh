// Kernel launchers (host side) implemented in k_*.cu.
#pragma once
#include "engine.cuh"

namespace dum {

// k_record.cu  (a1 + a2)
cudaError_t launch_record(dum_engine *e, const uint64_t *hash, const uint64_t *off, uint32_t n_launch,
                          const uint32_t *faults, uint64_t n_fault, uint32_t *out_exec, cudaStream_t s);
// k_build.cu   (a3 - a6)
cudaError_t launch_build(dum_engine *e, cudaStream_t s);
cudaError_t launch_build_head(dum_engine *e, uint32_t n, cudaStream_t s);
cudaError_t launch_walk_commit(dum_engine *e, cudaStream_t s);
cudaError_t launch_jump_tables(dum_engine *e, cudaStream_t s);
// k_predict.cu (a6 + a7)
cudaError_t launch_make_queries(dum_engine *e, const uint32_t *exec_seq, uint32_t n_seq, uint32_t first,
                                uint32_t degree, dum_query *out, cudaStream_t s);
struct SelectOut;
cudaError_t launch_predict(dum_engine *e, const dum_query *q, uint32_t nq, uint32_t *pairs, uint64_t cap,
                           uint64_t *range, uint32_t *kern_off, uint32_t *chain, uint64_t *needed,
                           const SelectOut *sel, uint64_t *sel_needed, cudaStream_t s);
// k_select.cu  (a8)
cudaError_t launch_select(dum_engine *e, const uint64_t *range, const uint32_t *pairs, uint32_t nq,
                          const dum_query *q, uint32_t *wb, uint32_t *inv, uint64_t cap, uint64_t *out_range,
                          uint64_t *needed, cudaStream_t s);
// k_migrate.cu (a9, residency)
cudaError_t launch_reset_residency(dum_engine *e, cudaStream_t s);
cudaError_t launch_load_residency(dum_engine *e, const uint32_t *lrm, uint32_t n, cudaStream_t s);
cudaError_t launch_mark_inactive(dum_engine *e, const uint32_t *blocks, uint32_t n, int flag, cudaStream_t s);
cudaError_t launch_migrate(dum_engine *e, int dir, const uint32_t *blocks, const uint32_t *dst, uint32_t n,
                           uint32_t method, cudaStream_t s, const uint64_t *rng = nullptr);
cudaError_t launch_checksums(dum_engine *e, int where, const uint32_t *ids, uint32_t n, uint64_t *out,
                             cudaStream_t s);

// k_sim.cu
cudaError_t launch_simulate(dum_engine *e, const uint64_t *hash, uint32_t n_launch, const uint64_t *acc_off,
                            const uint32_t *acc_blk, uint32_t n_kernels, uint32_t degree, uint32_t flags,
                            dum_sim_stats *stats, cudaStream_t s);

// walk geometry helpers shared by k_build.cu and k_predict.cu
struct WalkScratch {
  uint32_t *seen, *chain, *tmp;
  uint32_t cap;       // pow2 capacity of each hash set
  uint32_t tmp_cap;   // entries in tmp (slot log)
};

}  // namespace dum
