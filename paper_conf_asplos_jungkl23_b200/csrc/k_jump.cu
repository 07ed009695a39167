// Jump tables over the execution ID correlation table, so that a query's
// chain of up to N next-kernel predictions (D16)
// costs O(log N) dependent loads instead of N.
//
// For record r = (owner e; h1, h2, h3 -> succ n), the next lookup of the chain
// is the record (n; h2, h3, e) (D16: the history shifts in the predicted ID),
// so next(r) is a function of r alone.  J_0 = next, J_{k+1} = J_k o J_k;
// the chain of a query whose first record is r0 is succ(next^d(r0)) for
// d = 0, 1, ... until next^d(r0) is absent.  Rebuilt after every build on a
// side stream (it only reads the correlation table) while the block tables
// are applied; the next reader of the correlation table waits for it.
#include <algorithm>

#include "corr.cuh"
#include "device_util.cuh"
#include "kernels.cuh"

namespace dum {

constexpr int JUMP_NT = 256;

__global__ void __launch_bounds__(JUMP_NT) k_jump0(const CorrSlot *corr, uint32_t cap, const uint32_t *rec_slot,
                                                   uint32_t *j0, const DevState *st) {
  const uint32_t nrec = min(*(const volatile uint32_t *)&st->corr_used, cap);
  for (uint32_t r = blockIdx.x * JUMP_NT + threadIdx.x; r < nrec; r += gridDim.x * JUMP_NT) {
    const uint32_t s = rec_slot[r];
    const uint4 kk = __ldcg(reinterpret_cast<const uint4 *>(corr + s));
    const uint32_t succ = (uint32_t)(__ldcg(&corr[s].last) & 0xFFFFFFFFull);
    uint32_t dummy;
    j0[s] = corr_find(corr, cap, succ, kk.z, kk.w, kk.x, &dummy);
  }
}

// Levels 1 .. levels-1 in one launch: J_k(s) = J_0^(2^k)(s), each thread
// follows J_0 from its record and stores the positions 2, 4, 8, ... (2^(L-1)
// dependent loads of an L2-resident array instead of one launch per level).
__global__ void __launch_bounds__(JUMP_NT) k_jumpk(uint32_t cap, const uint32_t *rec_slot, uint32_t *jump,
                                                   uint32_t levels, const DevState *st) {
  const uint32_t nrec = min(*(const volatile uint32_t *)&st->corr_used, cap);
  for (uint32_t r = blockIdx.x * JUMP_NT + threadIdx.x; r < nrec; r += gridDim.x * JUMP_NT) {
    const uint32_t s = rec_slot[r];
    uint32_t x = __ldcg(jump + s);  // J_0(s)
    for (uint32_t k = 1, step = 1; k < levels; ++k) {
      for (const uint32_t target = 1u << k; step < target && x != NONE; ++step) x = __ldcg(jump + x);
      jump[(uint64_t)k * cap + s] = x;
    }
  }
}

cudaError_t launch_jump_tables(dum_engine *e, cudaStream_t s) {
  // records <= launches applied so far (one upsert each); the grid covers them
  const uint64_t nrec = std::min<uint64_t>(e->built_launches + e->n_staged, e->corr_cap);
  const uint32_t grid = (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>((nrec + JUMP_NT - 1) / JUMP_NT, 4 * 148));
  TimerScope t(e, DUM_T_JUMP, s);
  k_jump0<<<grid, JUMP_NT, 0, s>>>(e->d_corr, e->corr_cap, e->d_rec_slot, e->d_jump, e->d_state);
  if (e->jump_levels > 1) k_jumpk<<<grid, JUMP_NT, 0, s>>>(e->corr_cap, e->d_rec_slot, e->d_jump, e->jump_levels, e->d_state);
  e->kernel_launches += e->jump_levels > 1 ? 2 : 1;
  return cudaGetLastError();
}

}  // namespace dum
