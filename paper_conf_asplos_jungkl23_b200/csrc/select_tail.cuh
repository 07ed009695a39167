// a8 selection tail shared by k_select (standalone call) and the fused
// predict+select kernel: given the window set (a shared-memory bitmap that
// also holds the anchor) and the number of window blocks without a frame,
// pick the victims (readings D18-D20).
#pragma once
#include "device_util.cuh"
#include "kernels.cuh"

namespace dum {

struct SelectOut {
  const uint32_t *frame_of, *stamp_of, *inactive, *lrm_blk, *lrm_stamp;
  uint32_t *wb, *inv;
  uint64_t cap;
  uint64_t *out_range;  // 4 per query
};

// All threads of the CTA must call it.  need = max(0, nonres - free); victims
// = the first `need` entries of the LRM log (oldest migration first) that are
// still resident with that stamp and not in the window bitmap; split into
// write-back / invalidate by the inactive bitmap, both in LRM order.
// Each thread examines ITEMS consecutive log entries per chunk, so one block
// scan covers NT * ITEMS entries.
template <int NT>
__device__ void select_tail(const SelectOut &so, uint32_t qi, uint32_t nonres, const uint32_t *bitmap, uint32_t W,
                            DevState *st, uint32_t *ws) {
  constexpr int ITEMS = 4;
  __shared__ uint32_t s_ok, s_cwb, s_cinv;
  __shared__ unsigned long long s_bwb, s_binv;
  const uint32_t tid = threadIdx.x;
  const uint32_t nfree = *(volatile uint32_t *)&st->free_count;
  const uint32_t need = nonres > nfree ? nonres - nfree : 0;
  const bool clean = *(volatile uint32_t *)&st->log_dirty == 0;
  if (tid == 0) {
    s_ok = 1;
    s_bwb = s_binv = 0;
    if (need) {
      s_bwb = atomicAdd(&st->pool_wb, (unsigned long long)need);
      s_binv = atomicAdd(&st->pool_inv, (unsigned long long)need);
      if (s_bwb + need > so.cap || s_binv + need > so.cap) {
        s_ok = 0;
        set_err(st, ERR_ECAPACITY, (s_bwb > s_binv ? s_bwb : s_binv) + need);
      }
    }
  }
  __syncthreads();
  const unsigned long long bwb = s_bwb, binv = s_binv;
  const bool ok = s_ok;
  uint32_t run_wb = 0, run_inv = 0, scanned = 0;
  const uint32_t head = *(volatile uint32_t *)&st->lrm_head, tail = *(volatile uint32_t *)&st->lrm_tail;
  for (uint32_t c = head; c < tail && run_wb + run_inv < need; c += NT * ITEMS) {
    scanned += min((uint32_t)(NT * ITEMS), tail - c);
    uint32_t blk[ITEMS];
    uint32_t flags = 0;  // bit k: eligible, bit 8+k: inactive
    uint32_t cw = 0, ci = 0;
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) {
      const uint32_t i = c + tid * ITEMS + k;
      blk[k] = NONE;
      if (i < tail) {
        const uint32_t b = so.lrm_blk[i];
        blk[k] = b;
        bool elig = !(bitmap[b >> 5] & (1u << (b & 31)));
        if (elig && !clean) elig = __ldg(&so.frame_of[b]) != NONE && __ldg(&so.stamp_of[b]) == so.lrm_stamp[i];
        if (elig) {
          const bool ina = (__ldg(&so.inactive[b >> 5]) >> (b & 31)) & 1u;
          flags |= (1u << k) | (ina ? (1u << (8 + k)) : 0u);
          ci += ina;
          cw += !ina;
        }
      }
    }
    uint32_t tot;
    const uint32_t pre = block_excl_scan((ci << 16) | cw, ws, &tot);
    const uint32_t left = need - run_wb - run_inv;
    uint32_t pw = pre & 0xFFFFu, pi = pre >> 16;
    uint32_t tw = 0, ti = 0;
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) {
      if (flags & (1u << k)) {
        const bool ina = flags & (1u << (8 + k));
        if (pw + pi < left) {
          if (ok) {
            if (ina) so.inv[binv + run_inv + pi] = blk[k];
            else so.wb[bwb + run_wb + pw] = blk[k];
          }
          if (ina) ++ti;
          else ++tw;
        }
        if (ina) ++pi;
        else ++pw;
      }
    }
    if (tid == 0) {
      s_cwb = 0;
      s_cinv = 0;
    }
    __syncthreads();
    if (tw) atomicAdd(&s_cwb, tw);
    if (ti) atomicAdd(&s_cinv, ti);
    __syncthreads();
    run_wb += s_cwb;
    run_inv += s_cinv;
    __syncthreads();
  }
  if (tid == 0) {
    uint64_t *o = so.out_range + 4ull * qi;
    o[0] = bwb;
    o[1] = bwb + (ok ? run_wb : 0);
    o[2] = binv;
    o[3] = binv + (ok ? run_inv : 0);
    ctr_add(st, DUM_CTR_SEL_SCANNED, scanned);
    ctr_add(st, DUM_CTR_SEL_VICTIMS, run_wb + run_inv);
  }
}

inline SelectOut make_select_out(dum_engine *e, uint32_t *wb, uint32_t *inv, uint64_t cap, uint64_t *out_range) {
  SelectOut so;
  so.frame_of = e->d_frame_of;
  so.stamp_of = e->d_stamp_of;
  so.inactive = e->d_inactive_bits;
  so.lrm_blk = e->d_lrm_blk;
  so.lrm_stamp = e->d_lrm_stamp;
  so.wb = wb;
  so.inv = inv;
  so.cap = cap;
  so.out_range = out_range;
  return so;
}

}  // namespace dum
