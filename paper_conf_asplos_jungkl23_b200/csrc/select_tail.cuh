// a8 selection tail shared by k_select (standalone call) and the fused
// predict+select kernel: given the window set (a shared-memory bitmap that
// also holds the anchor) and the number of window blocks without a frame,
// pick the victims (readings D18-D20).
#pragma once
#include "device_util.cuh"
#include "kernels.cuh"

namespace dum {

struct SelectOut {
  const uint32_t *frame_of, *stamp_of, *inactive, *res_bits, *lrm_blk, *lrm_stamp;
  uint32_t *wb, *inv;
  uint64_t cap;
  uint64_t *out_range;  // 4 per query
};

// All threads of the CTA must call it.  need = max(0, nonres - free); victims
// = the first `need` entries of the LRM log (oldest migration first) that are
// still resident with that stamp and not in the window bitmap; split into
// write-back / invalidate by the inactive bitmap, both in LRM order.
// Chunks of NT * 4 log entries; warp w owns 128 consecutive entries of a
// chunk (4 coalesced steps of 32), counts its eligible active / inactive
// entries with ballots, and the 32 warp totals are scanned by one warp -- one
// barrier pair per chunk.
template <int NT>
__device__ void select_tail(const SelectOut &so, uint32_t qi, uint32_t nonres, const uint32_t *bitmap, uint32_t W,
                            DevState *st, uint32_t *ws) {
  constexpr int NW = NT / 32;
  constexpr int ITEMS = 4;
  constexpr uint32_t CHUNK = NT * ITEMS;
  __shared__ uint32_t s_ok, s_wcnt[NW], s_icnt[NW], s_tw, s_ti, s_aw, s_ai, s_split, s_rem;
  __shared__ unsigned long long s_bwb, s_binv;
  const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
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
  const uint32_t lt = (1u << lane) - 1;
  for (uint32_t c = head; c < tail && run_wb + run_inv < need; c += CHUNK) {
    scanned += min(CHUNK, tail - c);
    uint32_t blk[ITEMS], me[ITEMS], mi[ITEMS];
    uint32_t cw = 0, ci = 0;
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) {
      const uint32_t i = c + wid * (32 * ITEMS) + 32 * k + lane;
      blk[k] = i < tail ? so.lrm_blk[i] : NONE;
    }
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) {
      const uint32_t i = c + wid * (32 * ITEMS) + 32 * k + lane;
      const uint32_t b = blk[k] & 0x7FFFFFFFu;  // log entry: block | inactive << 31
      bool elig = false, ina = false;
      if (i < tail) {
        elig = !(bitmap[b >> 5] & (1u << (b & 31)));
        if (elig && !clean) elig = __ldg(&so.frame_of[b]) != NONE && __ldg(&so.stamp_of[b]) == so.lrm_stamp[i];
        ina = blk[k] >> 31;
      }
      blk[k] = b;
      me[k] = __ballot_sync(0xffffffffu, elig && !ina);
      mi[k] = __ballot_sync(0xffffffffu, elig && ina);
      cw += __popc(me[k]);
      ci += __popc(mi[k]);
    }
    if (lane == 0) {
      s_wcnt[wid] = cw;
      s_icnt[wid] = ci;
    }
    __syncthreads();
    // exclusive prefix of the warp totals (log order = warp order): one
    // packed warp scan over the NW totals (counts <= 128 fit 16 bits)
    uint32_t pw, pi, tw, ti;
    {
      const uint32_t v = lane < NW ? (s_icnt[lane] << 16) | s_wcnt[lane] : 0;
      uint32_t x = v;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= (uint32_t)o) x += y;
      }
      const uint32_t ex = __shfl_sync(0xffffffffu, x - v, wid);
      const uint32_t tot = __shfl_sync(0xffffffffu, x, NW - 1);
      pw = ex & 0xFFFFu;
      pi = ex >> 16;
      tw = tot & 0xFFFFu;
      ti = tot >> 16;
    }
    const uint32_t left = need - run_wb - run_inv;
#pragma unroll
    for (int k = 0; k < ITEMS; ++k) {
      const uint32_t i = c + wid * (32 * ITEMS) + 32 * k + lane;
      const bool ew = (me[k] >> lane) & 1u, ei = (mi[k] >> lane) & 1u;
      const uint32_t rw = pw + __popc(me[k] & lt), ri = pi + __popc(mi[k] & lt);
      if ((ew || ei) && rw + ri < left && ok) {
        if (ei) so.inv[binv + run_inv + ri] = blk[k];
        else so.wb[bwb + run_wb + rw] = blk[k];
      }
      (void)i;
      pw += __popc(me[k]);
      pi += __popc(mi[k]);
    }
    // the taken entries are the first `left` eligible ones of the chunk; how
    // many of them are write-back vs invalidate
    uint32_t take_w = tw, take_i = ti;
    if (tw + ti > left) {
      // find the split inside the chunk: the warp holding eligible entry `left`
      if (tid == 0) {
        uint32_t aw = 0, ai = 0;
        s_split = NONE;
        for (int w = 0; w < NW; ++w) {
          if (aw + ai + s_wcnt[w] + s_icnt[w] > left) {
            s_split = w;
            s_rem = left - aw - ai;  // eligible entries of warp w that are taken
            break;
          }
          aw += s_wcnt[w];
          ai += s_icnt[w];
        }
        s_aw = aw;  // totals of the warps before the split warp
        s_ai = ai;
      }
      __syncthreads();
      const uint32_t w_split = s_split, rem = s_rem;
      const uint32_t aw = s_aw, ai = s_ai;
      if (wid == w_split) {
        // walk this warp's 4 steps in order; lanes count taken entries
        uint32_t r = rem, cw2 = 0, ci2 = 0;
#pragma unroll
        for (int k = 0; k < ITEMS; ++k) {
          const uint32_t all = me[k] | mi[k];
          const uint32_t nall = __popc(all);
          if (r >= nall) {
            cw2 += __popc(me[k]);
            ci2 += __popc(mi[k]);
            r -= nall;
          } else if (r > 0) {
            // first r set bits of `all`
            uint32_t m = all, sel = 0;
            for (uint32_t q = 0; q < r; ++q) {
              const uint32_t bit = m & (~m + 1u);
              sel |= bit;
              m &= m - 1;
            }
            cw2 += __popc(me[k] & sel);
            ci2 += __popc(mi[k] & sel);
            r = 0;
          }
        }
        if (lane == 0) {
          s_tw = aw + cw2;
          s_ti = ai + ci2;
        }
      }
      __syncthreads();
      take_w = s_tw;
      take_i = s_ti;
    }
    run_wb += take_w;
    run_inv += take_i;
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
  so.res_bits = e->d_res_bits;
  so.lrm_blk = e->d_lrm_blk;
  so.lrm_stamp = e->d_lrm_stamp;
  so.wb = wb;
  so.inv = inv;
  so.cap = cap;
  so.out_range = out_range;
  return so;
}

}  // namespace dum
