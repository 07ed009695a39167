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

// Per-CTA selection state, filled by select_reserve (one thread) before the
// barrier that precedes select_tail.
struct SelShared {
  unsigned long long bwb, binv;  // reserved output offsets (write-back, invalidate)
  uint32_t need, ok, head, tail, clean;
};

// One thread: need = max(0, nonres - free frames) (D18); reserve `need`
// entries in both output lists.  Issued as early as possible so that the
// contended bump-pointer atomics overlap other work of the CTA.
__device__ __forceinline__ void select_reserve(const SelectOut &so, uint32_t nonres, DevState *st, SelShared &ss) {
  const uint32_t nfree = *(volatile uint32_t *)&st->free_count;
  const uint32_t need = nonres > nfree ? nonres - nfree : 0;
  ss.need = need;
  ss.ok = 1;
  ss.bwb = ss.binv = 0;
  ss.head = *(volatile uint32_t *)&st->lrm_head;
  ss.tail = *(volatile uint32_t *)&st->lrm_tail;
  ss.clean = *(volatile uint32_t *)&st->log_dirty == 0;
  if (need) {
    ss.bwb = atomicAdd(&st->pool_wb, (unsigned long long)need);
    ss.binv = atomicAdd(&st->pool_inv, (unsigned long long)need);
    if (ss.bwb + need > so.cap || ss.binv + need > so.cap) {
      ss.ok = 0;
      set_err(st, ERR_ECAPACITY, (ss.bwb > ss.binv ? ss.bwb : ss.binv) + need);
    }
  }
}

// Barrier over the NT threads [0, NT) of the CTA: id 0 with NT = blockDim is
// __syncthreads; other ids are named barriers of a warp group.
template <int ID, int NT>
__device__ __forceinline__ void group_sync() {
  if (ID == 0) __syncthreads();
  else asm volatile("bar.sync %0, %1;" ::"n"(ID), "n"(NT) : "memory");
}

// Called by the NT threads tid = [0, NT) of a warp group synchronised by
// barrier BAR, after select_reserve and a barrier.  Victims = the first `need`
// entries of the LRM log (oldest migration first) that are still resident
// with that stamp and not in the window bitmap; split into write-back /
// invalidate by the inactive bit of the log entry, both in LRM order.
// The log is scanned in chunks of SEL_CHUNK entries aligned to 4: thread t
// owns IT consecutive entries (16 B loads) and keeps its eligible active /
// inactive entries as two bit masks; one group scan of the packed counts
// (inactive << 16 | active) ranks them; the taken entries are staged in
// shared memory (write-back from the front, invalidate from the back) and
// copied out with coalesced stores.  Warp totals are double-buffered: a chunk
// costs two barriers (three in the last one).
constexpr uint32_t SEL_CHUNK = 4096;  // stage capacity (words); a chunk is NT * IT <= SEL_CHUNK entries

// Window membership of a log entry (block b at log position p): the window
// set as a bitmap over the block-id space (built from the window's blocks).
struct InBlockBitmap {
  const uint32_t *bitmap;
  __device__ __forceinline__ uint32_t operator()(uint32_t b, uint32_t) const { return bitmap[b >> 5] >> (b & 31); }
};
// ... or as a bitmap over log positions [head, head + 32 * words) holding the
// positions of the window's resident blocks (k_window.cu fast path; the scan
// never passes head + 32 * words there).
struct InPosBitmap {
  const uint32_t *bits;
  uint32_t head, words;
  __device__ __forceinline__ uint32_t operator()(uint32_t, uint32_t p) const {
    const uint32_t r = p - head;
    return (p >= head && (r >> 5) < words) ? bits[r >> 5] >> (r & 31) : 0u;
  }
};

template <int NT, int BAR, class InWin, int CTR_SCAN = DUM_CTR_SEL_SCANNED, int CTR_VICT = DUM_CTR_SEL_VICTIMS,
          int ITP = 0>
__device__ void select_tail(const SelectOut &so, uint32_t qi, const SelShared &ss, const InWin &inwin,
                            DevState *st, uint32_t tid, uint32_t *stage /* SEL_CHUNK words of shared memory */) {
  constexpr int NW = NT / 32;
  constexpr uint32_t IT = ITP ? ITP : NT >= 512 ? 8 : NT >= 320 ? 12 : 16;  // entries per thread per chunk
  constexpr uint32_t CHUNK = NT * IT;
  static_assert(NW <= 32 && IT % 4 == 0 && CHUNK <= SEL_CHUNK, "one warp scans the warp totals; 16 B loads");
  __shared__ uint32_t s_wt[2][NW], s_tw, s_ti;
  const uint32_t lane = tid & 31, wid = tid >> 5;
  const uint32_t need = ss.need, head = ss.head, tail = ss.tail;
  const bool clean = ss.clean;
  const unsigned long long bwb = ss.bwb, binv = ss.binv;
  const bool ok = ss.ok;
  uint32_t run_wb = 0, run_inv = 0, scanned = 0;
  int buf = 0;
  for (uint32_t c = head & ~3u; c < tail && run_wb + run_inv < need; c += CHUNK, buf ^= 1) {
    scanned += min(c + CHUNK, tail) - max(c, head);
    const uint32_t i0 = c + IT * tid;
    uint32_t v[IT];
    const uint4 *p = reinterpret_cast<const uint4 *>(so.lrm_blk + i0);
#pragma unroll
    for (uint32_t k = 0; k < IT / 4; ++k) {
      uint4 x = make_uint4(0, 0, 0, 0);
      if (i0 + 4 * k < tail) x = p[k];  // log capacity is a multiple of 4: never past the allocation
      v[4 * k] = x.x;
      v[4 * k + 1] = x.y;
      v[4 * k + 2] = x.z;
      v[4 * k + 3] = x.w;
    }
    // entries of this thread inside [head, tail)
    uint32_t valid = 0;
    if (i0 < tail && i0 + IT > head) {
      const uint32_t lo = i0 < head ? head - i0 : 0, hi = min(IT, tail - i0);
      valid = (hi >= 32 ? 0xFFFFFFFFu : (1u << hi) - 1) & ~((1u << lo) - 1);
    }
    uint32_t em = 0, im = 0;  // eligible active / inactive entries (bit k = entry i0 + k)
#pragma unroll
    for (uint32_t k = 0; k < IT; ++k) {
      const uint32_t b = v[k] & 0x7FFFFFFFu;
      uint32_t e = ((valid >> k) & 1u) & ~inwin(b, i0 + k);
      if (!clean && (e & 1u))
        e = __ldg(&so.frame_of[b]) != NONE && __ldg(&so.stamp_of[b]) == so.lrm_stamp[i0 + k];
      const uint32_t ina = v[k] >> 31;
      em |= (e & ~ina & 1u) << k;
      im |= (e & ina & 1u) << k;
      v[k] = b;
    }
    // group exclusive scan of (popc(im) << 16 | popc(em))
    const uint32_t cnt = (__popc(im) << 16) | __popc(em);
    uint32_t x = cnt;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= (uint32_t)o) x += y;
    }
    if (lane == 31) s_wt[buf][wid] = x;
    group_sync<BAR, NT>();
    uint32_t wpre = 0, tot = 0;
    {
      const uint32_t t = lane < (uint32_t)NW ? s_wt[buf][lane] : 0;
      uint32_t z = t;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, z, o);
        if (lane >= (uint32_t)o) z += y;
      }
      wpre = __shfl_sync(0xffffffffu, z - t, wid);
      tot = __shfl_sync(0xffffffffu, z, NW - 1);
    }
    const uint32_t pre = wpre + x - cnt;
    const uint32_t pw = pre & 0xFFFFu, pi = pre >> 16;
    const uint32_t tw = tot & 0xFFFFu, ti = tot >> 16;
    const uint32_t left = need - run_wb - run_inv;
    // stage this thread's eligible entries of combined rank < left
    {
      uint32_t rw = pw, ri = pi;
#pragma unroll
      for (uint32_t k = 0; k < IT; ++k) {
        const uint32_t ew = (em >> k) & 1u, ei = (im >> k) & 1u;
        if ((ew | ei) && rw + ri < left) stage[ei ? CHUNK - 1 - ri : rw] = v[k];
        rw += ew;
        ri += ei;
      }
    }
    uint32_t take_w = tw, take_i = ti;
    if (tw + ti > left) {
      // the last chunk: the thread holding combined rank `left` reports how
      // many of the taken entries are of each kind
      const uint32_t p0 = pw + pi, nall = __popc(em | im);
      if (p0 <= left && left < p0 + nall) {
        uint32_t aw = pw, ai = pi;
#pragma unroll
        for (uint32_t k = 0; k < IT; ++k) {
          if (aw + ai < left) {
            aw += (em >> k) & 1u;
            ai += (im >> k) & 1u;
          }
        }
        s_tw = aw;
        s_ti = ai;
      }
      group_sync<BAR, NT>();
      take_w = s_tw;
      take_i = s_ti;
    } else {
      group_sync<BAR, NT>();
    }
    if (ok) {
      for (uint32_t j = tid; j < take_w; j += NT) so.wb[bwb + run_wb + j] = stage[j];
      for (uint32_t j = tid; j < take_i; j += NT) so.inv[binv + run_inv + j] = stage[CHUNK - 1 - j];
    }
    run_wb += take_w;
    run_inv += take_i;
  }
  if (tid == 0) {
    uint64_t *o = so.out_range + 4ull * qi;
    o[0] = bwb;
    o[1] = bwb + (ok ? run_wb : 0);
    o[2] = binv;
    o[3] = binv + (ok ? run_inv : 0);
    ctr_add(st, CTR_SCAN, scanned);
    ctr_add(st, CTR_VICT, run_wb + run_inv);
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
