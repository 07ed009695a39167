// a7 + a8 fast path: prefetch windows whose kernels' walks share no block.
//
// A window concatenates the cached walks of the
// current kernel and the next N predicted kernels, keeping the first
// occurrence of every block (D17).  Each cached walk is duplicate-free, and a
// kernel met twice in the chain adds nothing (k_chain), so a window can hold a
// duplicate only if two DISTINCT kernels of its chain have walks that share a
// block.  After every build the walk index records, per exec ID e, the exec
// IDs whose walk shares a block with walk(e) (the "conflicts" of e); k_chain
// sends a query to the exact kernel (k_predict.cu: window bitmap, duplicate
// and fallback paths) iff its chain holds a conflicting pair, an exec ID with
// too many conflicts to record, or an anchor (D14: WALK(e, anchor) is not a
// cached walk).  Every other window is the plain concatenation of its walks --
// no window set is needed to emit it.
//
// The pre-eviction selection of such a window (
// D18-D20) needs two facts about the window set:
//   #window blocks without a frame  = sum over its distinct walks of the
//                                     walk's non-resident count, and
//   "is the LRM entry at log position p in the window" = p is the log position
//                                     of a resident block of one of its walks.
// k_walk_res computes, per walk, the non-resident count and the log positions
// of its resident blocks (after every residency change, at predict time);
// the selection kernels mark those positions in a shared-memory bitmap over
// [head, head + POS_BITS) of the LRM log and runs the same ordered selection
// as the exact path (select_tail.cuh) on it.  k_chain only routes a query
// here when the selection provably ends inside that range.
//
//  k_walk_count  (build end)   holders of each block: bcnt[b], bhold[b][..]
//  k_walk_conf   (build end)   conflicts of each walk: conf[e][..], conf_n[e]
//  k_walk_res    (predict)     per walk: non-resident count, resident positions
//  k_copy_fast   (predict)     flat copy of every fast window (chunk map from k_chain)
//  k_select_fast (predict)     clean log: a CTA per big window, a warp per small one;
//                              marking + word-level selection
//  k_select_stale (predict)    stale log entries: a CTA per window, per-entry selection
#include <algorithm>

#include "device_util.cuh"
#include "kernels.cuh"
#include "predict.cuh"
#include "select_tail.cuh"

namespace dum {

constexpr int IX_NT = 512;
constexpr int IX_U = 4;              // walk entries per thread with their loads in flight together
constexpr uint32_t CONF_HCAP = 256;  // shared hash of one walk's conflicts (> CONF_MAX)

__global__ void __launch_bounds__(IX_NT) k_walk_count(const uint32_t *__restrict__ walk,
                                                      const uint32_t *__restrict__ walk_len, uint32_t walk_cap,
                                                      const DevState *st, uint32_t *bcnt, uint32_t *bhold) {
  const uint32_t E = __ldcg(&st->E);
  for (uint32_t e = blockIdx.x; e < E; e += gridDim.x) {
    const uint32_t n = walk_len[e];
    const uint32_t *w = walk + (uint64_t)e * walk_cap;
    for (uint32_t j0 = threadIdx.x; j0 < n; j0 += IX_NT * IX_U) {
      uint32_t b[IX_U], k[IX_U];
#pragma unroll
      for (int u = 0; u < IX_U; ++u) b[u] = j0 + u * IX_NT < n ? w[j0 + u * IX_NT] : NONE;
#pragma unroll
      for (int u = 0; u < IX_U; ++u) k[u] = b[u] != NONE ? atomicAdd(&bcnt[b[u]], 1u) : NONE;
#pragma unroll
      for (int u = 0; u < IX_U; ++u)
        if (k[u] < HOLD_MAX) bhold[(uint64_t)b[u] * HOLD_MAX + k[u]] = e;
    }
  }
}

__global__ void __launch_bounds__(IX_NT) k_walk_conf(const uint32_t *__restrict__ walk,
                                                     const uint32_t *__restrict__ walk_len, uint32_t walk_cap,
                                                     const DevState *st, const uint32_t *__restrict__ bcnt,
                                                     const uint32_t *__restrict__ bhold, uint32_t *conf,
                                                     uint32_t *conf_n) {
  __shared__ uint32_t hs[CONF_HCAP];
  __shared__ uint32_t s_n, s_ovf;
  const uint32_t E = __ldcg(&st->E);
  const uint32_t tid = threadIdx.x;
  for (uint32_t e = blockIdx.x; e < E; e += gridDim.x) {
    for (uint32_t k = tid; k < CONF_HCAP; k += IX_NT) hs[k] = NONE;
    if (tid == 0) {
      s_n = 0;
      s_ovf = 0;
    }
    __syncthreads();
    const uint32_t n = walk_len[e];
    const uint32_t *w = walk + (uint64_t)e * walk_cap;
    for (uint32_t j0 = tid; j0 < n; j0 += IX_NT * IX_U) {
      uint32_t b[IX_U], c[IX_U];
#pragma unroll
      for (int u = 0; u < IX_U; ++u) b[u] = j0 + u * IX_NT < n ? w[j0 + u * IX_NT] : NONE;
#pragma unroll
      for (int u = 0; u < IX_U; ++u) c[u] = b[u] != NONE ? bcnt[b[u]] : 0u;
#pragma unroll
      for (int u = 0; u < IX_U; ++u) {
        if (c[u] < 2) continue;
        if (c[u] > HOLD_MAX) {
          s_ovf = 1;  // holders not all recorded: e's windows take the exact path
          continue;
        }
        for (uint32_t k = 0; k < c[u]; ++k) {
          const uint32_t h = bhold[(uint64_t)b[u] * HOLD_MAX + k];
          if (h == e) continue;
          uint32_t sl = (h * 0x9E3779B1u) >> 24;  // 8 bits: CONF_HCAP = 256
          bool placed = false;
          for (uint32_t p = 0; p < CONF_HCAP; ++p, sl = (sl + 1) & (CONF_HCAP - 1)) {
            // most inserts repeat a recorded conflict: a plain read first (no
            // serialised shared atomics on the hot slots)
            const uint32_t cur = *(volatile uint32_t *)&hs[sl];
            if (cur == h) {
              placed = true;
              break;
            }
            if (cur != NONE) continue;
            const uint32_t old = atomicCAS(&hs[sl], NONE, h);
            if (old == h) {
              placed = true;
              break;
            }
            if (old == NONE) {
              const uint32_t i = atomicAdd(&s_n, 1u);
              if (i < CONF_MAX) conf[(uint64_t)e * CONF_MAX + i] = h;
              placed = true;
              break;
            }
          }
          if (!placed) s_ovf = 1;
        }
      }
    }
    __syncthreads();
    if (tid == 0) conf_n[e] = (s_ovf || s_n > CONF_MAX) ? NONE : s_n;
    __syncthreads();
  }
}

// Per walk: blocks without a frame (nr), and the LRM-log positions of the
// blocks with one (respos, any order).  Reads the residency of this call.
__global__ void __launch_bounds__(IX_NT) k_walk_res(const uint32_t *__restrict__ walk,
                                                    const uint32_t *__restrict__ walk_len, uint32_t walk_cap,
                                                    const DevState *st, const uint32_t *__restrict__ res_bits,
                                                    const uint32_t *__restrict__ logpos, uint32_t *wnr,
                                                    uint32_t *wnres, uint32_t *respos) {
  __shared__ uint32_t s_nres, s_nr;
  const uint32_t E = __ldcg(&st->E);
  const uint32_t tid = threadIdx.x, lane = tid & 31;
  for (uint32_t e = blockIdx.x; e < E; e += gridDim.x) {
    if (tid == 0) {
      s_nres = 0;
      s_nr = 0;
    }
    __syncthreads();
    const uint32_t n = walk_len[e];
    const uint32_t *w = walk + (uint64_t)e * walk_cap;
    uint32_t *rp = respos + (uint64_t)e * walk_cap;
    uint32_t nr = 0;
    for (uint32_t j0 = 0; j0 < n; j0 += IX_NT * IX_U) {
      uint32_t b[IX_U], rw[IX_U];
#pragma unroll
      for (int u = 0; u < IX_U; ++u) {
        const uint32_t j = j0 + u * IX_NT + tid;
        b[u] = j < n ? w[j] : NONE;
      }
#pragma unroll
      for (int u = 0; u < IX_U; ++u) rw[u] = b[u] != NONE ? __ldg(res_bits + (b[u] >> 5)) : 0u;
#pragma unroll
      for (int u = 0; u < IX_U; ++u) {
        const bool res = b[u] != NONE && ((rw[u] >> (b[u] & 31)) & 1u);
        nr += b[u] != NONE && !res;
        const uint32_t pos = res ? __ldg(logpos + b[u]) : 0u;
        const uint32_t m = __ballot_sync(0xffffffffu, res);
        uint32_t base = 0;
        if (lane == 0 && m) base = atomicAdd(&s_nres, (uint32_t)__popc(m));
        base = __shfl_sync(0xffffffffu, base, 0);
        if (res) rp[base + __popc(m & ((1u << lane) - 1))] = pos;
      }
    }
    nr = __reduce_add_sync(0xffffffffu, nr);
    if (lane == 0 && nr) atomicAdd(&s_nr, nr);
    __syncthreads();
    if (tid == 0) {
      wnr[e] = s_nr;
      wnres[e] = s_nres;
    }
    __syncthreads();
  }
}

// Flat copy of every fast query's window: warp-granular work items of <= 128
// window blocks of one list of one query, each a 16 B descriptor written by
// k_chain (source walk + first entry, destination pair slot, length: one
// dependent load before the data), four in flight per warp, lane-consecutive
// 4 B loads of the cached walk and 8 B streaming stores of the (block, exec)
// pairs.  Persistent grid over the device count.
__global__ void __launch_bounds__(COPY_NT) k_copy_fast(PredArgs a) {
  constexpr uint32_t UN = 4;  // chunks per warp step, their loads in flight together
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t G = __ldcg(&a.st->pool_chunks);
  const uint64_t nw = (uint64_t)gridDim.x * (COPY_NT / 32);
  uint2 *out = reinterpret_cast<uint2 *>(a.pairs);
  unsigned long long emitted = 0;
  for (uint64_t c0 = (uint64_t)blockIdx.x * (COPY_NT / 32) + (threadIdx.x >> 5); c0 < G; c0 += nw * UN) {
    uint4 m[UN];
#pragma unroll
    for (uint32_t u = 0; u < UN; ++u)
      m[u] = c0 + u * nw < G ? __ldcg(a.chunk_map + c0 + u * nw) : make_uint4(0, 0, 0, 0);
    uint32_t b[UN][4];
#pragma unroll
    for (uint32_t u = 0; u < UN; ++u) {
      const uint32_t n = m[u].w >> 16;
      const uint32_t *lst = a.walk + (uint64_t)m[u].x * a.g.walk_cap + m[u].y;
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) b[u][k] = 32 * k + lane < n ? __ldg(lst + 32 * k + lane) : NONE;
    }
#pragma unroll
    for (uint32_t u = 0; u < UN; ++u) {
      const uint32_t n = m[u].w >> 16;
      uint2 *o = out + ((unsigned long long)(m[u].w & 0xFFFFu) << 32 | m[u].z);
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k)
        if (32 * k + lane < n) __stcs(o + 32 * k + lane, make_uint2(b[u][k], m[u].x));
      emitted += n;
    }
  }
  emitted = __reduce_add_sync(0xffffffffu, (unsigned)emitted) / 32;
  if (lane == 0 && emitted) {
    ctr_add(a.st, DUM_CTR_EMITTED, emitted);
    ctr_add(a.st, DUM_CTR_GATHERED, emitted);
    ctr_add(a.st, DUM_CTR_FAST_EMITTED, emitted);
  }
}

// a8 of the fast queries (k_chain's order: by decreasing `need`).  need =
// max(0, window blocks without a frame - free frames) and the victim ranges
// come from k_chain (D18).  The victims are the first `need` entries of the
// LRM log, oldest first, that are still resident with their stamp and not in
// the window, split by the inactive bit of the entry into
// invalidate / write-back (L285; D19, D20).  Every variant marks the log
// positions of the window's resident blocks (flat over the lists' respos
// entries, prefix qroff from k_chain) in a bitmap over [head, head + 32
// POS_WORDS) and selects in the log prefix [head, head + span), span = need +
// resident window blocks + stale entries (k_chain routes a query here only
// when the selection provably ends inside).  The window's pairs are written
// by k_copy_fast, concurrently.
//
// Clean log (every entry of [head, tail) valid, the normal case):
// k_select_fast.  A 32-position word's eligible entries are ~marked & valid,
// split by the log's inactive-entry bitmap (k_log_bits) into write-back /
// invalidate; a scan of the packed popcounts gives every word its rank base;
// then 4-word chunks (a lane per 4 consecutive entries, 16 B loads of the
// log) write the entries of combined rank < need at their ranks.  Work items
// in k_chain's class order: a big window (classes 0-2, need-key >= 6144) is
// one CTA item (all warps mark, one block scan, the warps split the chunks);
// the small ones go WSEL_NT / 32 to an item, a warp each (32-word groups, a
// warp scan per group, no CTA barrier).  A warp per window alone leaves the
// few biggest windows as a serial tail; a CTA per window leaves the SMs
// waiting on barriers for the many small ones.
//
// Stale entries (a log not compacted since an eviction): k_select_stale, a CTA
// per query, per-entry eligibility (frame + stamp check):
//   1. marks as above;  2. pass 1: eligible active / inactive entries per
//   1024-entry segment, a warp per segment;  3. one warp scans the segment
//   counts;  4. pass 2: each warp re-reads its segments and writes the
//   entries of combined rank < need.
constexpr uint32_t FSEG = 1024;                 // log entries per segment (32 per lane)
constexpr uint32_t FSEG_MAX = POS_WORDS * 32 / FSEG;
static_assert(FSEG_MAX <= 32, "one warp scans the segment counts");
constexpr uint32_t SEL_NW = WSEL_NT / 32;  // warps per selection CTA
constexpr uint32_t SW_KB = 2;              // warp path: 4-word chunks with their log loads in flight together
constexpr uint32_t BIG_CLS = 3;            // classes [0, BIG_CLS) take a CTA per window

__host__ __device__ constexpr uint32_t sw_words(uint32_t N) {  // shared words of one warp's window (16 B multiple)
  return (POS_WORDS + (N + 2) + (N + 1) + 3) & ~3u;
}
__host__ __device__ constexpr uint32_t sel_smem_words(uint32_t N) {  // k_select_fast dynamic shared memory
  return SEL_NW * sw_words(N) > 4 * POS_WORDS + sw_words(N) - POS_WORDS
             ? SEL_NW * sw_words(N)
             : 4 * POS_WORDS + sw_words(N) - POS_WORDS;
}

// the fast query of rank bq in k_chain's class lists
__device__ __forceinline__ uint32_t fast_query(const PredArgs &a, const uint32_t *ccnt, uint32_t bq) {
  uint32_t cq = NQCLS, rq = bq;
#pragma unroll
  for (int c = 0; c < NQCLS; ++c)
    if (cq == NQCLS) {
      if (rq < ccnt[c]) cq = c;
      else rq -= ccnt[c];
    }
  return __ldg(a.qperm + (uint64_t)cq * a.nq + rq);
}

struct SelLog {  // the log, fixed during the kernel
  uint32_t head, tail, stale;
  bool al;       // head 16 B aligned: vector loads of the log
};

struct SelQuery {
  uint32_t qi, nk, need;
  unsigned long long bwb, binv;
  bool ok;
};

__device__ __forceinline__ SelQuery load_query(const PredArgs &a, uint32_t qi) {
  SelQuery q;
  q.qi = qi;
  q.nk = __ldg(a.qnk + qi);
  q.need = __ldg(a.qneed + qi);
  q.bwb = __ldg(a.qvb + 2 * qi);
  q.binv = __ldg(a.qvb + 2 * qi + 1);
  q.ok = q.bwb + q.need <= a.so.cap && q.binv + q.need <= a.so.cap;
  return q;
}

__device__ __forceinline__ void write_range(const PredArgs &a, const SelQuery &q, uint32_t tw, uint32_t ti) {
  uint64_t *o = a.so.out_range + 4ull * q.qi;
  o[0] = q.bwb;
  o[1] = q.bwb + (q.ok ? tw : 0);
  o[2] = q.binv;
  o[3] = q.binv + (q.ok ? ti : 0);
}

// Marks: the log positions (relative to head) of the window's resident blocks
// below nbits, by threads t = t0, t0 + nt, ... (MU loads in flight each).
template <uint32_t MU>
__device__ __forceinline__ void mark_window(const PredArgs &a, const uint32_t *roff, const uint32_t *kern, uint32_t R,
                                            uint32_t head, uint32_t nbits, uint32_t *posmap, uint32_t t0,
                                            uint32_t nt) {
  uint32_t lo = 0;
  for (uint32_t x0 = t0; x0 < R; x0 += nt * MU) {
    uint32_t r[MU];
#pragma unroll
    for (uint32_t u = 0; u < MU; ++u) {
      const uint32_t x = x0 + u * nt;
      r[u] = NONE;
      if (x < R) {
        while (roff[lo + 1] <= x) ++lo;
        r[u] = __ldg(a.respos + (uint64_t)kern[lo] * a.g.walk_cap + (x - roff[lo])) - head;
      }
    }
#pragma unroll
    for (uint32_t u = 0; u < MU; ++u)
      if (r[u] < nbits) atomicOr(&posmap[r[u] >> 5], 1u << (r[u] & 31));
  }
}

// The eligible entries of UC 4-word chunks of one warp (a lane per 4
// consecutive entries): chunk u covers words wd[u] .. +3 relative to w0 (lane
// >> 3 picks the word), with em / im / pre the word's masks and rank base
// (packed inactive << 16 | active).  Entries of combined rank < need go to
// their ranks; returns the counts written (tw, ti).
template <uint32_t UC>
__device__ __forceinline__ void emit_chunks(const PredArgs &a, const SelQuery &q, const SelLog &lg, uint32_t lane,
                                            const uint32_t *wpos, const uint32_t *em, const uint32_t *im,
                                            const uint32_t *pre, uint32_t &tw, uint32_t &ti) {
  const SelectOut &so = a.so;
  uint32_t a4[UC], i4[UC], ra[UC], rr[UC], vv[UC][4];
  const uint32_t sh = (lane & 7) * 4;
#pragma unroll
  for (uint32_t u = 0; u < UC; ++u) {
    a4[u] = (em[u] >> sh) & 0xFu;
    i4[u] = (im[u] >> sh) & 0xFu;
    // ranks: the word's base + the eligible entries of the lower lanes of the same word
    const uint32_t cc = __popc(a4[u]) | (__popc(i4[u]) << 16);
    uint32_t y = cc;
#pragma unroll
    for (int o = 1; o < 8; o <<= 1) {
      const uint32_t t = __shfl_up_sync(0xffffffffu, y, o);
      if ((lane & 7) >= (uint32_t)o) y += t;
    }
    ra[u] = (pre[u] & 0xFFFFu) + ((y - cc) & 0xFFFFu);
    rr[u] = (pre[u] >> 16) + ((y - cc) >> 16);
    if (ra[u] + rr[u] >= q.need) a4[u] = i4[u] = 0;
    if (a4[u] | i4[u]) {
      const uint32_t p = lg.head + 32 * wpos[u] + sh;
      if (lg.al) {
        const uint4 v = __ldcg(reinterpret_cast<const uint4 *>(so.lrm_blk + p));
        vv[u][0] = v.x; vv[u][1] = v.y; vv[u][2] = v.z; vv[u][3] = v.w;
      } else {
#pragma unroll
        for (uint32_t k = 0; k < 4; ++k) vv[u][k] = ((a4[u] | i4[u]) >> k) & 1u ? __ldcg(so.lrm_blk + p + k) : 0u;
      }
    }
  }
#pragma unroll
  for (uint32_t u = 0; u < UC; ++u) {
    if (!(a4[u] | i4[u])) continue;
#pragma unroll
    for (uint32_t k = 0; k < 4; ++k) {
      const bool ea = (a4[u] >> k) & 1u, ei = (i4[u] >> k) & 1u;
      if ((ea || ei) && ra[u] + rr[u] < q.need) {
        if (q.ok) {
          if (ei) so.inv[q.binv + rr[u]] = vv[u][k] & 0x7FFFFFFFu;
          else so.wb[q.bwb + ra[u]] = vv[u][k];
        }
        tw += ea;
        ti += ei;
      }
      ra[u] += ea;
      rr[u] += ei;
    }
  }
}

// A small window, one warp: marks in the warp's bitmap, then 32-word groups
// (lane l: word w0 + l) with a warp scan each, until the cut.
__device__ __forceinline__ void warp_window(const PredArgs &a, const SelLog &lg, uint32_t qi, uint32_t *wsm,
                                            unsigned long long &scanned, unsigned long long &victims) {
  const uint32_t lane = threadIdx.x & 31;
  const Geo &g = a.g;
  uint32_t *posmap = wsm, *roff = wsm + POS_WORDS, *kern = roff + g.N + 2;
  const SelQuery q = load_query(a, qi);
  for (uint32_t d = lane; d <= q.nk; d += 32) {
    roff[d] = __ldg(a.qroff + (uint64_t)qi * (g.N + 2) + d);
    if (d < q.nk) kern[d] = __ldg(a.qkern + (uint64_t)qi * (g.N + 1) + d);
  }
  __syncwarp();
  const uint32_t R = roff[q.nk];
  const uint32_t span = min(lg.tail - lg.head, min(q.need + R + lg.stale, POS_WORDS * 32));
  const uint32_t nw = (span + 31) / 32;
  uint32_t tw = 0, ti = 0;
  if (q.need) {
    for (uint32_t w = lane; w < nw; w += 32) posmap[w] = 0;
    __syncwarp();
    mark_window<8>(a, roff, kern, R, lg.head, nw * 32, posmap, lane, 32);
    __syncwarp();
    uint32_t ba = 0, bi = 0, w0 = 0;
    for (; w0 < nw && ba + bi < q.need; w0 += 32) {
      const uint32_t w = w0 + lane;
      uint32_t em = 0, im = 0;
      if (w < nw) {
        const uint32_t lo = w * 32, valid = span - lo >= 32 ? 0xFFFFFFFFu : (1u << (span - lo)) - 1u;
        const uint32_t ib = __ldg(a.inact_bits + w), e = valid & ~posmap[w];
        em = e & ~ib;
        im = e & ib;
      }
      const uint32_t c = __popc(em) | (__popc(im) << 16);
      uint32_t x = c;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= (uint32_t)o) x += y;
      }
      const uint32_t wpre = (ba | (bi << 16)) + x - c;  // packed ranks: both < 2^15
      for (uint32_t k0 = 0; k0 < 8; k0 += SW_KB) {
        const uint32_t pre0 = __shfl_sync(0xffffffffu, wpre, 4 * k0);
        if (w0 + 4 * k0 >= nw || (pre0 & 0xFFFFu) + (pre0 >> 16) >= q.need) break;
        uint32_t wp[SW_KB], e32[SW_KB], i32[SW_KB], p32[SW_KB];
#pragma unroll
        for (uint32_t u = 0; u < SW_KB; ++u) {
          const uint32_t wd = 4 * (k0 + u) + (lane >> 3);
          wp[u] = w0 + wd;
          e32[u] = __shfl_sync(0xffffffffu, em, wd);
          i32[u] = __shfl_sync(0xffffffffu, im, wd);
          p32[u] = __shfl_sync(0xffffffffu, wpre, wd);
        }
        emit_chunks<SW_KB>(a, q, lg, lane, wp, e32, i32, p32, tw, ti);
      }
      const uint32_t tot = __shfl_sync(0xffffffffu, x, 31);
      ba += tot & 0xFFFFu;
      bi += tot >> 16;
    }
    tw = __reduce_add_sync(0xffffffffu, tw);
    ti = __reduce_add_sync(0xffffffffu, ti);
    if (lane == 0) scanned += min(span, 32 * w0);
  }
  if (lane == 0) {
    write_range(a, q, tw, ti);
    victims += tw + ti;
  }
}

// A big window, the whole CTA: marks, one block scan over the words (thread t
// owns words 4t .. 4t+3), the warps split the chunks.
__device__ __forceinline__ void cta_window(const PredArgs &a, const SelLog &lg, uint32_t qi, uint32_t *sm,
                                           uint32_t *ws, uint32_t *s_cnt, unsigned long long &scanned,
                                           unsigned long long &victims) {
  const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const Geo &g = a.g;
  uint32_t *posmap = sm, *wem = sm + POS_WORDS, *wim = wem + POS_WORDS, *wpre = wim + POS_WORDS;
  uint32_t *roff = wpre + POS_WORDS, *kern = roff + g.N + 2;
  const SelQuery q = load_query(a, qi);
  for (uint32_t d = tid; d <= q.nk; d += WSEL_NT) {
    roff[d] = __ldg(a.qroff + (uint64_t)qi * (g.N + 2) + d);
    if (d < q.nk) kern[d] = __ldg(a.qkern + (uint64_t)qi * (g.N + 1) + d);
  }
  for (uint32_t w = tid; w < POS_WORDS; w += WSEL_NT) posmap[w] = 0;
  if (tid == 0) s_cnt[0] = s_cnt[1] = 0;
  __syncthreads();
  const uint32_t R = roff[q.nk];
  const uint32_t span = min(lg.tail - lg.head, min(q.need + R + lg.stale, POS_WORDS * 32));
  const uint32_t nw = (span + 31) / 32;
  if (q.need) {
    mark_window<4>(a, roff, kern, R, lg.head, POS_WORDS * 32, posmap, tid, WSEL_NT);
    __syncthreads();
    uint32_t ca[4], ci[4], em[4], imk[4], tot = 0;
#pragma unroll
    for (uint32_t u = 0; u < 4; ++u) {  // nw <= POS_WORDS = 4 * WSEL_NT
      const uint32_t w = 4 * tid + u;
      em[u] = imk[u] = 0;
      if (w < nw) {
        const uint32_t lo = w * 32, valid = span - lo >= 32 ? 0xFFFFFFFFu : (1u << (span - lo)) - 1u;
        const uint32_t ib = __ldg(a.inact_bits + w), e = valid & ~posmap[w];
        em[u] = e & ~ib;
        imk[u] = e & ib;
      }
      ca[u] = __popc(em[u]);
      ci[u] = __popc(imk[u]);
      tot += ca[u] | (ci[u] << 16);
    }
    uint32_t tsum;
    uint32_t pre = block_excl_scan(tot, ws, &tsum);  // packed (inactive << 16 | active)
#pragma unroll
    for (uint32_t u = 0; u < 4; ++u) {
      const uint32_t w = 4 * tid + u;
      if (w < nw) {
        wem[w] = em[u];
        wim[w] = imk[u];
        wpre[w] = pre;
      }
      pre += ca[u] | (ci[u] << 16);
    }
    __syncthreads();
    constexpr uint32_t UC = 2;
    uint32_t tw = 0, ti = 0;
    const uint32_t nch = (nw + 3) / 4;
    for (uint32_t ch0 = wid; ch0 < nch; ch0 += SEL_NW * UC) {
      {
        const uint32_t p0 = wpre[4 * ch0];  // the step's first chunk starts past the cut: so do the rest
        if ((p0 & 0xFFFFu) + (p0 >> 16) >= q.need) break;
      }
      uint32_t wp[UC], e32[UC], i32[UC], p32[UC];
#pragma unroll
      for (uint32_t u = 0; u < UC; ++u) {
        const uint32_t w = 4 * (ch0 + u * SEL_NW) + (lane >> 3);
        wp[u] = w;
        e32[u] = w < nw ? wem[w] : 0u;
        i32[u] = w < nw ? wim[w] : 0u;
        p32[u] = w < nw ? wpre[w] : 0xFFFFFFFFu;
      }
      emit_chunks<UC>(a, q, lg, lane, wp, e32, i32, p32, tw, ti);
    }
    tw = __reduce_add_sync(0xffffffffu, tw);
    ti = __reduce_add_sync(0xffffffffu, ti);
    if (lane == 0 && (tw | ti)) {
      atomicAdd(&s_cnt[0], tw);
      atomicAdd(&s_cnt[1], ti);
    }
    __syncthreads();
  }
  if (tid == 0) {
    write_range(a, q, s_cnt[0], s_cnt[1]);
    victims += s_cnt[0] + s_cnt[1];
    if (q.need) scanned += span;
  }
}

__global__ void __launch_bounds__(WSEL_NT, 4) k_select_fast(PredArgs a) {
  extern __shared__ uint4 sel4[];
  __shared__ uint32_t ws[SEL_NW], s_cnt[2];
  const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  if (__ldcg(&a.st->log_dirty)) return;  // k_select_stale's case
  uint32_t *sm = reinterpret_cast<uint32_t *>(sel4);
  uint32_t ccnt[NQCLS], nfast = 0, nbig = 0;
#pragma unroll
  for (int c = 0; c < NQCLS; ++c) {
    ccnt[c] = __ldcg(&a.st->q_cls[c]);
    nfast += ccnt[c];
    if (c < (int)BIG_CLS) nbig += ccnt[c];
  }
  SelLog lg;
  lg.head = __ldcg(&a.st->lrm_head);
  lg.tail = __ldcg(&a.st->lrm_tail);
  lg.stale = lg.tail - lg.head - __ldcg(&a.st->n_resident);
  lg.al = (lg.head & 3u) == 0;
  const uint32_t nitems = nbig + (nfast - nbig + SEL_NW - 1) / SEL_NW;
  unsigned long long scanned = 0, victims = 0;
  for (uint32_t it = blockIdx.x; it < nitems; it += gridDim.x) {
    if (it < nbig) {
      cta_window(a, lg, fast_query(a, ccnt, it), sm, ws, s_cnt, scanned, victims);
    } else {
      const uint32_t j = nbig + (it - nbig) * SEL_NW + wid;
      if (j < nfast) warp_window(a, lg, fast_query(a, ccnt, j), sm + wid * sw_words(a.g.N), scanned, victims);
    }
    __syncthreads();  // the next item reuses the shared state
  }
  scanned = __reduce_add_sync(0xffffffffu, (unsigned)scanned);
  victims = __reduce_add_sync(0xffffffffu, (unsigned)victims);
  if (lane == 0 && (scanned | victims)) {
    ctr_add(a.st, DUM_CTR_FAST_SCANNED, scanned);
    ctr_add(a.st, DUM_CTR_FAST_VICTIMS, victims);
  }
}

// One warp step of the stale-entry path: the 32 log entries at positions
// head + r0 + lane (r0 a multiple of 32 relative to head, so that one
// broadcast word of the position bitmap covers them).  Eligible = inside the
// log, not a resident window block, still resident with its stamp; returns the
// active / inactive eligible ballots.  v = the entry (block | inactive << 31).
__device__ __forceinline__ void step_masks(const SelectOut &so, const uint32_t *posmap, uint32_t head,
                                           uint32_t tail, uint32_t lane, uint32_t r0, uint32_t v, uint32_t &ma,
                                           uint32_t &mi) {
  const uint32_t p = head + r0 + lane;
  const uint32_t w = (r0 >> 5) < POS_WORDS ? posmap[r0 >> 5] : 0xFFFFFFFFu;  // beyond the map: never reached
  bool el = p < tail && !((w >> lane) & 1u);
  if (el) {
    const uint32_t b = v & 0x7FFFFFFFu;
    el = __ldg(&so.frame_of[b]) != NONE && __ldg(&so.stamp_of[b]) == __ldcg(so.lrm_stamp + p);
  }
  ma = __ballot_sync(0xffffffffu, el && !(v >> 31));
  mi = __ballot_sync(0xffffffffu, el && (v >> 31));
}

constexpr uint32_t FB = 8;  // warp steps with their entry loads in flight together

__global__ void __launch_bounds__(WSEL_NT) k_select_stale(PredArgs a) {
  __shared__ uint32_t kern[MAXN + 1], roff[MAXN + 2];
  __shared__ uint32_t posmap[POS_WORDS];
  __shared__ uint32_t seg_cnt[FSEG_MAX], seg_pre[FSEG_MAX];
  __shared__ uint32_t s_tw, s_ti;
  constexpr uint32_t NW = WSEL_NT / 32;
  const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const Geo &g = a.g;
  const SelectOut &so = a.so;
  if (!__ldcg(&a.st->log_dirty)) return;  // k_select_fast's case
  uint32_t ccnt[NQCLS], nfast = 0;
#pragma unroll
  for (int c = 0; c < NQCLS; ++c) {
    ccnt[c] = __ldcg(&a.st->q_cls[c]);
    nfast += ccnt[c];
  }
  const uint32_t head = __ldcg(&a.st->lrm_head);
  const uint32_t tail = __ldcg(&a.st->lrm_tail);
  const uint32_t stale = tail - head - __ldcg(&a.st->n_resident);
  for (uint32_t bq = blockIdx.x; bq < nfast; bq += gridDim.x) {
    const uint32_t qi = fast_query(a, ccnt, bq);
    const uint32_t nk = __ldg(a.qnk + qi);
    for (uint32_t d = tid; d <= nk; d += WSEL_NT) {
      roff[d] = __ldg(a.qroff + (uint64_t)qi * (g.N + 2) + d);
      if (d < nk) kern[d] = __ldg(a.qkern + (uint64_t)qi * (g.N + 1) + d);
    }
    for (uint32_t w = tid; w < POS_WORDS; w += WSEL_NT) posmap[w] = 0;
    if (tid == 0) {
      s_tw = 0;
      s_ti = 0;
    }
    const uint32_t need = __ldg(a.qneed + qi);
    const unsigned long long bwb = __ldg(a.qvb + 2 * qi), binv = __ldg(a.qvb + 2 * qi + 1);
    const bool ok = bwb + need <= so.cap && binv + need <= so.cap;
    __syncthreads();
    const uint32_t R = nk ? roff[nk] : 0;
    uint32_t nseg = 0;
    if (need) {
      // 1. the window's resident blocks: their log positions into the bitmap
      {
        constexpr uint32_t MU = 4;  // loads in flight per thread
        uint32_t lo = 0;
        for (uint32_t x0 = tid; x0 < R; x0 += WSEL_NT * MU) {
          uint32_t r[MU];
#pragma unroll
          for (uint32_t u = 0; u < MU; ++u) {
            const uint32_t x = x0 + u * WSEL_NT;
            r[u] = NONE;
            if (x < R) {
              while (roff[lo + 1] <= x) ++lo;
              r[u] = __ldg(a.respos + (uint64_t)kern[lo] * g.walk_cap + (x - roff[lo])) - head;
            }
          }
#pragma unroll
          for (uint32_t u = 0; u < MU; ++u)
            if (r[u] < POS_WORDS * 32) atomicOr(&posmap[r[u] >> 5], 1u << (r[u] & 31));
        }
      }
      const uint32_t span = min(tail - head, min(need + R + stale, POS_WORDS * 32));
      // segments of FSEG positions relative to head; a warp step covers 32
      nseg = (span + FSEG - 1) / FSEG;
      __syncthreads();
      // 2. pass 1: eligible entries per segment (active | inactive << 16)
      for (uint32_t sg = wid; sg < nseg; sg += NW) {
        uint32_t na = 0, ni = 0;
        for (uint32_t k0 = 0; k0 < FSEG / 32; k0 += FB) {
          uint32_t v[FB];
#pragma unroll
          for (uint32_t u = 0; u < FB; ++u) {
            const uint32_t p = head + sg * FSEG + 32 * (k0 + u) + lane;
            v[u] = p < tail ? __ldcg(so.lrm_blk + p) : 0u;
          }
#pragma unroll
          for (uint32_t u = 0; u < FB; ++u) {
            uint32_t ma, mi;
            step_masks(so, posmap, head, tail, lane, sg * FSEG + 32 * (k0 + u), v[u], ma, mi);
            na += __popc(ma);
            ni += __popc(mi);
          }
        }
        if (lane == 0) seg_cnt[sg] = na | (ni << 16);
      }
      __syncthreads();
      // 3. segment prefix (one warp; nseg <= 32)
      if (wid == 0) {
        const uint32_t c = lane < nseg ? seg_cnt[lane] : 0u;
        uint32_t x = c;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
          if (lane >= (uint32_t)o) x += y;
        }
        if (lane < nseg) seg_pre[lane] = x - c;
      }
      __syncthreads();
      // 4. pass 2: the entries of combined rank < need, at their list ranks
      const uint32_t lt = (1u << lane) - 1;
      uint32_t tw = 0, ti = 0;
      for (uint32_t sg = wid; sg < nseg; sg += NW) {
        const uint32_t pre = seg_pre[sg];
        uint32_t rw = pre & 0xFFFFu, ri = pre >> 16;
        for (uint32_t k0 = 0; k0 < FSEG / 32 && rw + ri < need; k0 += FB) {
          uint32_t v[FB];
#pragma unroll
          for (uint32_t u = 0; u < FB; ++u) {
            const uint32_t p = head + sg * FSEG + 32 * (k0 + u) + lane;
            v[u] = p < tail ? __ldcg(so.lrm_blk + p) : 0u;
          }
#pragma unroll
          for (uint32_t u = 0; u < FB; ++u) {
            uint32_t ma, mi;
            step_masks(so, posmap, head, tail, lane, sg * FSEG + 32 * (k0 + u), v[u], ma, mi);
            const uint32_t ra = rw + __popc(ma & lt), rr = ri + __popc(mi & lt);
            const bool ea = (ma >> lane) & 1u, ei = (mi >> lane) & 1u;
            if ((ea || ei) && ra + rr < need) {
              if (ok) {
                if (ei) so.inv[binv + rr] = v[u] & 0x7FFFFFFFu;
                else so.wb[bwb + ra] = v[u];
              }
              tw += ea;
              ti += ei;
            }
            rw += __popc(ma);
            ri += __popc(mi);
          }
        }
      }
      tw = __reduce_add_sync(0xffffffffu, tw);
      ti = __reduce_add_sync(0xffffffffu, ti);
      if (lane == 0 && (tw | ti)) {
        atomicAdd(&s_tw, tw);
        atomicAdd(&s_ti, ti);
      }
      __syncthreads();
    }
    if (tid == 0) {
      uint64_t *o = so.out_range + 4ull * qi;
      o[0] = bwb;
      o[1] = bwb + (ok ? s_tw : 0);
      o[2] = binv;
      o[3] = binv + (ok ? s_ti : 0);
      // log entries read by the selection: the segments (each pass reads them)
      ctr_add(a.st, DUM_CTR_FAST_SCANNED, need ? min(tail - head, nseg * FSEG) : 0u);
      ctr_add(a.st, DUM_CTR_FAST_VICTIMS, s_tw + s_ti);
      ctr_add(a.st, DUM_CTR_FAST_DIRTY, 1);
    }
    __syncthreads();  // the next query reuses the shared state
  }
}

static uint32_t index_grid(const dum_engine *e) {
  return std::max<uint32_t>(1, std::min<uint32_t>(e->g.Emax, 148 * 4));
}

// Build end: the walk index of the walks just rebuilt (k_walk / k_walk_slow).
cudaError_t launch_walk_index(dum_engine *e, cudaStream_t main) {
  // on the third side stream: the next predict's prelude (residency load, ingest,
  // queries, walk residency facts) overlaps it; k_chain waits for ev_widx
  cudaEventRecord(e->ev_fork2, main);
  cudaStream_t s = e->side3;
  cudaStreamWaitEvent(s, e->ev_fork2, 0);
  const uint32_t grid = index_grid(e);
  TimerScope t(e, DUM_T_WALK_INDEX, s);
  cudaMemsetAsync(e->d_bcnt, 0, 4ull * e->g.W, s);
  k_walk_count<<<grid, IX_NT, 0, s>>>(e->d_walk, e->d_walk_len, e->g.walk_cap, e->d_state, e->d_bcnt, e->d_bhold);
  k_walk_conf<<<grid, IX_NT, 0, s>>>(e->d_walk, e->d_walk_len, e->g.walk_cap, e->d_state, e->d_bcnt, e->d_bhold,
                                     e->d_conf, e->d_conf_n);
  cudaEventRecord(e->ev_widx, s);
  e->kernel_launches += 2;
  return cudaGetLastError();
}

// The LRM log's inactive entries as a bitmap over positions relative to the
// head (bit l of word w = entry head + 32 w + l is inactive): the fast
// selection's clean-log path splits write-back / invalidate by popcounts.
__global__ void __launch_bounds__(256) k_log_bits(const uint32_t *__restrict__ lrm_blk, const DevState *st,
                                                  uint32_t *bits) {
  const uint32_t head = __ldcg(&st->lrm_head), tail = __ldcg(&st->lrm_tail);
  const uint32_t nw = (tail - head + 31) / 32, lane = threadIdx.x & 31;
  for (uint32_t w = (blockIdx.x * 256 + threadIdx.x) >> 5; w < nw; w += gridDim.x * 8) {
    const uint32_t p = head + 32 * w + lane;
    const uint32_t m = __ballot_sync(0xffffffffu, p < tail && (__ldg(lrm_blk + p) >> 31));
    if (lane == 0) bits[w] = m;
  }
}

// Predict time: per-walk residency facts for the fast selection.
cudaError_t launch_walk_res(dum_engine *e, cudaStream_t s) {
  TimerScope t(e, DUM_T_WALK_RES, s);
  k_walk_res<<<index_grid(e), IX_NT, 0, s>>>(e->d_walk, e->d_walk_len, e->g.walk_cap, e->d_state, e->d_res_bits,
                                             e->d_logpos, e->d_wnr, e->d_wnres, e->d_respos);
  k_log_bits<<<std::min<uint32_t>(e->lrm_cap / 256 + 1, 148 * 4), 256, 0, s>>>(e->d_lrm_blk, e->d_state,
                                                                              e->d_log_bits);
  e->kernel_launches += 2;
  return cudaGetLastError();
}

cudaError_t launch_window(dum_engine *e, const PredArgs &a, bool select, cudaStream_t s) {
  const int ssmem = (int)(sel_smem_words(e->g.N) * 4);
  if (!e->copy_grid || e->sel_smem != ssmem) {
    int dev = 0, sms = 148, nc = 1, ns = 1, nt = 1;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    // the attribute is per device and function: raised by every engine on its own device
    if (ssmem > 48 * 1024) cudaFuncSetAttribute(k_select_fast, cudaFuncAttributeMaxDynamicSharedMemorySize, ssmem);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nc, k_copy_fast, COPY_NT, 0);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ns, k_select_fast, WSEL_NT, ssmem);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nt, k_select_stale, WSEL_NT, 0);
    e->copy_grid = (uint32_t)std::max(1, nc * sms);
    e->sel_grid = (uint32_t)std::max(1, ns * sms);
    e->stale_grid = (uint32_t)std::max(1, nt * sms);
    e->sel_smem = ssmem;
  }
  if (select) {
    // the selection on the third side stream, beside the copy (each kernel
    // exits at once in the other's case: clean log / stale entries)
    cudaEventRecord(e->ev_fork2, s);
    cudaStreamWaitEvent(e->side3, e->ev_fork2, 0);
    {
      TimerScope t(e, DUM_T_SELECT_FAST, e->side3);
      k_select_fast<<<std::min(a.nq, e->sel_grid), WSEL_NT, ssmem, e->side3>>>(a);
      k_select_stale<<<std::min(a.nq, e->stale_grid), WSEL_NT, 0, e->side3>>>(a);
    }
    cudaEventRecord(e->ev_join3, e->side3);
    e->kernel_launches += 2;
  }
  {  // every fast window's pairs: the flat copy over k_chain's chunk map
    TimerScope t(e, DUM_T_PREDICT, s);
    k_copy_fast<<<e->copy_grid, COPY_NT, 0, s>>>(a);
  }
  e->kernel_launches += 1;
  if (select) cudaStreamWaitEvent(s, e->ev_join3, 0);
  return cudaGetLastError();
}

}  // namespace dum
