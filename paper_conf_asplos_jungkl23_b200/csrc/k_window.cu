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
// k_window marks those positions in a shared-memory bitmap over
// [head, head + POS_BITS) of the LRM log and runs the same ordered selection
// as the exact path (select_tail.cuh) on it.  k_chain only routes a query
// here when the selection provably ends inside that range.
//
//  k_walk_count  (build end)   holders of each block: bcnt[b], bhold[b][..]
//  k_walk_conf   (build end)   conflicts of each walk: conf[e][..], conf_n[e]
//  k_walk_res    (predict)     per walk: non-resident count, resident positions
//  k_copy_fast   (predict)     flat copy of every fast window (chunk map from k_chain)
//  k_select_fast (predict)     one CTA per fast query: marking + ordered selection
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
  const uint32_t E = *(const volatile uint32_t *)&st->E;
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
  const uint32_t E = *(const volatile uint32_t *)&st->E;
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
  const uint32_t E = *(const volatile uint32_t *)&st->E;
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

// Flat copy of every fast query's window: warp-granular work items of 128
// window blocks (one list of one query; chunk map from k_chain), two in flight
// per warp, lane-consecutive 4 B loads of the cached walk and 8 B streaming
// stores of the (block, exec) pairs.  Persistent grid over the device count.
__global__ void __launch_bounds__(COPY_NT) k_copy_fast(PredArgs a) {
  constexpr uint32_t UN = 2;
  const uint32_t lane = threadIdx.x & 31;
  const uint64_t G = *(volatile unsigned long long *)&a.st->pool_chunks;
  const uint64_t nw = (uint64_t)gridDim.x * (COPY_NT / 32);
  const uint32_t N = a.g.N;
  uint2 *out = reinterpret_cast<uint2 *>(a.pairs);
  unsigned long long emitted = 0;
  for (uint64_t c0 = (uint64_t)blockIdx.x * (COPY_NT / 32) + (threadIdx.x >> 5); c0 < G; c0 += nw * UN) {
    unsigned long long m[UN];
#pragma unroll
    for (uint32_t u = 0; u < UN; ++u) m[u] = c0 + u * nw < G ? __ldcg(a.chunk_map + c0 + u * nw) : ~0ull;
    uint32_t kd[UN], lo[UN], L[UN], i0[UN];
    unsigned long long base[UN];
#pragma unroll
    for (uint32_t u = 0; u < UN; ++u) {
      if (m[u] == ~0ull) continue;
      const uint32_t q = (uint32_t)(m[u] >> 40), d = (uint32_t)(m[u] >> 32) & 0xFFu;
      i0[u] = (uint32_t)(m[u] & 0xFFFFFFFFu) * CHUNK_B;
      kd[u] = __ldcg(a.qkern + (uint64_t)q * (N + 1) + d);
      lo[u] = __ldcg(a.qloff + (uint64_t)q * (N + 2) + d);
      L[u] = __ldcg(a.qloff + (uint64_t)q * (N + 2) + d + 1) - lo[u];
      base[u] = __ldcg(a.qbase + q);
    }
    uint32_t b[UN][4];
#pragma unroll
    for (uint32_t u = 0; u < UN; ++u) {
      if (m[u] == ~0ull) continue;
      const uint32_t *lst = a.walk + (uint64_t)kd[u] * a.g.walk_cap;
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) {
        const uint32_t i = i0[u] + 32 * k + lane;
        b[u][k] = i < L[u] ? __ldg(lst + i) : NONE;
      }
    }
#pragma unroll
    for (uint32_t u = 0; u < UN; ++u) {
      if (m[u] == ~0ull) continue;
      if (base[u] + lo[u] + L[u] > a.cap) continue;  // capacity error raised by k_chain
      uint2 *o = out + base[u] + lo[u];
#pragma unroll
      for (uint32_t k = 0; k < 4; ++k) {
        const uint32_t i = i0[u] + 32 * k + lane;
        if (i < L[u]) __stcs(o + i, make_uint2(b[u][k], kd[u]));
      }
      if (lane == 0) emitted += min(CHUNK_B, L[u] - i0[u]);
    }
  }
  emitted = __reduce_add_sync(0xffffffffu, (unsigned)emitted);
  if (lane == 0 && emitted) {
    ctr_add(a.st, DUM_CTR_EMITTED, emitted);
    ctr_add(a.st, DUM_CTR_GATHERED, emitted);
    ctr_add(a.st, DUM_CTR_FAST_EMITTED, emitted);
  }
}

// Fused a8 of one fast query per CTA (k_chain's order: fast queries by
// decreasing `need`).  need = max(0, window blocks without a frame - free
// frames) and the victim ranges come from k_chain (D18).  The victims are the
// first `need` entries of the LRM log, oldest first, that are still resident
// with their stamp and not in the window, split by the
// inactive bit of the entry into invalidate / write-back (L285; D19, D20).
//   1. mark the log positions of the window's resident blocks (flat over the
//      lists' respos entries, prefix qroff from k_chain) in a bitmap over
//      [head, head + 32 POS_WORDS);
//   2. the log prefix [head, head + span) (span = need + resident window
//      blocks + stale entries: the selection provably ends inside) is cut
//      into 1024-entry segments; pass 1: each warp counts the eligible
//      active / inactive entries of its segments;
//   3. one warp scans the segment counts;
//   4. pass 2: each warp re-reads its segments and writes the entries of
//      combined rank < need at their ranks in the two lists (LRM order).
// Two CTA barriers per query instead of two per 2048-entry chunk.
constexpr uint32_t FSEG = 1024;                 // log entries per segment (32 per lane)
constexpr uint32_t FSEG_MAX = POS_WORDS * 32 / FSEG;
static_assert(FSEG_MAX <= 32, "one warp scans the segment counts");

// One warp step of the selection: the 32 log entries at positions
// head + r0 + lane (r0 a multiple of 32 relative to head, so that one
// broadcast word of the position bitmap covers them).  Eligible = inside the
// log, not a resident window block, still resident with its stamp; returns the
// active / inactive eligible ballots.  v = the entry (block | inactive << 31).
__device__ __forceinline__ void step_masks(const SelectOut &so, const uint32_t *posmap, uint32_t head,
                                           uint32_t tail, bool clean, uint32_t lane, uint32_t r0, uint32_t v,
                                           uint32_t &ma, uint32_t &mi) {
  const uint32_t p = head + r0 + lane;
  const uint32_t w = (r0 >> 5) < POS_WORDS ? posmap[r0 >> 5] : 0xFFFFFFFFu;  // beyond the map: never reached
  bool el = p < tail && !((w >> lane) & 1u);
  if (!clean && el) {
    const uint32_t b = v & 0x7FFFFFFFu;
    el = __ldg(&so.frame_of[b]) != NONE && __ldg(&so.stamp_of[b]) == __ldcg(so.lrm_stamp + p);
  }
  ma = __ballot_sync(0xffffffffu, el && !(v >> 31));
  mi = __ballot_sync(0xffffffffu, el && (v >> 31));
}

constexpr uint32_t FB = 8;  // warp steps with their entry loads in flight together

__global__ void __launch_bounds__(WSEL_NT, 6) k_select_fast(PredArgs a) {
  __shared__ uint32_t kern[MAXN + 1], roff[MAXN + 2], loff[MAXN + 2], goff[MAXN + 2];
  __shared__ uint32_t posmap[POS_WORDS];
  __shared__ uint32_t seg_cnt[FSEG_MAX], seg_pre[FSEG_MAX];
  __shared__ uint32_t wem[POS_WORDS], wim[POS_WORDS], wpre[POS_WORDS];  // clean-log word path
  __shared__ uint32_t s_need, s_head, s_tail, s_clean, s_ok, s_tw, s_ti, s_nres;
  __shared__ unsigned long long s_bwb, s_binv;
  constexpr uint32_t NW = WSEL_NT / 32;
  const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const Geo &g = a.g;
  const SelectOut &so = a.so;
  // the fast queries, class by class (k_chain: by decreasing `need`)
  uint32_t ccnt[NQCLS];
#pragma unroll
  for (int c = 0; c < NQCLS; ++c) ccnt[c] = *(volatile uint32_t *)&a.st->q_cls[c];
  uint32_t nfast = 0;
#pragma unroll
  for (int c = 0; c < NQCLS; ++c) nfast += ccnt[c];
  for (uint32_t bq = blockIdx.x; bq < nfast; bq += gridDim.x) {
    uint32_t cq = NQCLS, rq = bq;
#pragma unroll
    for (int c = 0; c < NQCLS; ++c)
      if (cq == NQCLS) {
        if (rq < ccnt[c]) cq = c;
        else rq -= ccnt[c];
      }
    const uint32_t qi = a.qperm[(uint64_t)cq * a.nq + rq];
    const uint32_t nk = a.qnk[qi];
    for (uint32_t d = tid; d <= nk; d += WSEL_NT) {
      roff[d] = a.qroff[(uint64_t)qi * (g.N + 2) + d];
      loff[d] = a.qloff[(uint64_t)qi * (g.N + 2) + d];
      goff[d] = a.qgoff[(uint64_t)qi * (g.N + 2) + d];
      if (d < nk) kern[d] = a.qkern[(uint64_t)qi * (g.N + 1) + d];
    }
    for (uint32_t w = tid; w < POS_WORDS; w += WSEL_NT) posmap[w] = 0;
    if (tid == 0) {
      const uint32_t need = a.qneed[qi];
      s_need = need;
      s_bwb = a.qvb[2 * qi];
      s_binv = a.qvb[2 * qi + 1];
      s_ok = s_bwb + need <= so.cap && s_binv + need <= so.cap;
      s_head = *(volatile uint32_t *)&a.st->lrm_head;
      s_tail = *(volatile uint32_t *)&a.st->lrm_tail;
      s_clean = *(volatile uint32_t *)&a.st->log_dirty == 0;
      s_nres = *(volatile uint32_t *)&a.st->n_resident;
      s_tw = 0;
      s_ti = 0;
    }
    __syncthreads();
    const uint32_t need = s_need, head = s_head, tail = s_tail;
    const bool clean = s_clean, ok = s_ok;
    const unsigned long long bwb = s_bwb, binv = s_binv;
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
      const uint32_t stale = tail - head - s_nres;
      const uint32_t span = min(tail - head, min(need + R + stale, POS_WORDS * 32));
      __syncthreads();
      if (clean && a.inact_bits) {
        // ---- clean log: word-level selection.  Every entry of [head, tail) is
        // valid, so a 32-position word's eligible entries are ~excluded & valid,
        // split by the log's inactive-entry bitmap (k_log_bits): counts and
        // ranks come from popcounts; only the taken entries are read. ----
        const uint32_t nw = (span + 31) / 32;
        uint32_t ca[4], ci[4], em[4], imk[4];
        uint32_t tot = 0;
#pragma unroll
        for (uint32_t u = 0; u < 4; ++u) {  // thread t owns words 4t .. 4t+3 (nw <= POS_WORDS = 4 * WSEL_NT)
          const uint32_t w = 4 * tid + u;
          em[u] = imk[u] = 0;
          if (w < nw) {
            const uint32_t lo = w * 32, valid = span - lo >= 32 ? 0xFFFFFFFFu : (1u << (span - lo)) - 1u;
            const uint32_t ib = __ldg(a.inact_bits + w);
            const uint32_t e = valid & ~posmap[w];
            em[u] = e & ~ib;
            imk[u] = e & ib;
          }
          ca[u] = __popc(em[u]);
          ci[u] = __popc(imk[u]);
          tot += ca[u] | (ci[u] << 16);
        }
        uint32_t tsum;
        const uint32_t tpre = block_excl_scan(tot, seg_pre, &tsum);  // packed (inactive << 16 | active)
        {
          uint32_t pre = tpre;
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
        }
        __syncthreads();
        // a warp per 128-position chunk (4 words), a lane per 4 consecutive
        // positions: the eligible entries of combined rank < need, written at
        // their list ranks.  head is 16 B aligned for the vector load when
        // possible; otherwise 4 scalar loads.
        uint32_t tw = 0, ti = 0;
        const uint32_t nch = (nw + 3) / 4;
        const bool al = (head & 3u) == 0;
        for (uint32_t ch = wid; ch < nch; ch += NW) {
          const uint32_t w = 4 * ch + (lane >> 3), sh = (lane & 7) * 4;
          const uint32_t pre = w < nw ? wpre[w] : 0xFFFFFFFFu;
          const uint32_t pre0 = __shfl_sync(0xffffffffu, pre, 0);
          if ((pre0 & 0xFFFFu) + (pre0 >> 16) >= need) break;  // chunks only grow: the cut is behind
          const uint32_t a4 = w < nw ? (wem[w] >> sh) & 0xFu : 0u, i4 = w < nw ? (wim[w] >> sh) & 0xFu : 0u;
          // ranks: the word's prefix + the eligible entries of the lower lanes of the same word
          uint32_t c = __popc(a4) | (__popc(i4) << 16), x = c;
#pragma unroll
          for (int o = 1; o < 8; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
            if ((lane & 7) >= (uint32_t)o) x += y;
          }
          uint32_t ra = (pre & 0xFFFFu) + ((x - c) & 0xFFFFu), rr = (pre >> 16) + ((x - c) >> 16);
          if ((a4 | i4) && ra + rr < need) {
            const uint32_t p = head + 32 * w + sh;
            uint32_t vv[4];
            if (al) {
              const uint4 q = __ldcg(reinterpret_cast<const uint4 *>(so.lrm_blk + p));
              vv[0] = q.x; vv[1] = q.y; vv[2] = q.z; vv[3] = q.w;
            } else {
#pragma unroll
              for (uint32_t u = 0; u < 4; ++u) vv[u] = ((a4 | i4) >> u) & 1u ? __ldcg(so.lrm_blk + p + u) : 0u;
            }
#pragma unroll
            for (uint32_t u = 0; u < 4; ++u) {
              const bool ea = (a4 >> u) & 1u, ei = (i4 >> u) & 1u;
              if ((ea || ei) && ra + rr < need) {
                if (ok) {
                  if (ei) so.inv[binv + rr] = vv[u] & 0x7FFFFFFFu;
                  else so.wb[bwb + ra] = vv[u];
                }
                tw += ea;
                ti += ei;
              }
              ra += ea;
              rr += ei;
            }
          }
        }
        tw = __reduce_add_sync(0xffffffffu, tw);
        ti = __reduce_add_sync(0xffffffffu, ti);
        if (lane == 0 && (tw | ti)) {
          atomicAdd(&s_tw, tw);
          atomicAdd(&s_ti, ti);
        }
        nseg = (span + FSEG - 1) / FSEG;  // (reported as scanned)
        __syncthreads();
      } else {
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
            step_masks(so, posmap, head, tail, clean, lane, sg * FSEG + 32 * (k0 + u), v[u], ma, mi);
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
            step_masks(so, posmap, head, tail, clean, lane, sg * FSEG + 32 * (k0 + u), v[u], ma, mi);
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
      }  // per-entry path (stale log entries)
    }
    if (tid == 0) {
      uint64_t *o = so.out_range + 4ull * qi;
      o[0] = bwb;
      o[1] = bwb + (ok ? s_tw : 0);
      o[2] = binv;
      o[3] = binv + (ok ? s_ti : 0);
      // log entries read by the selection: the segments (each pass reads them)
      ctr_add(a.st, DUM_CTR_FAST_SCANNED, need ? min(tail - head, nseg * FSEG) : 0u);  // (both passes read these)
      ctr_add(a.st, DUM_CTR_FAST_VICTIMS, s_tw + s_ti);
      if (!clean) ctr_add(a.st, DUM_CTR_FAST_DIRTY, 1);
    }
    // the window's (block, exec) pairs: every warp streams the lists (the copy
    // of this query overlaps the selection of the SM's other queries)
    {
      const unsigned long long base = a.qbase[qi];
      const uint32_t U = nk ? loff[nk] : 0;
      if (base + U <= a.cap) copy_window_lists(a, kern, loff, goff, nk, base, wid, NW, loff, nullptr);
      if (tid == 0) {
        ctr_add(a.st, DUM_CTR_EMITTED, U);
        ctr_add(a.st, DUM_CTR_GATHERED, U);
        ctr_add(a.st, DUM_CTR_FAST_EMITTED, U);
      }
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
  const uint32_t head = *(const volatile uint32_t *)&st->lrm_head, tail = *(const volatile uint32_t *)&st->lrm_tail;
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
  if (!e->copy_grid) {
    int dev = 0, sms = 148, nc = 1, ns = 1;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nc, k_copy_fast, COPY_NT, 0);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ns, k_select_fast, WSEL_NT, 0);
    e->copy_grid = (uint32_t)std::max(1, nc * sms);
    e->sel_grid = (uint32_t)std::max(1, ns * sms);
  }
  if (!select) {  // prefetch windows only: the flat copy
    TimerScope t(e, DUM_T_PREDICT, s);
    k_copy_fast<<<e->copy_grid, COPY_NT, 0, s>>>(a);
  } else {  // one CTA per window: selection, then its pairs
    TimerScope t(e, DUM_T_PREDICT, s);
    k_select_fast<<<std::min(a.nq, e->sel_grid), WSEL_NT, 0, s>>>(a);
  }
  e->kernel_launches += 1;
  return cudaGetLastError();
}

}  // namespace dum
