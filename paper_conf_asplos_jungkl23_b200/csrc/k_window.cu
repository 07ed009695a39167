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
//  k_window_fast (predict+select) one persistent kernel, a work queue: the
//                              flat copy interleaved with the selection (clean
//                              log: marking + word-level ranks, then emit
//                              groups; stale entries: per-entry selection)
#include <algorithm>

#include "device_util.cuh"
#include "kernels.cuh"
#include "predict.cuh"
#include "select_tail.cuh"

#ifdef EXP_TRACE
// experiment builds only: globaltimer stamps of k_window_fast's work items
__device__ unsigned long long g_tr[4096 * 4 + 8 * 65536];
__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}
#define TR(i, v) (g_tr[(i)] = (v))
static void *g_tr_ptr() {
  void *p = nullptr;
  cudaGetSymbolAddress(&p, g_tr);
  return p;
}
#else
#define TR(i, v) ((void)0)
#endif

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
// Clean log (every entry of [head, tail) valid, the normal case): sel_staged,
// a query per item of the selection group (4 warps of a k_window_fast CTA).
// The window's resident-position lists, the log's inactive-entry words and the
// log prefix are staged in shared memory by TMA bulk copies; the positions
// are marked in a bitmap; a 32-position word's eligible entries are ~marked &
// valid, split by the inactive bits into write-back / invalidate; one group
// scan of the packed popcounts gives every word its rank base and locates the
// cut (the need-th eligible entry); then a lane per 4 consecutive entries of a
// word writes the entries of combined rank < need at their ranks, reading the
// log from the staged segments.
//
// Stale entries (a log not compacted since an eviction): sel_stale, a CTA
// item per query (same queue), per-entry eligibility (frame + stamp check):
//   1. marks as above;  2. pass 1: eligible active / inactive entries per
//   1024-entry segment, a warp per segment;  3. one warp scans the segment
//   counts;  4. pass 2: each warp re-reads its segments and writes the
//   entries of combined rank < need.
constexpr uint32_t FSEG = 1024;                 // log entries per segment (32 per lane)
constexpr uint32_t FSEG_MAX = POS_WORDS * 32 / FSEG;
static_assert(FSEG_MAX <= 32, "one warp scans the segment counts");

struct SelLog {  // the log, fixed during the kernel
  uint32_t head, tail, stale;
  bool al;       // head 16 B aligned: vector loads of the log
};

struct SelQuery {
  uint32_t qi, nk, need;
  unsigned long long bwb, binv;
  bool ok;
};

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

// The selection group of k_window_fast: warps [0, SG_NT / 32) of the CTA,
// synchronised by named barrier 1; the other warps copy pairs meanwhile.
constexpr uint32_t SG_NT = 128;
constexpr uint32_t SG_WPT = POS_WORDS / SG_NT;  // bitmap words per group thread
__device__ __forceinline__ void gsync() { asm volatile("bar.sync 1, %0;" ::"n"(SG_NT) : "memory"); }

// Exclusive scan of one value per group thread; ws holds SG_NT / 32 words.
__device__ __forceinline__ uint32_t group_excl_scan(uint32_t v, uint32_t *ws, uint32_t *total) {
  const uint32_t t = threadIdx.x, lane = t & 31, wid = t >> 5;
  uint32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= (uint32_t)o) x += y;
  }
  if (lane == 31) ws[wid] = x;
  gsync();
  uint32_t base = 0, tot = 0;
#pragma unroll
  for (uint32_t k = 0; k < SG_NT / 32; ++k) {
    const uint32_t c = ws[k];
    if (k < wid) base += c;
    tot += c;
  }
  gsync();  // ws is reused by the next call
  *total = tot;
  return base + x - v;
}

// A selection item's record (k_chain): {qi, nk, need, nw}, {first emit group,
// ok, -, -}, {wb base, inv base}.
struct SelRec {
  uint4 x, y, z;
};
__device__ __forceinline__ SelQuery rec_query(const SelRec &r) {
  SelQuery q;
  q.qi = r.x.x;
  q.nk = r.x.y;
  q.need = r.x.z;
  q.ok = r.y.y != 0;
  q.bwb = (unsigned long long)r.z.y << 32 | r.z.x;
  q.binv = (unsigned long long)r.z.w << 32 | r.z.z;
  return q;
}

// ---------------------------------------------------------------------------
// The clean-log selection of one fast query by the selection group.  The log
// prefix it scans is staged in shared memory by TMA bulk copies
// (cp.async.bulk, one mbarrier per buffer) in segments of SR_SEG entries,
// double-buffered so that the next segment lands while the current one is
// emitted, and so are the log's inactive-entry words; both are issued before
// the marking starts and land meanwhile.  (The resident-position lists are
// loaded with plain coalesced loads: one bulk copy per list -- ~33 small ones
// per query -- measured slower, 5-28 us to land.)
constexpr uint32_t SR_SEG = 4096;        // log entries per segment
constexpr uint32_t SR_SEGW = SR_SEG / 32;
constexpr uint32_t SR_SMEM_WORDS = POS_WORDS /*ibits*/ + POS_WORDS /*wpre*/ + 2 * (SR_SEG + 4);

__device__ __forceinline__ uint32_t sm_addr(const void *p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long *b) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sm_addr(b)) : "memory");
}
__device__ __forceinline__ void mbar_expect(unsigned long long *b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sm_addr(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, uint32_t bytes, unsigned long long *b) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
               ::"r"(sm_addr(dst)), "l"(src), "r"(bytes), "r"(sm_addr(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long *b, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n\tWAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra WAIT_%=;\n\t}" ::"r"(sm_addr(b)), "r"(parity) : "memory");
}

struct StageSm {
  uint32_t *ibits, *wpre, *lbuf;  // dynamic shared memory (SR_SMEM_WORDS)
  unsigned long long *bar;               // [3]: inactive-entry words, segment buffers 0 / 1
};

// Thread 0: the log segment k into buffer k & 1 (16 B aligned source; entries
// [k SR_SEG, min(span, (k + 1) SR_SEG)) relative to head, at offset head & 3).
__device__ __forceinline__ void issue_segment(const PredArgs &a, const SelLog &lg, const StageSm &S, uint32_t k,
                                              uint32_t span) {
  const uint32_t base = (lg.head + k * SR_SEG) & ~3u, o = (lg.head + k * SR_SEG) - base;
  uint32_t n = (min(SR_SEG, span - k * SR_SEG) + o + 3) & ~3u;
  n = min(n, a.lrm_cap - base);
  unsigned long long *b = S.bar + 1 + (k & 1);
  mbar_expect(b, 4 * n);
  bulk_g2s(S.lbuf + (k & 1) * (SR_SEG + 4), a.so.lrm_blk + base, 4 * n, b);
}

// Thread 0: the log's inactive-entry words [0, nw) (one bulk copy).
__device__ __forceinline__ void issue_bits(const PredArgs &a, const StageSm &S, uint32_t nw) {
  const uint32_t bytes = 4 * ((nw + 3) & ~3u);
  mbar_expect(S.bar, bytes);
  bulk_g2s(S.ibits, a.inact_bits, bytes, S.bar);
}

__device__ __forceinline__ void sel_staged(const PredArgs &a, const SelLog &lg, const SelRec &r, const StageSm &S,
                                           uint32_t *posmap, uint32_t *roff, uint32_t *kern, uint32_t *ws,
                                           uint32_t *s_cut, uint32_t (&ph)[3], unsigned long long &scanned,
                                           unsigned long long &victims, uint32_t it) {
  const uint32_t t = threadIdx.x, lane = t & 31, wid = t >> 5;  // t < SG_NT
#ifdef EXP_TRACE
#define TRI(j) if (t == 0) TR(4 * 4096 + 8 * it + (j), gtime())
#else
#define TRI(j) ((void)it)
#endif
  const Geo &g = a.g;
  const SelQuery q = rec_query(r);
  const uint32_t qi = q.qi, nw = q.need ? r.x.w : 0u;
  if (!nw) {  // nothing to evict: an empty range
    if (t == 0) write_range(a, q, 0, 0);
    return;
  }
  for (uint32_t d = t; d <= q.nk; d += SG_NT) {
    roff[d] = __ldg(a.qroff + (uint64_t)qi * (g.N + 2) + d);
    if (d < q.nk) kern[d] = __ldg(a.qkern + (uint64_t)qi * (g.N + 1) + d);
  }
  for (uint32_t w = t; w < nw; w += SG_NT) posmap[w] = 0;
  gsync();
  TRI(2);
  const uint32_t R = roff[q.nk];
#ifdef EXP_TRACE
  if (t == 0) TR(4 * 4096 + 8 * it + 6, (unsigned long long)R << 32 | nw);
  if (t == 0) TR(4 * 4096 + 8 * it + 7, (unsigned long long)q.nk << 32 | q.need);
#endif
  const uint32_t span = min(lg.tail - lg.head, min(q.need + R + lg.stale, POS_WORDS * 32));
  const uint32_t nseg = (span + SR_SEG - 1) / SR_SEG;
  if (t == 0) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");  // earlier generic accesses of the buffers
    issue_segment(a, lg, S, 0, span);
    if (nseg > 1) issue_segment(a, lg, S, 1, span);
    issue_bits(a, S, nw);
  }
  TRI(5);
  // marks: the window's resident positions below nw * 32, flat over the lists'
  // entries.  A walk's resident blocks sit mostly at consecutive log
  // positions: each lane takes ML consecutive entries (all loads in flight,
  // L1-served), ORs the bits of one bitmap word in a register and flushes it
  // with one shared atomic when the word changes.  (Measured against coalesced
  // loads + a warp match / reduce or a segmented shuffle OR per word: slower.)
  {
    constexpr uint32_t ML = 16;
    uint32_t lo = 0;
    for (uint32_t xb = 0; xb < R; xb += SG_NT * ML) {
      const uint32_t x0 = xb + t * ML;
      uint32_t rv[ML];
      uint32_t l2 = lo;
#pragma unroll
      for (uint32_t j = 0; j < ML; ++j) {
        const uint32_t x = x0 + j;
        rv[j] = NONE;
        if (x < R) {
          while (roff[l2 + 1] <= x) ++l2;
          rv[j] = __ldg(a.respos + (uint64_t)kern[l2] * g.walk_cap + (x - roff[l2])) - lg.head;
        }
      }
      lo = l2;
      uint32_t cw = NONE, cb = 0;
#pragma unroll
      for (uint32_t j = 0; j < ML; ++j) {
        const uint32_t wd = rv[j] < nw * 32 ? rv[j] >> 5 : NONE;
        if (wd != cw) {
          if (cw != NONE) atomicOr(&posmap[cw], cb);
          cw = wd;
          cb = 0;
        }
        if (wd != NONE) cb |= 1u << (rv[j] & 31);
      }
      if (cw != NONE) atomicOr(&posmap[cw], cb);
    }
  }
  TRI(3);
  mbar_wait(S.bar, ph[0]);  // the inactive-entry words
  ph[0] ^= 1u;
  gsync();
  // eligible entries per word (~marked & valid, split by the inactive bits),
  // rank bases by one group scan, the cut
  uint32_t em[SG_WPT], im[SG_WPT], tot = 0;
#pragma unroll
  for (uint32_t u = 0; u < SG_WPT; ++u) {
    const uint32_t w = SG_WPT * t + u;
    em[u] = im[u] = 0;
    if (w < nw) {
      const uint32_t lo = w * 32, valid = span - lo >= 32 ? 0xFFFFFFFFu : (1u << (span - lo)) - 1u;
      const uint32_t e = valid & ~posmap[w], ib = S.ibits[w];
      em[u] = e & ~ib;
      im[u] = e & ib;
    }
    tot += __popc(em[u]) | (__popc(im[u]) << 16);
  }
  if (t == 0) s_cut[0] = s_cut[1] = s_cut[2] = NONE;  // (ordered by the scan's barriers)
  uint32_t tsum;
  uint32_t pre = group_excl_scan(tot, ws, &tsum);  // packed (inactive << 16 | active); both <= 32768
#pragma unroll
  for (uint32_t u = 0; u < SG_WPT; ++u) {
    const uint32_t w = SG_WPT * t + u;
    if (w < nw) {
      S.wpre[w] = pre;
      posmap[w] = em[u];  // from here posmap holds the eligible write-back entries, ibits the invalidate ones
      S.ibits[w] = im[u];
      const uint32_t before = (pre & 0xFFFFu) + (pre >> 16), here = __popc(em[u] | im[u]);
      if (before < q.need && before + here >= q.need) {  // the cut is in this word: take k more entries
        uint32_t x = em[u] | im[u], mask = 0;
        for (uint32_t k = q.need - before; k; --k) {
          const uint32_t low = x & (0u - x);
          mask |= low;
          x ^= low;
        }
        s_cut[0] = (pre & 0xFFFFu) + __popc(em[u] & mask);  // taken write-back entries
        s_cut[1] = (pre >> 16) + __popc(im[u] & mask);     // taken invalidate entries
        s_cut[2] = w;
      }
    }
    pre += __popc(em[u]) | (__popc(im[u]) << 16);
  }
  gsync();
  TRI(4);
  const uint32_t wcut = s_cut[2] == NONE ? nw - 1 : s_cut[2];  // the last word with victims
  const uint32_t kend = (wcut * 32) / SR_SEG;                  // the last segment needed
  // emit, segment by segment: a lane per 4 consecutive entries of a word
  const uint32_t sh = (lane & 7) * 4, below = (1u << sh) - 1u;
  for (uint32_t k = 0; k <= kend; ++k) {
    mbar_wait(S.bar + 1 + (k & 1), ph[1 + (k & 1)]);
    ph[1 + (k & 1)] ^= 1u;
    const uint32_t *lb = S.lbuf + (k & 1) * (SR_SEG + 4) + ((lg.head + k * SR_SEG) & 3u);
    const uint32_t w0 = k * SR_SEGW, w1 = min(wcut + 1, w0 + SR_SEGW);
    for (uint32_t w = w0 + 4 * wid + (lane >> 3); w < w1; w += 4 * (SG_NT / 32)) {
      const uint32_t ea4 = posmap[w], ei4 = S.ibits[w], pw = S.wpre[w];
      uint32_t ra = (pw & 0xFFFFu) + __popc(ea4 & below), rr = (pw >> 16) + __popc(ei4 & below);
      const uint32_t am = (ea4 >> sh) & 0xFu, imk = (ei4 >> sh) & 0xFu;
      if (!(am | imk) || ra + rr >= q.need) continue;
      const uint32_t *e4 = lb + 32 * (w - w0) + sh;  // (the segment's start may not be 16 B aligned)
#pragma unroll
      for (uint32_t j = 0; j < 4; ++j) {
        const bool ea = (am >> j) & 1u, ei = (imk >> j) & 1u;
        if ((ea || ei) && ra + rr < q.need && q.ok) {
          if (ei) a.so.inv[q.binv + rr] = e4[j] & 0x7FFFFFFFu;
          else a.so.wb[q.bwb + ra] = e4[j];
        }
        ra += ea;
        rr += ei;
      }
    }
    if (k + 2 <= kend) {
      gsync();  // buffer k & 1 is read
      if (t == 0) {
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        issue_segment(a, lg, S, k + 2, span);
      }
    }
  }
  // segments issued but not needed (the cut came early): wait for them so
  // that the barriers' phases stay in step with the parities
  for (uint32_t k = kend + 1; k < min(nseg, 2u); ++k) {
    mbar_wait(S.bar + 1 + (k & 1), ph[1 + (k & 1)]);
    ph[1 + (k & 1)] ^= 1u;
  }
  if (t == 0) {
    uint32_t tw = s_cut[0], ti = s_cut[1];
    if (s_cut[2] == NONE) {  // fewer eligible entries than need: all of them
      tw = tsum & 0xFFFFu;
      ti = tsum >> 16;
    }
    write_range(a, q, tw, ti);
    victims += tw + ti;
    scanned += s_cut[2] == NONE ? span : min(span, 32 * (s_cut[2] + 1));
  }
}

// Copy chunks [c0, c1) of the chunk map, one warp (k_copy_fast's body over a
// contiguous range): four descriptors, then their walk loads, in flight together.
__device__ __forceinline__ void copy_range(const PredArgs &a, uint64_t c0, uint64_t c1,
                                           unsigned long long &emitted) {
  constexpr uint32_t UN = 4;
  const uint32_t lane = threadIdx.x & 31;
  uint2 *out = reinterpret_cast<uint2 *>(a.pairs);
  for (uint64_t c = c0; c < c1; c += UN) {
    uint4 m[UN];
#pragma unroll
    for (uint32_t u = 0; u < UN; ++u) m[u] = c + u < c1 ? __ldcg(a.chunk_map + c + u) : make_uint4(0, 0, 0, 0);
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
}

constexpr uint32_t CPW = 8;  // k_window_fast: copy chunks per claim of a copy warp

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

// The selection of one fast query over a log with stale entries (the selection group; see
// above): marks, pass 1 per-segment counts, segment prefix, pass 2 emit.
__device__ __forceinline__ void sel_stale(const PredArgs &a, uint32_t qi, uint32_t head, uint32_t tail,
                                        uint32_t stale, uint32_t *kern, uint32_t *roff, uint32_t *posmap,
                                        uint32_t *seg_cnt, uint32_t *seg_pre, uint32_t &s_tw, uint32_t &s_ti) {
  constexpr uint32_t NW = SG_NT / 32;
  const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const Geo &g = a.g;
  const SelectOut &so = a.so;
  const uint32_t nk = __ldg(a.qnk + qi);
  for (uint32_t d = tid; d <= nk; d += SG_NT) {
    roff[d] = __ldg(a.qroff + (uint64_t)qi * (g.N + 2) + d);
    if (d < nk) kern[d] = __ldg(a.qkern + (uint64_t)qi * (g.N + 1) + d);
  }
  for (uint32_t w = tid; w < POS_WORDS; w += SG_NT) posmap[w] = 0;
  if (tid == 0) {
    s_tw = 0;
    s_ti = 0;
  }
  const uint32_t need = __ldg(a.qneed + qi);
  const unsigned long long bwb = __ldg(a.qvb + 2 * qi), binv = __ldg(a.qvb + 2 * qi + 1);
  const bool ok = bwb + need <= so.cap && binv + need <= so.cap;
  gsync();
  const uint32_t R = nk ? roff[nk] : 0;
  uint32_t nseg = 0;
  if (need) {
    // 1. the window's resident blocks: their log positions into the bitmap
    {
      constexpr uint32_t MU = 4;  // loads in flight per thread
      uint32_t lo = 0;
      for (uint32_t x0 = tid; x0 < R; x0 += SG_NT * MU) {
        uint32_t r[MU];
#pragma unroll
        for (uint32_t u = 0; u < MU; ++u) {
          const uint32_t x = x0 + u * SG_NT;
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
    gsync();
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
    gsync();
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
    gsync();
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
    gsync();
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
}


// a7 + a8 of every fast query in one persistent, warp-specialised kernel.
// Warps [0, SG_NT / 32) of each CTA form the selection group: it claims
// queries (k_chain's class order, biggest selection first; sel_staged on a
// clean log, sel_stale on a log with stale entries) until the selection queue
// is empty, then joins the copy.  The other warps claim copy items (CPW
// chunks of k_chain's chunk map each) from the start, so that the pair stream
// keeps HBM busy while the selection waits on its staged loads.  Queues: the
// DevState counters sel_queue / copy_queue (k_pred_epilogue clears them).
__global__ void __launch_bounds__(WSEL_NT, 3) k_window_fast(PredArgs a) {
  extern __shared__ uint4 stage4[];  // SR_SMEM_WORDS: the staged selection's buffers
  __shared__ uint32_t posmap[POS_WORDS], roff[MAXN + 2], kern[MAXN + 1], ws[SG_NT / 32], s_cut[3], s_item;
  __shared__ uint32_t seg_cnt[FSEG_MAX], seg_pre[FSEG_MAX], s_tw, s_ti;
  __shared__ __align__(8) unsigned long long bar[3];
  const uint32_t tid = threadIdx.x, lane = tid & 31;
  StageSm S;
  S.ibits = reinterpret_cast<uint32_t *>(stage4);
  S.wpre = S.ibits + POS_WORDS;
  S.lbuf = S.wpre + POS_WORDS;
  S.bar = bar;
  if (tid == 0) {
    for (int i = 0; i < 3; ++i) mbar_init(&bar[i]);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  uint32_t ph[3] = {0, 0, 0};  // the barriers' phase parities (every selection-group thread in step)
#ifdef EXP_TRACE
  if (tid == 0) TR(4 * blockIdx.x, gtime());
#endif
  const bool sel = __ldcg(&a.st->log_dirty) == 0;  // a clean log: sel_staged; else sel_stale
  SelLog lg;
  lg.head = __ldcg(&a.st->lrm_head);
  lg.tail = __ldcg(&a.st->lrm_tail);
  lg.stale = lg.tail - lg.head - __ldcg(&a.st->n_resident);
  lg.al = (lg.head & 3u) == 0;
  unsigned long long scanned = 0, victims = 0, emitted = 0;
  if (tid < SG_NT) {  // the selection group: a query per item
    uint32_t ccnt[NQCLS], n1 = 0;
#pragma unroll
    for (int c = 0; c < NQCLS; ++c) {
      ccnt[c] = __ldcg(&a.st->q_cls[c]);
      n1 += ccnt[c];
    }
    for (;;) {
      if (tid == 0) s_item = atomicAdd(&a.st->sel_queue, 1u);
      gsync();
      const uint32_t it = s_item;
      if (it >= n1) break;
      SelRec r;
      {  // the item's record: class-order position -> (class, rank) as in qperm
        uint32_t cq = NQCLS, rq = it;
#pragma unroll
        for (int c = 0; c < NQCLS; ++c)
          if (cq == NQCLS) {
            if (rq < ccnt[c]) cq = c;
            else rq -= ccnt[c];
          }
        const uint4 *p = a.selrec + 3 * ((uint64_t)cq * a.nq + rq);
        r.x = __ldcg(p);
        r.y = __ldcg(p + 1);
        r.z = __ldcg(p + 2);
      }
#ifdef EXP_TRACE
      if (tid == 0) TR(4 * 4096 + 8 * it, gtime());
#endif
      if (sel)
        sel_staged(a, lg, r, S, posmap, roff, kern, ws, s_cut, ph, scanned, victims, it);
      else
        sel_stale(a, r.x.x, lg.head, lg.tail, lg.stale, kern, roff, posmap, seg_cnt, seg_pre, s_tw, s_ti);
#ifdef EXP_TRACE
      if (tid == 0) TR(4 * 4096 + 8 * it + 1, gtime());
#endif
      gsync();  // the next item reuses the shared state
    }
#ifdef EXP_TRACE
    if (tid == 0) TR(4 * blockIdx.x + 1, gtime());
#endif
  }
  {  // the copy warps; the selection group joins them once its queue is empty
    const unsigned long long G = min((unsigned long long)a.chunk_cap, __ldcg(&a.st->pool_chunks));
    for (;;) {
      unsigned long long c0 = 0;
      if (lane == 0) c0 = atomicAdd(&a.st->copy_queue, (unsigned long long)CPW);
      c0 = __shfl_sync(0xffffffffu, c0, 0);
      if (c0 >= G) break;
      copy_range(a, c0, min((unsigned long long)G, c0 + CPW), emitted);
    }
#ifdef EXP_TRACE
    if (tid == SG_NT) TR(4 * blockIdx.x + 2, gtime());  // (a copy warp's end)
#endif
  }
#ifdef EXP_TRACE
  if (lane == 0) atomicMax(&g_tr[4 * blockIdx.x + 3], gtime());
#endif
  emitted = __reduce_add_sync(0xffffffffu, (unsigned)emitted) / 32;
  if (lane == 0 && emitted) {
    ctr_add(a.st, DUM_CTR_EMITTED, emitted);
    ctr_add(a.st, DUM_CTR_GATHERED, emitted);
    ctr_add(a.st, DUM_CTR_FAST_EMITTED, emitted);
  }
  if (tid == 0 && (scanned | victims)) {
    ctr_add(a.st, DUM_CTR_FAST_SCANNED, scanned);
    ctr_add(a.st, DUM_CTR_FAST_VICTIMS, victims);
  }
}

static uint32_t index_grid(const dum_engine *e) {
  return std::max<uint32_t>(1, std::min<uint32_t>(e->g.Emax, 148 * 4));
}

// Build end: the walk index of the walks just rebuilt (k_walk / k_walk_slow).
cudaError_t launch_walk_index(dum_engine *e, cudaStream_t main) {
  if (!e->fast_windows) return cudaSuccess;  // every window takes the exact kernel: no conflicts needed
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
  if (!e->fast_windows) return cudaSuccess;
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
    // the attribute is per device and function: every engine sets it on its own device
    cudaFuncSetAttribute(k_window_fast, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(SR_SMEM_WORDS * 4));
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&ns, k_window_fast, WSEL_NT, SR_SMEM_WORDS * 4);
    e->copy_grid = (uint32_t)std::max(1, nc * sms);
    e->sel_grid = (uint32_t)std::max(1, ns * sms);
  }
  if (select) {  // the pairs and the selection of the fast windows: one persistent kernel
    TimerScope t(e, DUM_T_SELECT_FAST, s);
    k_window_fast<<<e->sel_grid, WSEL_NT, SR_SMEM_WORDS * 4, s>>>(a);
  } else {  // the pairs only: the flat copy over k_chain's chunk map
    TimerScope t(e, DUM_T_PREDICT, s);
    k_copy_fast<<<e->copy_grid, COPY_NT, 0, s>>>(a);
  }
  e->kernel_launches += 1;
  return cudaGetLastError();
}

}  // namespace dum

#ifdef EXP_TRACE
extern "C" int dum_exp_trace(void *dst, unsigned long long bytes, int clear) {
  if (clear) return (int)cudaMemset(g_tr_ptr(), 0, sizeof(g_tr));
  return (int)cudaMemcpyFromSymbol(dst, g_tr, bytes < sizeof(g_tr) ? bytes : sizeof(g_tr));
}
#endif
