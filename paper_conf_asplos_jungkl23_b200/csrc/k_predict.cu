// a6 + a7 (+ fused a8): prefetch-window prediction.
//
//  k_make_queries  transition queries from an exec-ID sequence.
//  k_anchor_walk   WALK(e, anchor) for fault-anchored queries (PAPER.md L156:
//                  "calculates the UM block addresses for prefetching with the
//                  faulted block address"; D14) with the sequential walker.
//  k_chain         one warp per query: chain up to n next-kernel predictions
//                  through the execution ID correlation table (PAPER.md,
//                  L220; D15, D16); lane d reaches the record of step d with
//                  popcount(d) loads from the jump tables (k_jump.cu), so the
//                  chain costs O(log n) dependent loads instead of n; window
//                  layout (per-kernel offsets) and the query's output
//                  reservation.
//  k_predict       one CTA per query: gather the walk lists of the window's
//                  kernels and keep the first occurrence of every block (D17),
//                  emitting (block, exec ID) prefetch commands.
//                  Fast path: one pass writes every element at its concatenated
//                  position while a warp-aggregated atomicOr into a shared-memory
//                  bitmap over the block-id space detects whether any block
//                  occurs twice; only then (never on the measured traces) the
//                  exact order-free dedupe (min-position hash) and an ordered
//                  re-compaction overwrite the output.
//                  SELECT: the fused pre-eviction selection of a8 reuses the
//                  window bitmap (select_tail.cuh).
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "corr.cuh"
#include "device_util.cuh"
#include "kernels.cuh"
#include "predict.cuh"
#include "select_tail.cuh"
#include "walk_seq.cuh"

namespace dum {

constexpr int PRED_NT = 512;
constexpr int NWARP = PRED_NT / 32;
constexpr uint32_t DLCAP = 512;   // duplicated blocks recorded by pass 1 (more: hash every element)
constexpr uint32_t DHCAP = 2048;  // shared hash of the duplicated blocks (block -> min position + 1)
static_assert(2 * DHCAP >= SEL_CHUNK, "the dup hash region doubles as the selection stage");

__global__ void k_make_queries(const uint32_t *__restrict__ seq, uint32_t n_seq, uint32_t first, uint32_t degree,
                               dum_query *__restrict__ out) {
  const uint32_t i = first + blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n_seq) return;
  dum_query q;
  q.exec = seq[i];
  q.hist[0] = i >= 3 ? seq[i - 3] : NONE;
  q.hist[1] = i >= 2 ? seq[i - 2] : NONE;
  q.hist[2] = i >= 1 ? seq[i - 1] : NONE;
  q.anchor = NONE;
  q.n = degree;
  out[i - first] = q;
}

__global__ void k_anchor_walk(Geo g, const dum_query *__restrict__ q, uint32_t nq, const uint32_t *tbl,
                              const uint32_t *start_end, uint32_t *slot_out, uint32_t *pool, uint64_t pool_cap,
                              uint64_t *range, WalkScratch ws, DevState *st) {
  const uint32_t E = __ldcg(&st->E);
  uint32_t *out = slot_out + (uint64_t)blockIdx.x * g.walk_cap;
  const uint32_t lane = threadIdx.x & 31;
  for (uint32_t q0 = blockIdx.x * 32; q0 < nq; q0 += gridDim.x * 32) {
   // lanes test 32 queries at once; anchored ones are walked one after another
   const bool anch = q0 + lane < nq && q[q0 + lane].anchor != NONE;
   if (!anch && q0 + lane < nq) {
     range[2 * (q0 + lane)] = 0;
     range[2 * (q0 + lane) + 1] = 0;
   }
   uint32_t todo = __ballot_sync(0xffffffffu, anch);
   while (todo) {
    const uint32_t qi = q0 + __ffs(todo) - 1;
    todo &= todo - 1;
    const dum_query Q = q[qi];
    uint32_t n = 0;
    if (Q.anchor != NONE && Q.exec < E) {
      const uint32_t *tbl_e = tbl + (uint64_t)Q.exec * g.R * g.stride;
      n = walk_seq(g, tbl_e, start_end[2 * Q.exec], start_end[2 * Q.exec + 1], Q.anchor, out, g.walk_cap, ws,
                   blockIdx.x);
      if (n == NONE) {
        if (threadIdx.x == 0) set_err(st, ERR_ECAPACITY, g.walk_cap + 1ull);
        n = 0;
      }
    }
    if (threadIdx.x == 0) ctr_add(st, DUM_CTR_ANCHOR_WALKS, 1);
    unsigned long long base = 0;
    if (threadIdx.x == 0 && n) base = atomicAdd(&st->pool_anchor, (unsigned long long)n);
    base = __shfl_sync(0xffffffffu, base, 0);
    if (base + n > pool_cap) {
      if (threadIdx.x == 0) set_err(st, ERR_ECAPACITY, base + n);
      n = 0;
    }
    for (uint32_t p = threadIdx.x; p < n; p += 32) pool[base + p] = out[p];
    if (threadIdx.x == 0) {
      range[2 * qi] = base;
      range[2 * qi + 1] = n;
    }
    __syncwarp();
   }
  }
}



constexpr int CHAIN_WARPS = 8;

__global__ void __launch_bounds__(CHAIN_WARPS * 32) k_chain(PredArgs a) {
  extern __shared__ uint32_t cbits_dyn[];  // [CHAIN_WARPS][cwords] chain bitsets (when Emax fits)
  const uint32_t cwords = (a.g.Emax + 31) / 32;
  uint32_t *cbits = a.chain_bitset ? cbits_dyn : nullptr;
  if (cbits)
    for (uint32_t x = threadIdx.x; x < CHAIN_WARPS * cwords; x += blockDim.x) cbits[x] = 0;
  __syncthreads();
  __shared__ uint32_t skern[CHAIN_WARPS][MAXN + 1], sgoff[CHAIN_WARPS][MAXN + 2];
  __shared__ uint32_t s_u[CHAIN_WARPS], s_need[CHAIN_WARPS], s_gu[CHAIN_WARPS];
  __shared__ unsigned long long s_base, s_wbase, s_ibase, s_gbase;
  const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint32_t qi = blockIdx.x * CHAIN_WARPS + w;
  const uint32_t below = (1u << lane) - 1;
  const Geo &g = a.g;
  uint32_t U = 0;
  bool slow = false;   // the query goes to the exact kernel (k_predict) instead of k_window
  uint32_t qneed = 0;  // fast query, fused select: victims to reserve in each output list
  uint32_t GUq = 0;    // copy chunks of the window (k_copy_fast)
  uint32_t qres = 0;   // fast query, fused select: resident window blocks (marks of the selection)
  uint32_t qnw = 0;    // fast query, fused select: log-bitmap words k_window_fast scans at most
  if (qi < a.nq) {
    const dum_query Q = a.q[qi];
    const bool anchored = Q.anchor != NONE;
    const uint32_t E = __ldcg(&a.st->E);
    uint32_t *kern = skern[w];
    uint32_t nk = 0;
    if (Q.exec < E) {
      const uint32_t n = Q.n < g.N ? Q.n : g.N;
      uint32_t dummy = 0;
      // record of step 0: (e; h1, h2, h3) (D15); every lane reads the same slots
      const uint32_t r0 = n ? corr_find(a.corr, a.corr_cap, Q.exec, Q.hist[0], Q.hist[1], Q.hist[2], &dummy) : NONE;
      if (lane == 0) kern[0] = Q.exec;
      nk = 1;
      for (uint32_t d0 = 0; d0 < n && r0 != NONE; d0 += 32) {
        // lane d: record of step d = next^d(r0) (D16's shifted history), via
        // the binary digits of d; absent anywhere on the way -> NONE
        const uint32_t d = d0 + lane;
        uint32_t s = d < n ? r0 : NONE;
        for (uint32_t k = 0; s != NONE && (d >> k); ++k)
          if ((d >> k) & 1u) s = __ldcg(a.jump + (uint64_t)k * a.corr_cap + s);
        if (s != NONE) kern[d + 1] = (uint32_t)(__ldcg(&a.corr[s].last) & 0xFFFFFFFFull);
        const uint32_t valid = __ballot_sync(0xffffffffu, s != NONE);  // a prefix of the lanes
        const uint32_t cnt = valid == 0xffffffffu ? 32u : (uint32_t)__ffs(~valid) - 1;
        nk += cnt;
        if (cnt < 32) break;
      }
    }
    __syncwarp();
    // the chain as a bitset over exec IDs (conflict test below), if it fits
    uint32_t *cset = cbits ? cbits + (uint64_t)w * cwords : nullptr;
    if (cset)
      for (uint32_t d = lane; d < nk; d += 32) atomicOr(&cset[kern[d] >> 5], 1u << (kern[d] & 31));
    __syncwarp();
    // window layout: walk lengths; a kernel met earlier in the chain with the
    // same (unanchored) walk adds nothing (exact; keeps the reservation tight)
    uint32_t *gkern = a.qkern + (uint64_t)qi * (g.N + 1);
    uint32_t *loff = a.qloff + (uint64_t)qi * (g.N + 2);
    uint32_t *eoff = a.qeoff + (uint64_t)qi * (g.N + 2);
    uint32_t *goff = a.qgoff + (uint64_t)qi * (g.N + 2);
    uint32_t RU = 0;  // bitmap-run entries of the window (k_predict pass 1)
    uint32_t GU = 0;  // 128-block copy chunks of the window (k_predict copy)
    uint32_t *roff = a.qroff + (uint64_t)qi * (g.N + 2);  // prefix of the lists' resident blocks
    bool conflict = false, unrec = false;
    uint32_t nonres = 0;  // (per lane) window blocks without a frame
    uint32_t nwres = 0;   // (warp-uniform) window blocks with a frame
    for (uint32_t d0 = 0; d0 < nk; d0 += 32) {
      const uint32_t d = d0 + lane;
      const bool v = d < nk, anc0 = d == 0 && anchored;
      const uint32_t e = v ? kern[d] : NONE;
      uint32_t len = v ? (anc0 ? (uint32_t)a.anchor_range[2 * qi + 1] : __ldg(a.walk_len + e)) : 0u;
      const uint32_t key = (v && !anc0) ? e : NONE;
      const uint32_t m = __match_any_sync(0xffffffffu, key);
      if (key != NONE && (m & below)) len = 0;  // an earlier step of this pass
      if (len)
        for (uint32_t d2 = anchored ? 1u : 0u; d2 < d0; ++d2)
          if (kern[d2] == e) {
            len = 0;
            break;
          }
      // fast-path test (k_window.cu): a walk whose recorded conflicts meet
      // the chain, or whose conflicts were too many to record
      uint32_t wres = 0;  // this step's resident window blocks (k_window marks their log positions)
      if (len && !anc0 && a.fast) {
        const uint32_t cn = __ldg(a.conf_n + e);
        if (cn == NONE) {
          conflict = true;
          unrec = true;
        } else {
          // the conflict row, 4 entries per 16 B load (CONF_MAX words, 16 B aligned)
          const uint4 *cr = reinterpret_cast<const uint4 *>(a.conf + (uint64_t)e * CONF_MAX);
          for (uint32_t k0 = 0; k0 < cn; k0 += 4) {
            const uint4 x = __ldg(cr + k0 / 4);
            const uint32_t c4[4] = {x.x, x.y, x.z, x.w};
            for (uint32_t k = 0; k < 4 && k0 + k < cn; ++k) {
              const uint32_t c = c4[k];
              if (cset) {  // the chain's exec-ID bitset (one shared load)
                conflict |= c < a.g.Emax && ((cset[c >> 5] >> (c & 31)) & 1u);
              } else {
                for (uint32_t y = 0; y < nk; ++y) conflict |= kern[y] == c;
              }
            }
          }
        }
        if (a.select) {
          nonres += __ldg(a.wnr + e);
          wres = __ldg(a.wnres + e);
        }
      }
      // an anchored query's own walk has no runs: its blocks enter one by one
      const uint32_t rl = len ? (anc0 ? len : __ldg(a.wrun_len + e)) : 0u;
      const uint32_t gl = (len + CHUNK_B - 1) / CHUNK_B;
      uint32_t incl = len, rincl = rl, gincl = gl, wincl = wres;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
        const uint32_t z = __shfl_up_sync(0xffffffffu, rincl, o);
        const uint32_t u = __shfl_up_sync(0xffffffffu, gincl, o);
        const uint32_t t = __shfl_up_sync(0xffffffffu, wincl, o);
        if (lane >= (uint32_t)o) {
          incl += y;
          rincl += z;
          gincl += u;
          wincl += t;
        }
      }
      if (v) {
        gkern[d] = e;
        loff[d + 1] = U + incl;
        eoff[d + 1] = RU + rincl;
        goff[d + 1] = GU + gincl;
        sgoff[w][d + 1] = GU + gincl;
        if (a.select) roff[d + 1] = nwres + wincl;
      }
      U += __shfl_sync(0xffffffffu, incl, 31);
      RU += __shfl_sync(0xffffffffu, rincl, 31);
      GU += __shfl_sync(0xffffffffu, gincl, 31);
      nwres += __shfl_sync(0xffffffffu, wincl, 31);
    }
    if (lane == 0) {
      loff[0] = 0;
      eoff[0] = 0;
      goff[0] = 0;
      sgoff[w][0] = 0;
      roff[0] = 0;
      a.qnk[qi] = nk;
    }
    slow = anchored || __any_sync(0xffffffffu, conflict) || !a.fast;
    const bool s_unrec = __any_sync(0xffffffffu, unrec);
    if (lane == 0 && slow && (a.fast || anchored)) ctr_add(a.st, anchored ? DUM_CTR_SLOW_ANCHOR : s_unrec ? DUM_CTR_SLOW_UNRECORDED
                                                                           : DUM_CTR_SLOW_CONFLICT, 1);
    nonres = __reduce_add_sync(0xffffffffu, nonres);
    if (a.select && !slow) {
      // need = max(0, window blocks without a frame - free frames) (D18);
      // k_window's selection scans log positions [head, head + need + nwres +
      // stale entries) at most: it must stay inside its position bitmap
      const uint32_t nfree = __ldcg(&a.st->free_count);
      qneed = nonres > nfree ? nonres - nfree : 0;
      const uint32_t span = __ldcg(&a.st->lrm_tail) - __ldcg(&a.st->lrm_head);
      const uint32_t stale = span - __ldcg(&a.st->n_resident);
      if ((uint64_t)qneed + nwres + stale > POS_WORDS * 32ull) {
        slow = true;
        if (lane == 0) ctr_add(a.st, DUM_CTR_SLOW_SPAN, 1);
      } else if (qneed) {
        qnw = (min(span, qneed + nwres + stale) + 31) / 32;
      }
    }
    if (slow) qneed = qnw = 0;  // the exact kernel reserves its own victim ranges
    qres = nwres;
    GUq = slow ? 0u : GU;
    __syncwarp();
    if (cset)
      for (uint32_t d = lane; d < nk; d += 32) cset[kern[d] >> 5] = 0;
  }
  // CTA-aggregated output reservation and window-size class counts (one
  // global atomic per CTA and class instead of one per query)
  __shared__ uint32_t s_cls[2 * NQCLS], s_cbase[2 * NQCLS], s_wcls[CHAIN_WARPS];
  // window-size class (largest first) for the CTA order of k_window / k_predict:
  // the big windows start first instead of forming the tail; fast-path
  // queries (classes 0 .. NQCLS-1) before exact-path ones
  // (fast queries of a fused select: by their selection work -- the marks of
  // the resident window blocks plus the log entries up to the cut, need +
  // resident ones at most -- the selection items' order in k_window_fast)
  const uint32_t key = (a.select && !slow) ? (qneed ? qneed + 2 * qres : 0u) : U;
  const uint32_t cls = (key >= 14336 ? 0u : key >= 10240 ? 1u : key >= 6144 ? 2u : key >= 2048 ? 3u : 4u) +
                       (slow ? (uint32_t)NQCLS : 0u);
  if (threadIdx.x < 2 * NQCLS) s_cls[threadIdx.x] = 0;
  if (lane == 0) {
    s_u[w] = U;
    s_need[w] = qneed;
    s_gu[w] = GUq;  // copy chunks of k_copy_fast
  }
  __syncthreads();
  if (qi < a.nq && lane == 0) s_wcls[w] = atomicAdd(&s_cls[cls], 1u);  // rank within the CTA
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long tot = 0;
    for (int i = 0; i < CHAIN_WARPS; ++i) tot += s_u[i];
    s_base = tot ? atomicAdd(&a.st->pool_pairs, tot) : 0ull;
  } else if (threadIdx.x == 64) {
    unsigned long long tot = 0;
    for (int i = 0; i < CHAIN_WARPS; ++i) tot += s_gu[i];
    s_gbase = tot ? atomicAdd(&a.st->pool_chunks, tot) : 0ull;
  } else if (threadIdx.x == 32 && a.select) {
    // victim ranges of the fast queries: `need` entries in each list (D18-D20)
    unsigned long long tot = 0;
    for (int i = 0; i < CHAIN_WARPS; ++i) tot += s_need[i];
    s_wbase = tot ? atomicAdd(&a.st->pool_wb, tot) : 0ull;
    s_ibase = tot ? atomicAdd(&a.st->pool_inv, tot) : 0ull;
  }
  if (threadIdx.x < 2 * NQCLS)
    s_cbase[threadIdx.x] = s_cls[threadIdx.x] ? atomicAdd(&a.st->q_cls[threadIdx.x], s_cls[threadIdx.x]) : 0u;
  __syncthreads();
  if (qi < a.nq && lane == 0) {
    unsigned long long base = s_base, nb = 0;
    for (uint32_t i = 0; i < w; ++i) {
      base += s_u[i];
      nb += s_need[i];
    }
    a.qbase[qi] = base;
    if (a.select) {
      a.qneed[qi] = qneed;
      a.qvb[2 * qi] = s_wbase + nb;
      a.qvb[2 * qi + 1] = s_ibase + nb;
      if (qneed && (s_wbase + nb + qneed > a.so.cap || s_ibase + nb + qneed > a.so.cap))
        set_err(a.st, ERR_ECAPACITY, (s_wbase > s_ibase ? s_wbase : s_ibase) + nb + qneed);
    }
    if (base + U > a.cap) set_err(a.st, ERR_ECAPACITY, base + U);
    // class lists: query order for k_window_fast / k_predict = class by class
    // (fast classes 0 .. NQCLS-1 largest first, then the exact-path ones)
    a.qperm[(uint64_t)cls * a.nq + s_cbase[cls] + s_wcls[w]] = qi;
  }
  // fast queries: the per-query outputs are known here (k_copy_fast writes the pairs)
  if (qi < a.nq && !slow) {
    __syncwarp();
    const unsigned long long base = a.qbase[qi];
    const uint32_t nk = a.qnk[qi];
    const bool ok = base + U <= a.cap;
    if (lane == 0) {
      a.range[2 * qi] = base;
      a.range[2 * qi + 1] = base + (ok ? U : 0);
      ctr_add(a.st, DUM_CTR_QUERIES, 1);
      ctr_add(a.st, DUM_CTR_Q_FAST, 1);
      ctr_add(a.st, DUM_CTR_CHAIN, nk);
    }
    if (a.kern_off) {
      const uint32_t *lo = a.qloff + (uint64_t)qi * (g.N + 2);
      uint32_t *ko = a.kern_off + (uint64_t)qi * (g.N + 2);
      for (uint32_t d = lane; d <= g.N + 1; d += 32) ko[d] = d <= nk ? __ldcg(lo + d) : U;
    }
    if (a.chain) {
      uint32_t *ch = a.chain + (uint64_t)qi * (g.N + 1);
      for (uint32_t d = lane; d <= g.N; d += 32) ch[d] = d < nk ? skern[w][d] : NONE;
    }
  }
  // k_window_fast's selection record of a fast query (at its class position, like qperm)
  if (qi < a.nq && a.select && !slow && lane == 0) {
    unsigned long long nb = 0;
    for (uint32_t i = 0; i < w; ++i) nb += s_need[i];
    const unsigned long long bwb = s_wbase + nb, binv = s_ibase + nb;
    const uint32_t ok = bwb + qneed <= a.so.cap && binv + qneed <= a.so.cap;
    uint4 *r = a.selrec + 3 * ((uint64_t)cls * a.nq + s_cbase[cls] + s_wcls[w]);
    r[0] = make_uint4(qi, __ldcg(a.qnk + qi), qneed, qnw);
    r[1] = make_uint4(0u, ok, 0u, 0u);
    r[2] = make_uint4((uint32_t)bwb, (uint32_t)(bwb >> 32), (uint32_t)binv, (uint32_t)(binv >> 32));
  }
  // the chunk map of k_copy_fast: chunk j of list d of a fast query -> its
  // source (walk, first entry), destination slot and length; a query whose
  // pairs do not fit the pool gets empty chunks (capacity error raised above)
  if (qi < a.nq && s_gu[w]) {
    __syncwarp();  // the lanes' qloff entries
    unsigned long long gb = s_gbase, base = s_base;
    for (uint32_t i = 0; i < w; ++i) {
      gb += s_gu[i];
      base += s_u[i];
    }
    const uint32_t G = s_gu[w], nk = a.qnk[qi];
    const bool fits = base + s_u[w] <= a.cap;
    const uint32_t *lo = a.qloff + (uint64_t)qi * (g.N + 2);
    for (uint32_t d = lane; d < nk; d += 32) {  // lane d: the chunks of list d
      const uint32_t g0 = sgoff[w][d], g1 = sgoff[w][d + 1], l0 = lo[d], L = lo[d + 1] - l0, e = skern[w][d];
      for (uint32_t x = g0; x < g1; ++x)
        if (gb + x < a.chunk_cap) {
          const uint32_t i0 = (x - g0) * CHUNK_B, n = fits ? min(CHUNK_B, L - i0) : 0u;
          const unsigned long long dst = base + l0 + i0;
          a.chunk_map[gb + x] = make_uint4(e, i0, (uint32_t)dst, (uint32_t)(dst >> 32) | (n << 16));
        }
    }
    if (lane == 0 && gb + G > a.chunk_cap) set_err(a.st, ERR_ECAPACITY, gb + G);
  }
}

// Warp-specialised: warps [0, GRP_W) build the window set from the runs
// (pass 1) and then run the selection (a8) on it; warps [GRP_W, NWARP) stream
// the (block, exec) pairs meanwhile.  Duplicates (rare) are only known after
// pass 1: the duplicate path then rewrites the pairs and redoes the selection
// with the whole CTA.
constexpr int GRP_W = 10;  // window set + selection warps; the other NWARP - GRP_W copy (6, 8 measured: slower)
constexpr int GRP_NT = GRP_W * 32;
constexpr uint32_t OCCAP = 1024;   // duplicate occurrences (list, block) tracked by the duplicate path
constexpr uint32_t DWCAP = 1024;   // duplicate-word hash slots (word -> mask of duplicated blocks)
constexpr uint32_t DBCAP = 1024;   // duplicate-block hash slots (block -> first list + 1)
static_assert(2 * DWCAP + 2 * DBCAP <= 2 * DHCAP, "duplicate hashes live in the dup/stage region");
static_assert(OCCAP >= DLCAP, "s_dup doubles as the occurrence list");

template <bool SELECT>
__global__ void __launch_bounds__(PRED_NT, 2) k_predict(PredArgs a) {
  extern __shared__ uint4 sm4[];  // [nwords rounded up to 4] window set bitmap | dup hashes / select stage
  uint32_t *bitmap = reinterpret_cast<uint32_t *>(sm4);
  uint32_t *dk = bitmap + ((a.nwords + 3) & ~3u);  // [2 * DHCAP]
  __shared__ SelShared ss;
  __shared__ uint32_t kern[MAXN + 1], loff[MAXN + 2], kcnt[MAXN + 1], eoff[MAXN + 2], goff[MAXN + 2];
  __shared__ uint32_t noff[MAXN + 2], dl_d[MAXN + 1], dl_off[MAXN + 2], dl_base[MAXN + 1];
  __shared__ uint32_t ws[NWARP];
  __shared__ uint32_t s_ndup, s_nonres, s_flag, s_nocc, s_dnr, s_nd;
  __shared__ uint32_t s_dup[2 * OCCAP];  // pass 1: duplicated blocks; duplicate path: occurrences (list, block)
  __shared__ unsigned long long s_hoff;
  const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  // persistent over the exact-path queries (class lists NQCLS .. 2 NQCLS-1 of
  // k_chain, largest windows first; the fast path answers the others)
  uint32_t ccnt[NQCLS];
#pragma unroll
  for (int c = 0; c < NQCLS; ++c) ccnt[c] = __ldcg(&a.st->q_cls[NQCLS + c]);
  uint32_t nslow = 0;
#pragma unroll
  for (int c = 0; c < NQCLS; ++c) nslow += ccnt[c];
  for (uint32_t bq = blockIdx.x; bq < nslow; bq += gridDim.x) {
  uint32_t cq = NQCLS, rq = bq;
#pragma unroll
  for (int c = 0; c < NQCLS; ++c)
    if (cq == NQCLS) {
      if (rq < ccnt[c]) cq = c;
      else rq -= ccnt[c];
    }
  const uint32_t qi = a.qperm[(uint64_t)(NQCLS + cq) * a.nq + rq];
  const Geo &g = a.g;
  const uint32_t anchor = a.q[qi].anchor;
  const bool anchored = anchor != NONE;
  const uint32_t nk = a.qnk[qi];
  const unsigned long long base = a.qbase[qi];
  for (uint32_t w = tid; w < (a.nwords + 3) / 4; w += PRED_NT) sm4[w] = make_uint4(0, 0, 0, 0);
  for (uint32_t d = tid; d <= nk; d += PRED_NT) {
    loff[d] = a.qloff[(uint64_t)qi * (g.N + 2) + d];
    eoff[d] = a.qeoff[(uint64_t)qi * (g.N + 2) + d];
    goff[d] = a.qgoff[(uint64_t)qi * (g.N + 2) + d];
    kcnt[d] = 0;
    if (d < nk) kern[d] = a.qkern[(uint64_t)qi * (g.N + 1) + d];
  }
  if (tid == 0) {
    s_ndup = 0;
    s_nonres = 0;
    s_nocc = 0;
    s_dnr = 0;
  }
  __syncthreads();
  const uint32_t U = nk ? loff[nk] : 0;
  const bool ok = base + U <= a.cap;
  const uint32_t *apool = a.anchor_pool + (anchored ? a.anchor_range[2 * qi] : 0);
  auto list_of = [&](uint32_t d) -> const uint32_t * {
    return (d == 0 && anchored) ? apool : a.walk + (uint64_t)kern[d] * g.walk_cap;
  };
  auto search = [&](const uint32_t *off, uint32_t x) -> uint32_t {  // largest d < nk with off[d] <= x
    uint32_t lo = 0, hi = nk;
    while (hi - lo > 1) {
      const uint32_t mid = (lo + hi) >> 1;
      if (off[mid] <= x) lo = mid;
      else hi = mid;
    }
    return lo;
  };
  // run entry x of the window: (word, mask) of list `lo`
  auto run_at = [&](uint32_t x, uint32_t &lo, uint32_t &w, uint32_t &m) {
    lo = search(eoff, x);
    const uint32_t i = x - eoff[lo];
    if (lo == 0 && anchored) {
      const uint32_t b = apool[i];
      w = b >> 5;
      m = 1u << (b & 31);
    } else {
      const uint2 r = __ldg(reinterpret_cast<const uint2 *>(a.wrun) + (uint64_t)kern[lo] * g.walk_cap + i);
      w = r.x;
      m = r.y;
    }
  };
  // Copy of whole lists: flat over the window's 128-block chunks (chunks
  // never straddle lists); warp-uniform chunk lookup, lane-consecutive 4 B
  // loads and 8 B streaming stores (128 B / 256 B per warp instruction), two
  // chunks in flight.  List d goes to pairs[base + oofs[d] ...]; lists with
  // skip[d] != 0 are left out.
  auto copy_lists = [&](uint32_t cw, uint32_t ncw, const uint32_t *oofs, const uint32_t *skip) {
    constexpr uint32_t UN = 2;
    const uint32_t G = nk ? goff[nk] : 0;
    uint2 *out = reinterpret_cast<uint2 *>(a.pairs) + base;
    uint32_t cur = 0;  // list of the chunk (chunks only grow: a running cursor)
    for (uint32_t c0 = cw; c0 < G; c0 += ncw * UN) {
      uint32_t b[UN][4], dd[UN], i0[UN], L[UN];
#pragma unroll
      for (uint32_t u = 0; u < UN; ++u) {
        const uint32_t c = c0 + u * ncw;
        dd[u] = NONE;
        if (c < G) {
          while (goff[cur + 1] <= c) ++cur;
          const uint32_t lo = cur;
          if (skip && skip[lo]) continue;
          dd[u] = lo;
          i0[u] = (c - goff[lo]) * CHUNK_B;
          L[u] = loff[lo + 1] - loff[lo];
          const uint32_t *lst = list_of(lo);
#pragma unroll
          for (uint32_t k = 0; k < 4; ++k) {
            const uint32_t i = i0[u] + 32 * k + lane;
            b[u][k] = i < L[u] ? __ldg(lst + i) : NONE;
          }
        }
      }
#pragma unroll
      for (uint32_t u = 0; u < UN; ++u) {
        if (dd[u] == NONE) continue;
        const uint32_t kd = kern[dd[u]];
        uint2 *o = out + oofs[dd[u]];
#pragma unroll
        for (uint32_t k = 0; k < 4; ++k) {
          const uint32_t i = i0[u] + 32 * k + lane;
          if (i < L[u]) __stcs(o + i, make_uint2(b[u][k], kd));
        }
      }
    }
  };
  auto record_dup = [&](uint32_t w, uint32_t dup) {
    while (dup) {  // rare
      const uint32_t bit = __ffs(dup) - 1;
      dup &= dup - 1;
      const uint32_t k = atomicAdd(&s_ndup, 1u);
      if (k < DLCAP) s_dup[k] = w * 32 + bit;
    }
  };
  // ---------------- pass 1: window set, duplicate test, non-resident count ----------------
  // by threads t = [0, nt): one shared atomicOr per run.  Within one walk the
  // runs are disjoint, so a bit found already set means the block occurs in
  // two lists of the window, or is the anchor (in the window set, never
  // emitted; D14).
  auto pass1 = [&](uint32_t t, uint32_t nt) {
    const uint32_t etot = nk ? eoff[nk] : 0;
    uint32_t nonres = 0;
    if (t == 0 && anchored && anchor < g.W) {
      const uint32_t m = 1u << (anchor & 31);
      record_dup(anchor >> 5, atomicOr(&bitmap[anchor >> 5], m) & m);
    }
    uint32_t lo = 0;  // list of run x (x only grows: a running cursor, no search)
    constexpr int RB = 4;  // runs per thread with their loads in flight together
    for (uint32_t x0 = t; x0 < etot; x0 += nt * RB) {
      uint32_t w[RB], m[RB];
#pragma unroll
      for (int q = 0; q < RB; ++q) {
        const uint32_t x = x0 + q * nt;
        w[q] = NONE;
        m[q] = 0;
        if (x < etot) {
          while (eoff[lo + 1] <= x) ++lo;
          const uint32_t i = x - eoff[lo];
          if (lo == 0 && anchored) {
            const uint32_t b = apool[i];
            w[q] = b >> 5;
            m[q] = 1u << (b & 31);
          } else {
            const uint2 r = __ldg(reinterpret_cast<const uint2 *>(a.wrun) + (uint64_t)kern[lo] * g.walk_cap + i);
            w[q] = r.x;
            m[q] = r.y;
          }
        }
      }
      uint32_t rb[RB];
#pragma unroll
      for (int q = 0; q < RB; ++q) rb[q] = (SELECT && w[q] != NONE) ? __ldg(&a.so.res_bits[w[q]]) : 0u;
#pragma unroll
      for (int q = 0; q < RB; ++q) {
        if (w[q] == NONE) continue;
        record_dup(w[q], atomicOr(&bitmap[w[q]], m[q]) & m[q]);
        if (SELECT) nonres += __popc(m[q] & ~rb[q]);
      }
    }
    if (SELECT) {
#pragma unroll
      for (int o = 16; o; o >>= 1) nonres += __shfl_xor_sync(0xffffffffu, nonres, o);
      if (lane == 0 && nonres) atomicAdd(&s_nonres, nonres);
    }
  };
  if (SELECT) {
    // warps [0, GRP_W): pass 1, then -- without duplicates, the normal case --
    // the selection (a8); warps [GRP_W, NWARP) stream the pairs meanwhile,
    // speculatively: a window with duplicates is rewritten by the duplicate
    // path below (whole CTA), which also redoes the selection
    if (wid < GRP_W) {
      pass1(tid, GRP_NT);
      group_sync<1, GRP_NT>();
      if (s_ndup == 0) {
        if (tid == 0) select_reserve(a.so, s_nonres, a.st, ss);
        group_sync<1, GRP_NT>();
        select_tail<GRP_NT, 1>(a.so, qi, ss, InBlockBitmap{bitmap}, a.st, tid, dk);
      }
    } else if (ok) {
      copy_lists(wid - GRP_W, NWARP - GRP_W, loff, nullptr);
    }
  } else {  // predict only: pass 1 by the whole CTA, then every warp streams (no duplicates)
    pass1(tid, PRED_NT);
    __syncthreads();
    if (s_ndup == 0 && ok) copy_lists(wid, NWARP, loff, nullptr);
  }
  __syncthreads();
  const uint32_t ndup = s_ndup;
  uint32_t run = U;
  if (ndup) {
    // ---------------- duplicate path (D17: first occurrence wins) ----------------
    // The window is the concatenation of the lists; a list holds a block at
    // most once, so an occurrence is kept iff no earlier list holds the block
    // (and it is not the anchor, "list -1").  Per duplicated block the first
    // list is found from the runs (a word hash filters the runs that hold
    // duplicated blocks), every other occurrence is dropped, the lists keep
    // their order and shift left; the few lists that lose blocks are
    // compacted together by the whole CTA, the others are copied again.
    uint32_t *wk = dk, *wm = dk + DWCAP;                      // word -> duplicated-block mask
    uint32_t *bk = dk + 2 * DWCAP, *bv = bk + DBCAP;          // block -> first list + 1 (anchor: 0)
    bool fallback = ndup > DLCAP;
    if (!fallback) {
      for (uint32_t p = tid; p < 2 * DHCAP; p += PRED_NT) dk[p] = NONE;
      __syncthreads();
      for (uint32_t p = tid; p < ndup; p += PRED_NT) {
        const uint32_t b = s_dup[p];
        hmap_insert_min(bk, bv, DBCAP, b, NONE);
        // word -> mask: claim the word's slot, then OR the bit in
        for (uint32_t sl = hslot(b >> 5, DWCAP);; sl = (sl + 1) & (DWCAP - 1)) {
          const uint32_t old = atomicCAS(&wk[sl], NONE, b >> 5);
          if (old == NONE || old == (b >> 5)) break;
        }
      }
      __syncthreads();
      // claimed words: clear the mask, then set the duplicated bits
      for (uint32_t p = tid; p < DWCAP; p += PRED_NT)
        if (wk[p] != NONE) wm[p] = 0;
      __syncthreads();
      for (uint32_t p = tid; p < ndup; p += PRED_NT) {
        const uint32_t b = s_dup[p];
        for (uint32_t sl = hslot(b >> 5, DWCAP);; sl = (sl + 1) & (DWCAP - 1))
          if (wk[sl] == (b >> 5)) {
            atomicOr(&wm[sl], 1u << (b & 31));
            break;
          }
      }
      if (tid == 0 && anchored) hmap_insert_min(bk, bv, DBCAP, anchor, 0);
      __syncthreads();
      // occurrences: runs holding duplicated blocks -> (list, block); first list per block
      const uint32_t etot = nk ? eoff[nk] : 0;
      for (uint32_t x = tid; x < etot; x += PRED_NT) {
        uint32_t lo, w, m;
        run_at(x, lo, w, m);
        uint32_t hit = 0;
        for (uint32_t sl = hslot(w, DWCAP);; sl = (sl + 1) & (DWCAP - 1)) {
          const uint32_t kk = wk[sl];
          if (kk == NONE) break;
          if (kk == w) {
            hit = m & wm[sl];
            break;
          }
        }
        while (hit) {
          const uint32_t bit = __ffs(hit) - 1;
          hit &= hit - 1;
          const uint32_t b = w * 32 + bit;
          hmap_insert_min(bk, bv, DBCAP, b, lo + 1);
          const uint32_t k = atomicAdd(&s_nocc, 1u);
          if (k < OCCAP) {
            s_dup[2 * k] = lo;
            s_dup[2 * k + 1] = b;
          }
        }
      }
      __syncthreads();
      fallback = s_nocc > OCCAP;
    }
    if (!fallback) {
      // dropped occurrences: per-list counts (kcnt) and the non-resident ones
      const uint32_t nocc = s_nocc;
      for (uint32_t k = tid; k < nocc; k += PRED_NT) {
        const uint32_t d = s_dup[2 * k], b = s_dup[2 * k + 1];
        if (hmap_get(bk, bv, DBCAP, b) != d + 1) {
          atomicAdd(&kcnt[d], 1u);
          if (SELECT && !((__ldg(&a.so.res_bits[b >> 5]) >> (b & 31)) & 1u)) atomicAdd(&s_dnr, 1u);
        }
      }
      __syncthreads();
      // output offsets of the shifted lists (warp 0)
      if (wid == 0) {
        uint32_t acc = 0;
        for (uint32_t d0 = 0; d0 < nk; d0 += 32) {
          const uint32_t d = d0 + lane;
          const uint32_t len = d < nk ? loff[d + 1] - loff[d] - kcnt[d] : 0;
          uint32_t incl = len;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= (uint32_t)o) incl += y;
          }
          if (d < nk) noff[d] = acc + incl - len;
          acc += __shfl_sync(0xffffffffu, incl, 31);
        }
        if (lane == 0) noff[nk] = acc;
      }
      __syncthreads();
      run = noff[nk];
      if (ok) {
        // lists that lose blocks: one ordered compaction by the whole CTA over
        // their concatenation (rank r -> list dl_d[r], offsets dl_off), chunks
        // of 4 * PRED_NT elements (thread tid owns 4 consecutive ones), one
        // block scan of the keep counts per chunk; a kept element's slot in
        // its list is (kept before it) - (kept before its list), the latter
        // recorded in dl_base by the thread owning the list's first element
        if (wid == 0) {
          uint32_t acc = 0, nd = 0;
          for (uint32_t d0 = 0; d0 < nk; d0 += 32) {
            const uint32_t d = d0 + lane;
            const bool f = d < nk && kcnt[d];
            const uint32_t len = f ? loff[d + 1] - loff[d] : 0;
            const uint32_t bal = __ballot_sync(0xffffffffu, f);
            uint32_t incl = len;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
              const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
              if (lane >= (uint32_t)o) incl += y;
            }
            if (f) {
              const uint32_t r = nd + __popc(bal & ((1u << lane) - 1u));
              dl_d[r] = d;
              dl_off[r] = acc + incl - len;
            }
            acc += __shfl_sync(0xffffffffu, incl, 31);
            nd += __popc(bal);
          }
          if (lane == 0) {
            dl_off[nd] = acc;
            s_nd = nd;
          }
        }
        __syncthreads();
        const uint32_t T = dl_off[s_nd];
        uint32_t kept = 0, cur = 0;
        for (uint32_t c = 0; c < T; c += 4 * PRED_NT) {
          uint32_t bb[4], lr[4], keep = 0;
#pragma unroll
          for (uint32_t u = 0; u < 4; ++u) {
            const uint32_t t = c + 4 * tid + u;
            bb[u] = NONE;
            lr[u] = cur;
            if (t >= T) continue;
            while (dl_off[cur + 1] <= t) ++cur;
            lr[u] = cur;
            const uint32_t d = dl_d[cur];
            bb[u] = __ldg(list_of(d) + (t - dl_off[cur]));
            const uint32_t f = hmap_get(bk, bv, DBCAP, bb[u]);
            if (f == NONE || f == d + 1) keep |= 1u << u;
          }
          uint32_t tot;
          const uint32_t pre = block_excl_scan(__popc(keep), ws, &tot);
#pragma unroll
          for (uint32_t u = 0; u < 4; ++u)
            if (c + 4 * tid + u < T && c + 4 * tid + u == dl_off[lr[u]])
              dl_base[lr[u]] = kept + pre + __popc(keep & ((1u << u) - 1u));
          __syncthreads();
#pragma unroll
          for (uint32_t u = 0; u < 4; ++u)
            if ((keep >> u) & 1u) {
              const uint32_t d = dl_d[lr[u]];
              const uint32_t k = kept + pre + __popc(keep & ((1u << u) - 1u)) - dl_base[lr[u]];
              __stcs(reinterpret_cast<uint2 *>(a.pairs) + base + noff[d] + k, make_uint2(bb[u], kern[d]));
            }
          kept += tot;
        }
        // the other lists at their shifted offsets
        copy_lists(wid, NWARP, noff, kcnt);
      }
      if (SELECT && tid == 0) s_nonres -= s_dnr;
      if (tid == 0) ctr_add(a.st, DUM_CTR_Q_DUP, 1);
    } else {
      // ---------------- fallback: min-position hash over every element ----------------
      const uint32_t hcap = pow2ceil(2 * (U + 1));
      if (tid == 0) {
        ctr_add(a.st, DUM_CTR_Q_FALLBACK, 1);
        s_nonres = 0;
        const unsigned long long o = atomicAdd(&a.st->pool_big, 2ull * hcap);
        s_flag = o + 2ull * hcap <= a.big_entries * 2;
        s_hoff = o;
        if (!s_flag) set_err(a.st, ERR_ECAPACITY, o + 2ull * hcap);
      }
      for (uint32_t d = tid; d <= nk; d += PRED_NT) kcnt[d] = 0;
      __syncthreads();
      if (s_flag) {
        uint32_t *hk = a.big_pool + s_hoff, *hv = hk + hcap;
        for (uint32_t p = tid; p < hcap; p += PRED_NT) {
          hk[p] = NONE;
          hv[p] = NONE;
        }
        __syncthreads();
        if (tid == 0 && anchored) hmap_insert_min(hk, hv, hcap, anchor, 0);
        for (uint32_t t = tid; t < U; t += PRED_NT) {
          const uint32_t d = search(loff, t);
          hmap_insert_min(hk, hv, hcap, __ldg(list_of(d) + (t - loff[d])), t + 1);
        }
        __syncthreads();
        // ordered compaction: chunks of 4 * PRED_NT positions, thread tid owns
        // 4 consecutive ones; one block scan of the keep counts per chunk
        uint32_t outn = 0, nr = 0;
        for (uint32_t c = 0; c < U; c += 4 * PRED_NT) {
          const uint32_t t0 = c + 4 * tid;
          uint32_t bb[4], dd[4], keep = 0;
#pragma unroll
          for (uint32_t u = 0; u < 4; ++u) {
            const uint32_t t = t0 + u;
            dd[u] = NONE;
            bb[u] = NONE;
            if (t < U) {
              dd[u] = search(loff, t);
              bb[u] = __ldg(list_of(dd[u]) + (t - loff[dd[u]]));
              if (hmap_get(hk, hv, hcap, bb[u]) == t + 1) keep |= 1u << u;
            }
          }
          uint32_t tot;
          const uint32_t pre = block_excl_scan(__popc(keep), ws, &tot);
          uint32_t r = 0;
#pragma unroll
          for (uint32_t u = 0; u < 4; ++u) {
            if (!((keep >> u) & 1u)) continue;
            if (ok) reinterpret_cast<uint2 *>(a.pairs)[base + outn + pre + r] = make_uint2(bb[u], kern[dd[u]]);
            if (SELECT) nr += !((__ldg(&a.so.res_bits[bb[u] >> 5]) >> (bb[u] & 31)) & 1u);
            atomicAdd(&kcnt[dd[u]], 1u);  // kept per list
            ++r;
          }
          outn += tot;
        }
        if (SELECT) {
#pragma unroll
          for (int o = 16; o; o >>= 1) nr += __shfl_xor_sync(0xffffffffu, nr, o);
          if (lane == 0 && nr) atomicAdd(&s_nonres, nr);
        }
        __syncthreads();
        // kept per list -> dropped per list (kern_off below uses the same form)
        for (uint32_t d = tid; d < nk; d += PRED_NT) kcnt[d] = loff[d + 1] - loff[d] - kcnt[d];
        run = outn;
      } else {
        run = 0;
      }
    }
    __syncthreads();
    if (SELECT) {
      if (tid == 0) select_reserve(a.so, s_nonres, a.st, ss);
      __syncthreads();
      select_tail<PRED_NT, 0>(a.so, qi, ss, InBlockBitmap{bitmap}, a.st, tid, dk);
    }
  }
  if (tid == 0) {
    a.range[2 * qi] = base;
    a.range[2 * qi + 1] = base + (ok ? run : 0);
    ctr_add(a.st, DUM_CTR_QUERIES, 1);
    ctr_add(a.st, DUM_CTR_CHAIN, nk);
    ctr_add(a.st, DUM_CTR_GATHERED, U);
    ctr_add(a.st, DUM_CTR_EMITTED, run);
    ctr_add(a.st, DUM_CTR_RUNS, nk ? eoff[nk] : 0);
    if (ndup == 0) ctr_add(a.st, DUM_CTR_Q_NODUP, 1);
  }
  if (a.kern_off) {
    // kern_off[d] = pairs emitted before kernel d (kcnt = occurrences dropped per list)
    uint32_t *ko = a.kern_off + (uint64_t)qi * (g.N + 2);
    for (uint32_t d = tid; d <= g.N + 1; d += PRED_NT) {
      uint32_t v;
      if (ndup == 0) {
        v = d <= nk ? loff[d] : U;
      } else {
        v = 0;
        for (uint32_t x = 0; x < d && x < nk; ++x) v += loff[x + 1] - loff[x] - kcnt[x];
      }
      ko[d] = v;
    }
  }
  if (a.chain) {
    uint32_t *ch = a.chain + (uint64_t)qi * (g.N + 1);
    for (uint32_t d = tid; d <= g.N; d += PRED_NT) ch[d] = d < nk ? kern[d] : NONE;
  }
  if (tid == 0) ctr_add(a.st, DUM_CTR_Q_SLOW, 1);
  __syncthreads();  // the next query reuses the shared state
  }
}

// Predict epilogue: the selection pools' size for the caller, then the call's
// bump pointers and k_chain's class counters are cleared for the next call
// (they start cleared: k_init_state).
__global__ void k_pred_epilogue(DevState *st, uint64_t *needed, uint64_t *sel_needed) {
  const uint32_t t = threadIdx.x;
  if (t == 0) {
    if (needed) *needed = st->pool_pairs;  // every reservation is made: the pool size is the call's `needed`
    if (sel_needed) *sel_needed = st->pool_wb > st->pool_inv ? st->pool_wb : st->pool_inv;
    st->pool_pairs = 0;
    st->pool_chunks = 0;
    st->sel_queue = 0;
    st->copy_queue = 0;
    st->pool_wb = 0;
    st->pool_inv = 0;
    st->pool_anchor = 0;
    st->pool_big = 0;
    st->chain_done = 0;
  }
  if (t < 16) st->q_cls[t] = 0;
}

cudaError_t launch_make_queries(dum_engine *e, const uint32_t *exec_seq, uint32_t n_seq, uint32_t first,
                                uint32_t degree, dum_query *out, cudaStream_t s) {
  if (first >= n_seq) return cudaSuccess;
  const uint32_t n = n_seq - first;
  TimerScope t(e, DUM_T_MAKE_QUERIES, s);
  k_make_queries<<<(n + 255) / 256, 256, 0, s>>>(exec_seq, n_seq, first, degree, out);
  e->kernel_launches += 1;
  return cudaGetLastError();
}

cudaError_t launch_predict(dum_engine *e, const dum_query *q, uint32_t nq, uint32_t *pairs, uint64_t cap,
                           uint64_t *range, uint32_t *kern_off, uint32_t *chain, uint64_t *needed,
                           const SelectOut *sel, uint64_t *sel_needed, cudaStream_t s) {
  if (nq == 0) return cudaSuccess;
  if (nq > e->anchor_range_cap) return cudaErrorInvalidValue;
  WalkScratch ws{e->d_walk_seen, e->d_walk_chain, e->d_walk_tmp, e->walk_hash_cap,
                 e->g.walk_cap + e->g.R * e->g.A + 4};
  if (!e->bhead_n) {  // (dum_step's queries are transition queries: no anchors, no anchored walks)
    TimerScope t(e, DUM_T_ANCHOR_WALK, s);
    k_anchor_walk<<<e->n_walk_slots, 32, 0, s>>>(e->g, q, nq, e->d_tbl, e->d_start_end, e->d_walk_out,
                                                 e->d_anchor_pool, e->anchor_pool_entries, e->d_anchor_range, ws,
                                                 e->d_state);
  }
  PredArgs a;
  a.g = e->g;
  a.q = q;
  a.nq = nq;
  a.corr = e->d_corr;
  a.corr_cap = e->corr_cap;
  a.jump = e->d_jump;
  a.walk = e->d_walk;
  a.walk_len = e->d_walk_len;
  a.wrun = e->d_wrun;
  a.wrun_len = e->d_wrun_len;
  a.anchor_pool = e->d_anchor_pool;
  a.anchor_range = e->d_anchor_range;
  a.pairs = pairs;
  a.cap = cap;
  a.range = range;
  a.kern_off = kern_off;
  a.chain = chain;
  a.st = e->d_state;
  a.nwords = (e->g.W + 31) / 32;
  a.qkern = e->d_qkern;
  a.qloff = e->d_qloff;
  a.qeoff = e->d_qeoff;
  a.qgoff = e->d_qgoff;
  a.qrank = e->d_qrank;
  a.qperm = e->d_qperm;
  a.qnk = e->d_qnk;
  a.qbase = e->d_qbase;
  a.big_pool = e->d_big_pool;
  a.big_entries = e->big_pool_entries;
  if (sel) {
    a.so = *sel;
  } else {
    a.so.res_bits = e->d_res_bits;
  }
  a.needed = needed;
  a.select = sel ? 1u : 0u;
  a.conf = e->d_conf;
  a.conf_n = e->d_conf_n;
  a.wnr = e->d_wnr;
  a.wnres = e->d_wnres;
  a.respos = e->d_respos;
  a.inact_bits = sel ? e->d_log_bits : nullptr;
  a.qroff = e->d_qroff;
  a.qneed = e->d_qneed;
  a.qvb = e->d_qvb;
  a.selrec = e->d_selrec;
  a.fast = e->fast_windows ? 1u : 0u;
  a.lrm_cap = e->lrm_cap;
  {
    // the chunk map holds every copy chunk of the call: <= cap / 128 + nq (N + 1)
    const uint64_t bound = cap / CHUNK_B + (uint64_t)nq * (e->g.N + 1) + 1;
    if (bound > e->chunk_cap && e->capturing) return cudaErrorInvalidValue;  // grown before a capture
    if (bound > e->chunk_cap) {
      cudaError_t ce = cudaStreamSynchronize(s);  // growth only: the old map may be in use
      if (ce == cudaSuccess) ce = cudaFree(e->d_chunk_map);
      e->d_chunk_map = nullptr;
      if (ce == cudaSuccess) ce = cudaMalloc((void **)&e->d_chunk_map, 16 * bound);
      if (ce != cudaSuccess) return ce;
      e->chunk_cap = bound;
    }
  }
  a.chunk_map = e->d_chunk_map;
  a.chunk_cap = e->chunk_cap;
  cudaError_t err;
  if (sel && e->wres_pending) {  // issued beside the ingest by dum_step: join it
    cudaStreamWaitEvent(s, e->ev_wres, 0);
    e->wres_pending = false;
  } else if (sel && (err = launch_walk_res(e, s)) != cudaSuccess) {  // residency facts per walk
    return err;
  }
  if (!e->capturing && e->commit_stale && (err = launch_walk_commit(e, s)) != cudaSuccess) return err;
  if (e->commit_inflight && !e->capturing) {  // the last build's walks (side-stream commit)
    cudaStreamWaitEvent(s, e->ev_commit, 0);
    e->commit_inflight = false;
  }
  if (!e->capturing) {  // (a captured step joins its side streams before it ends)
    if (e->widx_stale) {  // the last build was a replayed step: its walk index is due
      if ((err = launch_walk_index(e, s)) != cudaSuccess) return err;
      e->widx_stale = false;
    }
    if (e->jump_stale) {  // ... and so are its jump tables
      cudaEventRecord(e->ev_fork, s);
      cudaStreamWaitEvent(e->side, e->ev_fork, 0);
      if ((err = launch_jump_tables(e, e->side)) != cudaSuccess) return err;
      cudaEventRecord(e->ev_join, e->side);
      e->jump_stale = false;
    }
  }
  // jump tables of the last build (side stream; in a captured step: forked at
  // its start, beside the ingest)
  cudaStreamWaitEvent(s, e->ev_join, 0);
  cudaStreamWaitEvent(s, e->ev_widx, 0);  // walk index of the last build (third side stream)
  {
    TimerScope t(e, DUM_T_CHAIN, s);
    // chain bitsets in shared memory when max_exec_ids fits (<= 8 KB per warp)
    const uint32_t cwords = (e->g.Emax + 31) / 32;
    a.chain_bitset = cwords <= 2048 ? 1u : 0u;
    const size_t csmem = a.chain_bitset ? (size_t)CHAIN_WARPS * cwords * 4 : 0;
    if ((int)csmem > e->chain_smem) {
      cudaFuncSetAttribute(k_chain, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)csmem);
      e->chain_smem = (int)csmem;
    }
    k_chain<<<(nq + CHAIN_WARPS - 1) / CHAIN_WARPS, CHAIN_WARPS * 32, csmem, s>>>(a);
  }
  if (e->bhead_n) {  // dum_step: the staged batch's build head beside the predict kernels (k_build.cu)
    if ((err = launch_build_head(e, e->bhead_n, s)) != cudaSuccess) return err;
  }
  // exact path (windows that may hold duplicates, anchored queries) first on
  // `s` -- its few CTAs are dispatched before the fast path's persistent grid
  // fills the SMs -- and the fast path beside it on the second side stream
  cudaEventRecord(e->ev_fork2, s);
  cudaStreamWaitEvent(e->side2, e->ev_fork2, 0);
  const size_t smem = (size_t)((a.nwords + 3) & ~3u) * 4 + 2 * DHCAP * 4;
  // fast windows: persistent over the few exact-path queries; else a CTA per query
  const uint32_t pgrid = e->fast_windows ? std::min<uint32_t>(nq, 148) : nq;
  if (sel) {
    // the attribute is per device and function: raised by every engine on its own device
    if ((int)smem > e->select_smem) {
      cudaFuncSetAttribute(k_predict<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      e->select_smem = (int)smem;
    }
    TimerScope t(e, DUM_T_EXACT, s);
    k_predict<true><<<pgrid, PRED_NT, smem, s>>>(a);
  } else {
    if ((int)smem > e->predict_smem) {
      cudaFuncSetAttribute(k_predict<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
      e->predict_smem = (int)smem;
    }
    TimerScope t(e, DUM_T_EXACT, s);
    k_predict<false><<<pgrid, PRED_NT, smem, s>>>(a);
  }
  if (e->fast_windows && (err = launch_window(e, a, sel != nullptr, e->side2)) != cudaSuccess) return err;
  cudaEventRecord(e->ev_join2, e->side2);
  cudaStreamWaitEvent(s, e->ev_join2, 0);
  e->kernel_launches += 2;
  k_pred_epilogue<<<1, 32, 0, s>>>(e->d_state, needed, sel ? sel_needed : nullptr);
  e->kernel_launches += 1;
  return cudaGetLastError();
}

}  // namespace dum
