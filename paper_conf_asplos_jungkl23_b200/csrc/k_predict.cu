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
#include "corr.cuh"
#include "device_util.cuh"
#include "kernels.cuh"
#include "select_tail.cuh"
#include "walk_seq.cuh"

namespace dum {

constexpr int PRED_NT = 512;
constexpr int NWARP = PRED_NT / 32;
constexpr uint32_t MAXN = 128;   // degree_n limit
constexpr uint32_t DCAP = 2048;  // shared hash of duplicated blocks (block -> min window position)

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
  const uint32_t E = *(volatile uint32_t *)&st->E;
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

struct PredArgs {
  Geo g;
  const dum_query *q;
  uint32_t nq;
  const CorrSlot *corr;
  uint32_t corr_cap;
  const uint32_t *jump;  // [levels][corr_cap]
  const uint32_t *walk, *walk_len;
  const uint32_t *anchor_pool;
  const uint64_t *anchor_range;
  uint32_t *pairs;
  uint64_t cap;
  uint64_t *range;
  uint32_t *kern_off, *chain;
  DevState *st;
  uint32_t nwords;  // bitmap words
  // per-query scratch written by k_chain
  uint32_t *qkern;  // [nq][N+1]
  uint32_t *qloff;  // [nq][N+2]
  uint32_t *qnk;    // [nq]
  unsigned long long *qbase;  // [nq]
  uint32_t *big_pool;         // scratch for the exact slow path
  uint64_t big_entries;
  SelectOut so;     // fused a8 outputs (SELECT only)
};

constexpr int CHAIN_WARPS = 8;

__global__ void __launch_bounds__(CHAIN_WARPS * 32) k_chain(PredArgs a) {
  __shared__ uint32_t skern[CHAIN_WARPS][MAXN + 1];
  __shared__ uint32_t s_u[CHAIN_WARPS];
  __shared__ unsigned long long s_base;
  const uint32_t lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const uint32_t qi = blockIdx.x * CHAIN_WARPS + w;
  const uint32_t below = (1u << lane) - 1;
  const Geo &g = a.g;
  uint32_t U = 0;
  if (qi < a.nq) {
    const dum_query Q = a.q[qi];
    const bool anchored = Q.anchor != NONE;
    const uint32_t E = *(volatile uint32_t *)&a.st->E;
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
    // window layout: walk lengths; a kernel met earlier in the chain with the
    // same (unanchored) walk adds nothing (exact; keeps the reservation tight)
    uint32_t *gkern = a.qkern + (uint64_t)qi * (g.N + 1);
    uint32_t *loff = a.qloff + (uint64_t)qi * (g.N + 2);
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
      uint32_t incl = len;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= (uint32_t)o) incl += y;
      }
      if (v) {
        gkern[d] = e;
        loff[d + 1] = U + incl;
      }
      U += __shfl_sync(0xffffffffu, incl, 31);
    }
    if (lane == 0) {
      loff[0] = 0;
      a.qnk[qi] = nk;
    }
  }
  // CTA-aggregated output reservation
  if (lane == 0) s_u[w] = U;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long tot = 0;
    for (int i = 0; i < CHAIN_WARPS; ++i) tot += s_u[i];
    s_base = tot ? atomicAdd(&a.st->pool_pairs, tot) : 0ull;
  }
  __syncthreads();
  if (qi < a.nq && lane == 0) {
    unsigned long long base = s_base;
    for (uint32_t i = 0; i < w; ++i) base += s_u[i];
    a.qbase[qi] = base;
    if (base + U > a.cap) set_err(a.st, ERR_ECAPACITY, base + U);
  }
}

template <bool SELECT>
__global__ void __launch_bounds__(PRED_NT, 3) k_predict(PredArgs a) {
  extern __shared__ uint32_t bitmap[];  // [nwords] window set | dk[DCAP] | dv[DCAP]
  __shared__ uint32_t kern[MAXN + 1], loff[MAXN + 2], kcnt[MAXN + 1];
  __shared__ uint32_t ws[NWARP], wtot[NWARP];
  __shared__ uint32_t s_ndup, s_nonres, s_flag, s_ovf;
  __shared__ unsigned long long s_hoff;
  const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const uint32_t qi = blockIdx.x;
  const Geo &g = a.g;
  const uint32_t anchor = a.q[qi].anchor;
  const bool anchored = anchor != NONE;
  const uint32_t nk = a.qnk[qi];
  const unsigned long long base = a.qbase[qi];
  uint32_t *dk = bitmap + ((a.nwords + 3) & ~3u), *dv = dk + DCAP;
  {
    uint4 *b4 = reinterpret_cast<uint4 *>(bitmap);
    for (uint32_t w = tid; w < a.nwords / 4; w += PRED_NT) b4[w] = make_uint4(0, 0, 0, 0);
    for (uint32_t w = (a.nwords & ~3u) + tid; w < a.nwords; w += PRED_NT) bitmap[w] = 0;
    uint4 *d4 = reinterpret_cast<uint4 *>(dk);
    for (uint32_t w = tid; w < 2 * DCAP / 4; w += PRED_NT) d4[w] = make_uint4(NONE, NONE, NONE, NONE);
  }
  for (uint32_t d = tid; d <= nk; d += PRED_NT) {
    loff[d] = a.qloff[(uint64_t)qi * (g.N + 2) + d];
    if (d < nk) kern[d] = a.qkern[(uint64_t)qi * (g.N + 1) + d];
  }
  if (tid == 0) {
    s_ndup = 0;
    s_nonres = 0;
    s_ovf = 0;
  }
  __syncthreads();
  const uint32_t U = nk ? loff[nk] : 0;
  const bool ok = base + U <= a.cap;
  if (tid == 0 && anchored && anchor < g.W) {
    bitmap[anchor >> 5] |= 1u << (anchor & 31);
    hmap_insert_min(dk, dv, DCAP, anchor, 0);  // position 0: never kept
  }
  __syncthreads();
  const uint32_t *apool = a.anchor_pool + (anchored ? a.anchor_range[2 * qi] : 0);
  auto list_of = [&](uint32_t d) -> const uint32_t * {
    return (d == 0 && anchored) ? apool : a.walk + (uint64_t)kern[d] * g.walk_cap;
  };
  // ---------------- fast path: one pass ----------------
  // warp w owns the contiguous segment [t0, t1), walked kernel by kernel
  // (no per-element kernel search), 4 loads in flight per lane
  const uint32_t seg = ((U + NWARP - 1) / NWARP + 127) & ~127u;
  const uint32_t t0 = min(U, wid * seg), t1 = min(U, t0 + seg);
  uint32_t nonres = 0, ndup = 0;
  if (t0 < t1) {
    uint32_t d = 0;
    while (d + 1 < nk && loff[d + 1] <= t0) ++d;
    for (; d < nk && loff[d] < t1; ++d) {
      const uint32_t k0 = max(t0, loff[d]), k1 = min(t1, loff[d + 1]);
      if (k0 >= k1) continue;
      const uint32_t *lst = list_of(d) - loff[d];  // indexed by window position
      const uint32_t kd = kern[d];
      for (uint32_t c = k0; c < k1; c += 128) {
        uint32_t b[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const uint32_t t = c + 32 * k + lane;
          b[k] = t < k1 ? __ldg(lst + t) : NONE;
        }
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const uint32_t t = c + 32 * k + lane;
          const bool valid = t < k1;
          if (c + 32 * k >= k1) break;  // warp-uniform
          if (warp_test_and_set(bitmap, b[k], valid)) {
            ++ndup;
            if (!hmap_insert_min(dk, dv, DCAP, b[k], t + 1)) s_ovf = 1;
          }
          if (valid) {
            if (ok) reinterpret_cast<uint2 *>(a.pairs)[base + t] = make_uint2(b[k], kd);
            if (SELECT) nonres += !((__ldg(&a.so.res_bits[b[k] >> 5]) >> (b[k] & 31)) & 1u);
          }
        }
      }
    }
  }
  if (ndup) atomicAdd(&s_ndup, ndup);
  if (SELECT) {
#pragma unroll
    for (int o = 16; o; o >>= 1) nonres += __shfl_xor_sync(0xffffffffu, nonres, o);
    if (lane == 0 && nonres) atomicAdd(&s_nonres, nonres);
  }
  __syncthreads();
  uint32_t run = U;
  const bool dedup = s_ndup != 0;
  if (dedup) {
    // ---------------- exact slow path (some block occurs twice) ----------------
    // keep(t) = t is the minimum window position of its block, the anchor
    // pre-seeded at position 0 (D17).  Normally only the duplicated blocks
    // (found in the fast pass) sit in the shared hash and every occurrence of
    // them lowers the min position; if that hash overflowed, all elements go
    // into a global scratch hash instead.
    const bool ovf = s_ovf != 0;
    uint32_t hcap = DCAP;
    uint32_t *hk = dk, *hv = dv;
    if (tid == 0) {
      s_nonres = 0;
      s_flag = 1;
      if (ovf) {
        const uint32_t hc = pow2ceil(2 * (U + 1));
        const unsigned long long o = atomicAdd(&a.st->pool_big, 2ull * hc);
        s_flag = o + 2ull * hc <= a.big_entries * 2;
        s_hoff = o;
        if (!s_flag) set_err(a.st, ERR_ECAPACITY, o + 2ull * hc);
      }
    }
    for (uint32_t d = tid; d <= nk; d += PRED_NT) kcnt[d] = 0;
    __syncthreads();
    if (ovf) {
      hcap = pow2ceil(2 * (U + 1));
      hk = a.big_pool + s_hoff;
      hv = hk + hcap;
    }
    if (s_flag) {
      if (ovf) {
        for (uint32_t p = tid; p < hcap; p += PRED_NT) {
          hk[p] = NONE;
          hv[p] = NONE;
        }
        __syncthreads();
        if (tid == 0 && anchored) hmap_insert_min(hk, hv, hcap, anchor, 0);
      }
      for (uint32_t d = 0; d < nk; ++d) {
        const uint32_t *lst = list_of(d);
        for (uint32_t i = tid; i < loff[d + 1] - loff[d]; i += PRED_NT) {
          const uint32_t bb = __ldg(lst + i), pos = loff[d] + i + 1;
          if (ovf) {
            hmap_insert_min(hk, hv, hcap, bb, pos);
          } else {
            // lower the min position of duplicated blocks only
            for (uint32_t pp = 0, sl = hslot(bb, hcap); pp < hcap; ++pp, sl = (sl + 1) & (hcap - 1)) {
              const uint32_t kk = hk[sl];
              if (kk == NONE) break;
              if (kk == bb) {
                atomicMin(&hv[sl], pos);
                break;
              }
            }
          }
        }
      }
      __syncthreads();
      // per-warp keep counts over the warp segments, then ordered writes
      for (int pass = 0; pass < 2; ++pass) {
        uint32_t pos = pass ? wtot[wid] : 0, nr = 0;
        if (t0 < t1) {
          uint32_t d = 0;
          while (d + 1 < nk && loff[d + 1] <= t0) ++d;
          for (; d < nk && loff[d] < t1; ++d) {
            const uint32_t k0 = max(t0, loff[d]), k1 = min(t1, loff[d + 1]);
            if (k0 >= k1) continue;
            const uint32_t *lst = list_of(d) - loff[d];
            for (uint32_t c = k0; c < k1; c += 32) {
              const uint32_t t = c + lane;
              uint32_t bb = NONE;
              bool keep = false;
              if (t < k1) {
                bb = __ldg(lst + t);
                const uint32_t mp = hmap_get(hk, hv, hcap, bb);
                keep = ovf ? mp == t + 1 : (mp == NONE || mp == t + 1);
              }
              const uint32_t mask = __ballot_sync(0xffffffffu, keep);
              if (pass && keep) {
                if (ok) reinterpret_cast<uint2 *>(a.pairs)[base + pos + __popc(mask & ((1u << lane) - 1))] =
                    make_uint2(bb, kern[d]);
                if (SELECT) nr += !((__ldg(&a.so.res_bits[bb >> 5]) >> (bb & 31)) & 1u);
              }
              if (pass && lane == 0) atomicAdd(&kcnt[d], __popc(mask));
              pos += __popc(mask);
            }
          }
        }
        if (!pass) {
          if (lane == 0) wtot[wid] = pos;
          __syncthreads();
          if (tid == 0) {
            uint32_t acc = 0;
            for (int w = 0; w < NWARP; ++w) {
              const uint32_t v = wtot[w];
              wtot[w] = acc;
              acc += v;
            }
            ws[0] = acc;
          }
          __syncthreads();
        } else if (SELECT) {
#pragma unroll
          for (int o = 16; o; o >>= 1) nr += __shfl_xor_sync(0xffffffffu, nr, o);
          if (lane == 0 && nr) atomicAdd(&s_nonres, nr);
        }
      }
      __syncthreads();
      run = ws[0];
    } else {
      run = 0;
    }
  }
  if (tid == 0) {
    a.range[2 * qi] = base;
    a.range[2 * qi + 1] = base + (ok ? run : 0);
    ctr_add(a.st, DUM_CTR_QUERIES, 1);
    ctr_add(a.st, DUM_CTR_CHAIN, nk);
    ctr_add(a.st, DUM_CTR_GATHERED, U);
    ctr_add(a.st, DUM_CTR_EMITTED, run);
  }
  if (a.kern_off) {
    uint32_t *ko = a.kern_off + (uint64_t)qi * (g.N + 2);
    for (uint32_t d = tid; d <= g.N + 1; d += PRED_NT) {
      uint32_t v;
      if (!dedup) {
        v = d <= nk ? loff[d] : U;
      } else {
        v = 0;
        for (uint32_t x = 0; x < d && x < nk; ++x) v += kcnt[x];
      }
      ko[d] = v;
    }
  }
  if (a.chain) {
    uint32_t *ch = a.chain + (uint64_t)qi * (g.N + 1);
    for (uint32_t d = tid; d <= g.N; d += PRED_NT) ch[d] = d < nk ? kern[d] : NONE;
  }
  if (SELECT) select_tail<PRED_NT>(a.so, qi, s_nonres, bitmap, g.W, a.st, ws);
}

__global__ void k_copy_counter(const unsigned long long *src, uint64_t *dst) { *dst = *src; }
__global__ void k_copy_counters2(const unsigned long long *a, const unsigned long long *b, uint64_t *dst) {
  *dst = *a > *b ? *a : *b;
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
  cudaMemsetAsync(&e->d_state->pool_pairs, 0, 2 * sizeof(unsigned long long) * 2, s);  // pairs, wb, inv, anchor
  cudaMemsetAsync(&e->d_state->pool_big, 0, sizeof(unsigned long long), s);
  WalkScratch ws{e->d_walk_seen, e->d_walk_chain, e->d_walk_tmp, e->walk_hash_cap,
                 e->g.walk_cap + e->g.R * e->g.A + 4};
  {
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
  a.qnk = e->d_qnk;
  a.qbase = e->d_qbase;
  a.big_pool = e->d_big_pool;
  a.big_entries = e->big_pool_entries;
  if (sel) {
    a.so = *sel;
  } else {
    a.so.res_bits = e->d_res_bits;
  }
  {
    TimerScope t(e, DUM_T_CHAIN, s);
    k_chain<<<(nq + CHAIN_WARPS - 1) / CHAIN_WARPS, CHAIN_WARPS * 32, 0, s>>>(a);
  }
  const size_t smem = (size_t)((a.nwords + 3) & ~3u) * 4 + 2 * DCAP * 4;
  if (sel) {
    cudaFuncSetAttribute(k_predict<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    TimerScope t(e, DUM_T_PREDICT, s);
    k_predict<true><<<nq, PRED_NT, smem, s>>>(a);
  } else {
    cudaFuncSetAttribute(k_predict<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    TimerScope t(e, DUM_T_PREDICT, s);
    k_predict<false><<<nq, PRED_NT, smem, s>>>(a);
  }
  e->kernel_launches += 3;
  if (needed) {
    k_copy_counter<<<1, 1, 0, s>>>(&e->d_state->pool_pairs, needed);
    e->kernel_launches += 1;
  }
  if (sel && sel_needed) {
    k_copy_counters2<<<1, 1, 0, s>>>(&e->d_state->pool_wb, &e->d_state->pool_inv, sel_needed);
    e->kernel_launches += 1;
  }
  return cudaGetLastError();
}

}  // namespace dum
