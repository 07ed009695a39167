// a6 + a7: prefetch-window prediction.
//
//  k_make_queries  transition queries from an exec-ID sequence.
//  k_anchor_walk   WALK(e, anchor) for fault-anchored queries (PAPER.md L156:
//                  "calculates the UM block addresses for prefetching with the
//                  faulted block address"; D14) with the sequential walker.
//  k_predict       one CTA per query: chain up to n next-kernel predictions
//                  through the execution ID correlation table (PAPER.md,
//                  L220; D15, D16), then gather the walk lists of the window's
//                  kernels and keep the first occurrence of every block (D17),
//                  emitting (block, exec ID) prefetch commands.
//                  The window set lives in a shared-memory bitmap over the
//                  block-id space; duplicates inside one gather chunk are
//                  resolved by a chunk-local min-position hash so any chunking
//                  gives the sequential order's result.
#include "device_util.cuh"
#include "kernels.cuh"
#include "walk_seq.cuh"
#include "select_tail.cuh"

namespace dum {

constexpr int PRED_NT = 512;
constexpr uint32_t MAXN = 128;  // degree_n limit
constexpr uint32_t CH_CAP = 2 * PRED_NT;

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

// lookup(e, h1, h2, h3) -> successor or NONE (A9)
__device__ __forceinline__ uint32_t corr_lookup(const CorrSlot *corr, uint32_t cap, uint32_t owner, uint32_t h1,
                                                uint32_t h2, uint32_t h3) {
  const unsigned long long k0 = (unsigned long long)owner | ((unsigned long long)h1 << 32);
  const unsigned long long k1 = (unsigned long long)h2 | ((unsigned long long)h3 << 32);
  uint32_t s = (uint32_t)fmix64(k0 * 0x9E3779B97F4A7C15ull ^ fmix64(k1)) & (cap - 1);
  for (uint32_t p = 0; p < cap; ++p) {
    const uint4 kk = __ldcg(reinterpret_cast<const uint4 *>(corr[s].key));
    if (kk.x == NONE) return NONE;
    if (kk.x == owner && kk.y == h1 && kk.z == h2 && kk.w == h3)
      return (uint32_t)(__ldcg(&corr[s].last) & 0xFFFFFFFFull);
    s = (s + 1) & (cap - 1);
  }
  return NONE;
}

__global__ void k_anchor_walk(Geo g, const dum_query *__restrict__ q, uint32_t nq, const uint32_t *tbl,
                              const uint32_t *start_end, uint32_t *slot_out, uint32_t *pool, uint64_t pool_cap,
                              uint64_t *range, WalkScratch ws, DevState *st) {
  const uint32_t E = *(volatile uint32_t *)&st->E;
  uint32_t *out = slot_out + (uint64_t)blockIdx.x * g.walk_cap;
  for (uint32_t qi = blockIdx.x; qi < nq; qi += gridDim.x) {
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

struct PredArgs {
  Geo g;
  const dum_query *q;
  uint32_t nq;
  const CorrSlot *corr;
  uint32_t corr_cap;
  const uint32_t *walk, *walk_len;
  const uint32_t *anchor_pool;
  const uint64_t *anchor_range;
  uint32_t *pairs;
  uint64_t cap;
  uint64_t *range;
  uint32_t *kern_off, *chain;
  DevState *st;
  uint32_t nwords;  // bitmap words
  // fused select (a8) outputs; unused unless SELECT
  SelectOut so;
};

constexpr uint32_t DCAP = 2048;       // duplicate-block hash (window-wide)
constexpr uint32_t UCAP = 65536;      // keep-bit capacity (window elements)
constexpr int NWARP = PRED_NT / 32;

// Element t of the window's concatenated walk lists; d advances monotonically.
struct WinSrc {
  const uint32_t *walk, *apool;
  const uint32_t *kern, *loff;
  uint32_t nk, walk_cap;
  uint64_t abase;
  bool anchored;
  __device__ __forceinline__ uint32_t get(uint32_t t, uint32_t &d) const {
    while (d + 1 < nk && loff[d + 1] <= t) ++d;
    const uint32_t idx = t - loff[d];
    return (d == 0 && anchored) ? apool[abase + idx] : __ldg(walk + (uint64_t)kern[d] * walk_cap + idx);
  }
};

// One CTA per query.
//  phase 1  warp 0 lane 0 chains the next-kernel predictions (serial corr
//           lookups) and publishes kernel d as soon as it is known; warps 1..15
//           meanwhile insert the published kernels' walk lists into the window
//           bitmap (order-free atomicOr).  An element that finds its bit
//           already set marks its block as duplicated (hash: block -> min
//           position).
//  phase 2  (only if duplicates exist) every element of a duplicated block
//           lowers that block's min position to its own.
//  phase 3  keep(t) = block not duplicated, or t is its min position (the
//           anchor is pre-seeded at position 0 so it is never kept): exactly
//           the first-occurrence rule of D17 regardless of processing order.
//  phase 4  ordered compaction: per-warp contiguous segments, ballots, one
//           block scan of 16 warp totals; (block, exec) pairs written.
//  SELECT   (fused a8) the window set is the phase-1 bitmap: count window
//           blocks without a frame, then scan the LRM log for victims.
template <bool SELECT>
__global__ void __launch_bounds__(PRED_NT) k_predict(PredArgs a) {
  extern __shared__ uint32_t bitmap[];
  __shared__ uint32_t kern[MAXN + 1], loff[MAXN + 2], kcnt[MAXN + 1];
  __shared__ uint32_t dk[DCAP], dv[DCAP];
  __shared__ uint32_t keepbits[UCAP / 32];
  __shared__ uint32_t ws[NWARP], wtot[NWARP];
  __shared__ volatile uint32_t s_ready, s_done;
  __shared__ uint32_t s_ndup, s_ovf, s_ok, s_nonres;
  __shared__ unsigned long long s_base;
  const uint32_t tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const uint32_t qi = blockIdx.x;
  const Geo &g = a.g;
  const dum_query Q = a.q[qi];
  const bool anchored = Q.anchor != NONE;
  for (uint32_t w = tid; w < a.nwords; w += PRED_NT) bitmap[w] = 0;
  for (uint32_t p = tid; p < DCAP; p += PRED_NT) {
    dk[p] = NONE;
    dv[p] = NONE;
  }
  for (uint32_t p = tid; p <= g.N; p += PRED_NT) kcnt[p] = 0;
  if (tid == 0) {
    s_ready = 0;
    s_done = 0;
    s_ndup = 0;
    s_ovf = 0;
    s_nonres = 0;
    loff[0] = 0;
  }
  __syncthreads();
  if (tid == 0 && anchored && Q.anchor < g.W) {
    bitmap[Q.anchor >> 5] |= 1u << (Q.anchor & 31);
    hmap_insert_min(dk, dv, DCAP, Q.anchor, 0);  // position 0: never kept
    s_ndup = 1;
  }
  __syncthreads();
  WinSrc src{a.walk, a.anchor_pool, kern, loff, 0, g.walk_cap, anchored ? a.anchor_range[2 * qi] : 0, anchored};
  // ---------------- phase 1 ----------------
  if (wid == 0) {
    if (lane == 0) {
      const uint32_t E = *(volatile uint32_t *)&a.st->E;
      uint32_t nk = 0, tot = 0;
      auto publish = [&](uint32_t e, uint32_t d) {
        uint32_t len = (d == 0 && anchored) ? (uint32_t)a.anchor_range[2 * qi + 1] : a.walk_len[e];
        // a kernel met earlier in the chain with the same (unanchored) walk
        // cannot add anything (exact; keeps the reservation tight)
        for (uint32_t d2 = anchored ? 1u : 0u; d2 < d && len; ++d2)
          if (kern[d2] == e) len = 0;
        kern[d] = e;
        tot += len;
        loff[d + 1] = tot;
        __threadfence_block();
        s_ready = d + 1;
      };
      if (Q.exec < E) {
        const uint32_t n = Q.n < g.N ? Q.n : g.N;
        uint32_t cur = Q.exec, h1 = Q.hist[0], h2 = Q.hist[1], h3 = Q.hist[2];
        publish(cur, nk++);
        for (uint32_t i = 0; i < n; ++i) {
          const uint32_t nx = corr_lookup(a.corr, a.corr_cap, cur, h1, h2, h3);
          if (nx == NONE) break;
          publish(nx, nk++);
          h1 = h2;  // D16: shift register over predicted IDs
          h2 = h3;
          h3 = cur;
          cur = nx;
        }
      }
      __threadfence_block();
      s_done = 1;
    }
  } else {
    uint32_t d = 0;
    for (;;) {
      uint32_t ready = s_ready;
      if (d >= ready) {
        if (s_done) {
          __threadfence_block();
          ready = s_ready;
          if (d >= ready) break;
        } else {
          __nanosleep(64);
          continue;
        }
      }
      const uint32_t L = loff[d + 1] - loff[d];
      const uint32_t e = kern[d];
      const uint32_t *lst = (d == 0 && anchored) ? a.anchor_pool + src.abase : a.walk + (uint64_t)e * g.walk_cap;
      for (uint32_t idx = (wid - 1) * 32 + lane; idx < L; idx += (NWARP - 1) * 32) {
        const uint32_t b = __ldg(lst + idx);
        const uint32_t bit = 1u << (b & 31);
        const uint32_t old = atomicOr(&bitmap[b >> 5], bit);
        if (old & bit) {
          if (!hmap_insert_min(dk, dv, DCAP, b, loff[d] + idx + 1)) s_ovf = 1;
          atomicAdd(&s_ndup, 1u);
        }
      }
      ++d;
    }
  }
  __syncthreads();
  uint32_t nk = s_ready;
  const uint32_t U = loff[nk];
  src.nk = nk;
  if (tid == 0) {
    const unsigned long long base = atomicAdd(&a.st->pool_pairs, (unsigned long long)U);
    s_base = base;
    s_ok = base + U <= a.cap;
    if (!s_ok) set_err(a.st, ERR_ECAPACITY, base + U);
  }
  const bool ndup = s_ndup != 0;
  if (s_ovf) {
    // too many duplicated blocks for the window-wide hash: exact chunked
    // fallback (ordered chunks, chunk-local min-position hash)
    for (uint32_t w = tid; w < a.nwords; w += PRED_NT) bitmap[w] = 0;
    __syncthreads();
    if (tid == 0 && anchored && Q.anchor < g.W) bitmap[Q.anchor >> 5] |= 1u << (Q.anchor & 31);
    for (uint32_t p = tid; p < CH_CAP; p += PRED_NT) {
      dk[p] = NONE;
      dv[p] = NONE;
    }
    __syncthreads();
    const unsigned long long base = s_base;
    const bool ok = s_ok;
    uint32_t run = 0, d = 0;
    for (uint32_t c = 0; c < U; c += PRED_NT) {
      const uint32_t t = c + tid;
      uint32_t b = NONE;
      bool fresh = false;
      if (t < U) {
        b = src.get(t, d);
        fresh = !(bitmap[b >> 5] & (1u << (b & 31)));
        if (fresh) hmap_insert_min(dk, dv, CH_CAP, b, t);
      }
      __syncthreads();
      const uint32_t keep = fresh && hmap_get(dk, dv, CH_CAP, b) == t;
      if (keep) {
        atomicOr(&bitmap[b >> 5], 1u << (b & 31));
        atomicAdd(&kcnt[d], 1u);
        if (SELECT && __ldg(&a.so.frame_of[b]) == NONE) atomicAdd(&s_nonres, 1u);
      }
      uint32_t tot;
      const uint32_t pre = block_excl_scan(keep, ws, &tot);
      if (keep && ok) reinterpret_cast<uint2 *>(a.pairs)[base + run + pre] = make_uint2(b, kern[d]);
      run += tot;
      for (uint32_t p = tid; p < CH_CAP; p += PRED_NT) {
        dk[p] = NONE;
        dv[p] = NONE;
      }
      __syncthreads();
    }
    if (tid == 0) wtot[0] = run;
  } else {
    // ---------------- phase 2 ----------------
    if (ndup) {
      uint32_t d = 0;
      for (uint32_t t = tid; t < U; t += PRED_NT) {
        const uint32_t b = src.get(t, d);
        const uint32_t s0 = hslot(b, DCAP);
        for (uint32_t p = 0, s = s0; p < DCAP; ++p, s = (s + 1) & (DCAP - 1)) {
          const uint32_t k = dk[s];
          if (k == NONE) break;
          if (k == b) {
            atomicMin(&dv[s], t + 1);
            break;
          }
        }
      }
      __syncthreads();
    }
    // ---------------- phase 3: keep bits and per-warp counts ----------------
    const uint32_t seg = ((U + NWARP - 1) / NWARP + 31) & ~31u;
    const uint32_t t0 = wid * seg, t1 = min(U, t0 + seg);
    const bool bits = U <= UCAP;
    uint32_t cnt = 0;
    {
      uint32_t d = 0;
      for (uint32_t c = t0; c < t1; c += 32) {
        const uint32_t t = c + lane;
        bool keep = false;
        if (t < t1) {
          const uint32_t b = src.get(t, d);
          keep = !ndup;
          if (ndup) {
            const uint32_t m = hmap_get(dk, dv, DCAP, b);
            keep = (m == NONE) || (m == t + 1);
          }
        }
        const uint32_t mask = __ballot_sync(0xffffffffu, keep);
        if (bits && lane == 0) keepbits[c >> 5] = mask;
        cnt += __popc(mask);
      }
    }
    if (lane == 0) wtot[wid] = cnt;
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
    // ---------------- phase 4: ordered write ----------------
    const unsigned long long base = s_base;
    const bool ok = s_ok;
    uint32_t pos = wtot[wid];
    uint32_t nonres = 0;
    {
      uint32_t d = 0;
      for (uint32_t c = t0; c < t1; c += 32) {
        const uint32_t t = c + lane;
        uint32_t b = NONE;
        bool keep = false;
        if (t < t1) {
          b = src.get(t, d);
          if (bits) {
            keep = (keepbits[c >> 5] >> lane) & 1u;
          } else {
            keep = !ndup;
            if (ndup) {
              const uint32_t m = hmap_get(dk, dv, DCAP, b);
              keep = (m == NONE) || (m == t + 1);
            }
          }
        }
        const uint32_t mask = __ballot_sync(0xffffffffu, keep);
        if (keep) {
          if (ok) reinterpret_cast<uint2 *>(a.pairs)[base + pos + __popc(mask & ((1u << lane) - 1))] =
              make_uint2(b, kern[d]);
          if (SELECT) nonres += __ldg(&a.so.frame_of[b]) == NONE;
        }
        // per-kernel counts (kern_off): one add per distinct kernel among kept lanes
        const uint32_t grp = __match_any_sync(0xffffffffu, keep ? d : 0xFFFFFFFFu);
        if (keep && lane == __ffs(grp) - 1) atomicAdd(&kcnt[d], __popc(grp));
        pos += __popc(mask);
      }
    }
    if (SELECT) {
#pragma unroll
      for (int o = 16; o; o >>= 1) nonres += __shfl_xor_sync(0xffffffffu, nonres, o);
      if (lane == 0 && nonres) atomicAdd(&s_nonres, nonres);
    }
    __syncthreads();
    if (tid == 0) wtot[0] = ws[0];
  }
  __syncthreads();
  const uint32_t run = wtot[0];
  const unsigned long long base = s_base;
  if (tid == 0) {
    a.range[2 * qi] = base;
    a.range[2 * qi + 1] = base + (s_ok ? run : 0);
    ctr_add(a.st, DUM_CTR_QUERIES, 1);
    ctr_add(a.st, DUM_CTR_CHAIN, nk);
    ctr_add(a.st, DUM_CTR_GATHERED, U);
    ctr_add(a.st, DUM_CTR_EMITTED, run);
  }
  if (a.kern_off) {
    uint32_t *ko = a.kern_off + (uint64_t)qi * (g.N + 2);
    if (tid == 0) {
      uint32_t acc = 0;
      ko[0] = 0;
      for (uint32_t d = 0; d <= g.N; ++d) {
        if (d < nk) acc += kcnt[d];
        ko[d + 1] = acc;
      }
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
  cudaMemsetAsync(&e->d_state->pool_pairs, 0, sizeof(unsigned long long), s);
  cudaMemsetAsync(&e->d_state->pool_anchor, 0, sizeof(unsigned long long), s);
  if (sel) cudaMemsetAsync(&e->d_state->pool_wb, 0, 2 * sizeof(unsigned long long), s);
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
  if (sel) a.so = *sel;
  const size_t smem = (size_t)a.nwords * 4;
  if (sel) {
    cudaFuncSetAttribute(k_predict<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    TimerScope t(e, DUM_T_PREDICT, s);
    k_predict<true><<<nq, PRED_NT, smem, s>>>(a);
  } else {
    cudaFuncSetAttribute(k_predict<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    TimerScope t(e, DUM_T_PREDICT, s);
    k_predict<false><<<nq, PRED_NT, smem, s>>>(a);
  }
  e->kernel_launches += 2;
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
