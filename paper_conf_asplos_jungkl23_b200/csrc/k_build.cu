// a3 - a6: table build.
//
//  k_build_prep   one thread per staged launch k: upsert the record
//                 (e_{k-4}, e_{k-3}, e_{k-2} -> e_k) into entry e_{k-1} of the
//                 execution ID correlation table (PAPER.md; D5): key claimed
//                 with a 128-bit CAS, successor = max(k<<32 | e_k) ("last
//                 wins"), order = min(k) ("first seen") -- order-independent
//                 (SURVEY P4).  Links the launch into its exec ID's group.
//  k_apply_walk   one CTA per exec ID with faults in the batch (the group
//                 leader).  Applies the block-table operations of all its
//                 launches (D7-D11): per fault b_j,
//                 INSERT b_j into row(b_{j-1}) then TOUCH b_j.  Tables of
//                 different exec IDs are independent (P1) and operations on
//                 different sets commute (P2), so the ops are counting-sorted by
//                 set in shared memory and each set's ops are applied in order
//                 by one thread, with the set held in registers.  Then it
//                 rebuilds the walk cache WALK(e, NONE) (
//                 D13) in parallel -- see walk_fast() -- and records Start/End.
//  k_walk_slow    sequential one-warp walker; takes the exec IDs whose walk
//                 exceeded the parallel path's scratch (never on the configs
//                 measured; kept for exactness on any input).
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "device_util.cuh"
#include "kernels.cuh"
#include "corr.cuh"
#include "walk_seq.cuh"

namespace dum {

constexpr int BUILD_NT = 512;
constexpr uint32_t GCAP = 256;    // launches of one exec ID per build batch
constexpr uint32_t OPCAP = 2048;  // ops per apply round
constexpr uint32_t QCAP = 4096;   // smem walk-dedupe hash capacity (|Q| <= 2048)
constexpr uint32_t WCAP = 2048;   // smem per-row counts (latest launch <= 2048 faults)

// ---------------------------------------------------------------------------
// k_build_prep
// ---------------------------------------------------------------------------
__global__ void k_build_prep(uint32_t n_staged, uint32_t k0, const uint32_t *__restrict__ stage_exec,
                             const uint32_t *__restrict__ stage_cnt, CorrSlot *corr, uint32_t corr_cap,
                             uint32_t *rec_slot, uint32_t *head, uint32_t *__restrict__ next,
                             uint32_t *__restrict__ order, DevState *st) {
  const uint32_t j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j == 0) {
    st->pool_big = 0;
    st->n_slow = 0;
  }
  if (j >= n_staged) return;
  auto prev = [&](int m) -> uint32_t {
    long jj = (long)j - m;
    return jj >= 0 ? stage_exec[jj] : st->hist[4 + jj];
  };
  const uint32_t e = stage_exec[j];
  const uint32_t owner = prev(1);
  const bool up = owner != NONE && e != NONE;
  if (up) corr_upsert(corr, corr_cap, rec_slot, owner, prev(4), prev(3), prev(2), e, k0 + j, st);
  const uint32_t nup = __popc(__ballot_sync(__activemask(), up));
  if ((threadIdx.x & 31) == __ffs(__activemask()) - 1) ctr_add(st, DUM_CTR_CORR_UPSERTS, nup);
  if (e != NONE && stage_cnt[j] > 0) {
    next[j] = atomicExch(&head[e], j);
    // big launches first, so the longest CTAs of k_apply_walk start earliest
    const uint32_t c = stage_cnt[j] >= 1024 ? 0u : stage_cnt[j] >= 128 ? 1u : 2u;
    order[c * n_staged + atomicAdd(&st->cls_cnt[c], 1u)] = j;
  }
}

// ---------------------------------------------------------------------------
// set operations in registers (MAXA ways x MAXS successors, runtime A <= MAXA,
// S <= MAXS; all indices static so the set stays in registers)
// ---------------------------------------------------------------------------
template <int MAXA, int MAXS>
struct RegSet {
  uint32_t tag[MAXA];
  uint32_t sc[MAXA][MAXS];

  // Word k of the set when the geometry is exactly MAXA x MAXS (static index).
  static constexpr int NW = MAXA * (1 + MAXS);
  static constexpr int NV = (NW + 3) / 4;  // 16 B vectors covering the set (stride is 32 B aligned)
  __device__ __forceinline__ uint32_t &word(int k) {
    const int w = k / (1 + MAXS), r = k % (1 + MAXS);
    return r == 0 ? tag[w] : sc[w][r - 1];
  }
  __device__ __forceinline__ uint32_t word_c(int k) const {
    const int w = k / (1 + MAXS), r = k % (1 + MAXS);
    return r == 0 ? tag[w] : sc[w][r - 1];
  }
  __device__ __forceinline__ void load(const uint32_t *p, uint32_t A, uint32_t S) {
    if (A == MAXA && S == MAXS) {
      // exact geometry: a few 16 B vector loads instead of A(1+S) scalar ones
      const uint4 *p4 = reinterpret_cast<const uint4 *>(p);
      uint4 v[NV];
#pragma unroll
      for (int i = 0; i < NV; ++i) v[i] = p4[i];
#pragma unroll
      for (int k = 0; k < NW; ++k) {
        const uint4 &x = v[k / 4];
        word(k) = (k & 3) == 0 ? x.x : (k & 3) == 1 ? x.y : (k & 3) == 2 ? x.z : x.w;
      }
      return;
    }
#pragma unroll
    for (int w = 0; w < MAXA; ++w) {
      tag[w] = NONE;
#pragma unroll
      for (int j = 0; j < MAXS; ++j) sc[w][j] = NONE;
      if (w < (int)A) {
        tag[w] = p[w * (1 + S)];
#pragma unroll
        for (int j = 0; j < MAXS; ++j)
          if (j < (int)S) sc[w][j] = p[w * (1 + S) + 1 + j];
      }
    }
  }
  __device__ __forceinline__ void store(uint32_t *p, uint32_t A, uint32_t S) const {
    if (A == MAXA && S == MAXS) {
      uint4 *p4 = reinterpret_cast<uint4 *>(p);
#pragma unroll
      for (int i = 0; i < NV; ++i) {
        uint4 x;
        x.x = 4 * i + 0 < NW ? word_c(4 * i + 0) : NONE;
        x.y = 4 * i + 1 < NW ? word_c(4 * i + 1) : NONE;
        x.z = 4 * i + 2 < NW ? word_c(4 * i + 2) : NONE;
        x.w = 4 * i + 3 < NW ? word_c(4 * i + 3) : NONE;
        p4[i] = x;
      }
      return;
    }
#pragma unroll
    for (int w = 0; w < MAXA; ++w) {
      if (w < (int)A) {
        p[w * (1 + S)] = tag[w];
#pragma unroll
        for (int j = 0; j < MAXS; ++j)
          if (j < (int)S) p[w * (1 + S) + 1 + j] = sc[w][j];
      }
    }
  }
  // TOUCH: the block's row becomes MRU; allocate on a miss, dropping the LRU
  // way (D8, D10).
  __device__ __forceinline__ void touch(uint32_t b, uint32_t A) {
    int hit = -1;
#pragma unroll
    for (int w = 0; w < MAXA; ++w)
      if (w < (int)A && tag[w] == b) hit = w;
    const int lim = hit < 0 ? (int)A - 1 : hit;  // ways [0, lim) shift down by one
    uint32_t st = b;
    uint32_t ss[MAXS];
#pragma unroll
    for (int j = 0; j < MAXS; ++j) ss[j] = NONE;
    if (hit >= 0) {
#pragma unroll
      for (int w = 0; w < MAXA; ++w)
        if (w == hit) {
#pragma unroll
          for (int j = 0; j < MAXS; ++j) ss[j] = sc[w][j];
        }
    }
#pragma unroll
    for (int w = MAXA - 1; w >= 1; --w) {
      if (w <= lim) {
        tag[w] = tag[w - 1];
#pragma unroll
        for (int j = 0; j < MAXS; ++j) sc[w][j] = sc[w - 1][j];
      }
    }
    tag[0] = st;
#pragma unroll
    for (int j = 0; j < MAXS; ++j) sc[0][j] = ss[j];
  }
  // Row of block b (count + successors, or NONE count when absent) -> out[0..S].
  __device__ __forceinline__ void export_row(uint32_t b, uint32_t A, uint32_t S, uint32_t *out) const {
    int hit = -1;
#pragma unroll
    for (int w = 0; w < MAXA; ++w)
      if (w < (int)A && tag[w] == b) hit = w;
    uint32_t cnt = hit < 0 ? NONE : 0;
#pragma unroll
    for (int w = 0; w < MAXA; ++w) {
      if (w == hit) {
#pragma unroll
        for (int jj = 0; jj < MAXS; ++jj) {
          if (jj < (int)S) {
            out[1 + jj] = sc[w][jj];
            cnt += sc[w][jj] != NONE;
          }
        }
      }
    }
    out[0] = cnt;
  }
  // INSERT s as the MRU successor of the row in way 0 (D9).
  __device__ __forceinline__ void insert0(uint32_t s, uint32_t S) {
    if (s == tag[0]) return;
    int pos = -1;
#pragma unroll
    for (int j = 0; j < MAXS; ++j)
      if (j < (int)S && sc[0][j] == s) pos = j;
    const int lim = pos < 0 ? (int)S - 1 : pos;
#pragma unroll
    for (int j = MAXS - 1; j >= 1; --j)
      if (j <= lim) sc[0][j] = sc[0][j - 1];
    sc[0][0] = s;
  }
};

// ---------------------------------------------------------------------------
// k_apply_walk
// ---------------------------------------------------------------------------
struct BuildArgs {
  Geo g;
  uint32_t n_staged;
  const uint32_t *stage_exec, *stage_cnt, *stage_norm;
  const uint64_t *stage_off;
  uint32_t *head, *next;
  uint32_t *tbl, *start_end, *walk, *walk_len;
  uint32_t *big_pool;
  uint64_t big_entries;
  uint32_t *slow_list;
  uint32_t *wrun, *wrun_len;   // walk bitmap runs (read by k_predict)
  const uint32_t *order;       // [3][n_staged] faulting launches by size class
  DevState *st;
  unsigned long long *cta_clk;  // debug: per-CTA (start, end, n_ops | n << 32) or null
};

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Parallel WALK(e, NONE) right after the build (D13).  Let C = the latest
// faulting launch of e in this batch (deduplicated, n = |C|); then Start =
// C[0], End = C[n-1] (D11).  After the build, the row of C[i] (if still
// present) has C[i+1] as its MRU successor: INSERT(C[i] -> C[i+1]) was the last
// operation on that row, because C is duplicate-free and no later launch of e
// is in the batch.  C[i+1] is not among the chained nodes C[0..i], so the
// sequential walk's next chain node is exactly C[i+1] until the first i at
// which the row is missing or a successor equals End.  With t that index, the
// walk is the first-occurrence dedupe of
//   Q = [C[0]] ++ succ(row C[0]) ++ ... ++ succ(row C[t])   (row C[t] only if
//                                                            present).
// The speculation is still verified (succ[0] == C[i+1]); any violation sends e
// to the sequential walker.
//
// Shared-memory plan (u32 words): grp/seg | row cache of C (count + S succ
// per position, filled by the set owners right after applying the ops, so the
// walk never re-reads the table) | per-row Q offsets | a union of the apply
// arrays (per-set counts/offsets, non-empty-set list, ops, op order) and the
// walk's dedupe hash.
constexpr uint32_t RCCAP = 10240;  // row-cache words: n * (1 + S) <= RCCAP
constexpr uint32_t HCAPMAX = 2 * OPCAP;  // set-hash capacity for a full round

__host__ __device__ inline uint32_t apply_union_words(uint32_t) {
  const uint32_t ap = 2 * HCAPMAX + 3 * OPCAP, wk = 2 * QCAP;
  return ap > wk ? ap : wk;
}

// link op p at the head of its set's list (order fixed up by the owner)
__device__ __forceinline__ void sorted_link(uint32_t p, uint32_t slot, uint32_t *hh, uint32_t *lnk) {
  lnk[p] = atomicExch(&hh[slot], p);
}

template <int MAXA, int MAXS>
__global__ void __launch_bounds__(BUILD_NT, 2) k_apply_walk(BuildArgs a) {
  constexpr int OWN_B = (MAXA * (1 + MAXS) <= 10) ? 2 : 1;  // sets loaded per owner batch
  extern __shared__ uint32_t sm[];
  __shared__ uint32_t ws[BUILD_NT / 32];
  __shared__ uint32_t s_ng, s_tev, s_flag, s_sets, s_nnz, s_nrun;
  __shared__ unsigned long long goff[GCAP];  // stage offset of each group launch
  const Geo &g = a.g;
  const uint32_t tid = threadIdx.x;
  const unsigned long long t_begin = a.cta_clk ? gtimer() : 0;
  if (blockIdx.x == 0 && tid == 0) {
    // history shift register after this batch: the last four exec IDs of
    // (old history ++ staged launches); read by k_build_prep only.
    uint32_t h[4];
    for (int q = 0; q < 4; ++q) {
      const long jj = (long)a.n_staged - 4 + q;
      h[q] = jj >= 0 ? a.stage_exec[jj] : a.st->hist[4 + jj];
    }
    for (int q = 0; q < 4; ++q) a.st->hist[q] = h[q];
  }
  const uint32_t cls = blockIdx.x / a.n_staged, ci = blockIdx.x % a.n_staged;
  if (ci >= __ldcg(&a.st->cls_cnt[cls])) return;
  const uint32_t j = a.order[cls * a.n_staged + ci];
  const uint32_t e = a.stage_exec[j];
  if (e == NONE || a.stage_cnt[j] == 0) return;
  // Leader test, decided once per CTA: thread 0 resets head[e] below, so a
  // per-thread read could see the reset and drop part of the CTA.
  if (tid == 0) s_flag = __ldcg(&a.head[e]) == j;
  __syncthreads();
  if (!s_flag) return;  // not this exec ID's group leader

  const uint32_t R = g.R, A = g.A, S = g.S;
  uint32_t *grp = sm;             // [GCAP]
  uint32_t *seg = grp + GCAP;     // [GCAP + 1]
  uint32_t *rc = seg + GCAP + 1;  // [RCCAP]
  uint32_t *cqs = rc + RCCAP;     // [WCAP]
  uint32_t *U = cqs + WCAP;       // union region
#ifdef DUM_POISON
  {
    const uint32_t words = 2 * GCAP + 1 + RCCAP + WCAP + apply_union_words(R);
    for (uint32_t w = tid; w < words; w += BUILD_NT) sm[w] = 0xDEAD0000u | (w & 0xFFFF);
    __syncthreads();
  }
#endif

  // ---- collect and order the group's launches ----
  if (tid == 0) {
    uint32_t x = j, n = 0;
    while (x != NONE && n < GCAP) {
      if (!GUARD(a.st, x < a.n_staged && a.stage_exec[x] == e, x)) break;
      grp[n++] = x;
      x = __ldcg(&a.next[x]);
    }
    if (x != NONE) set_err(a.st, ERR_ECAPACITY, GCAP + 1);
    s_ng = n;
    s_sets = 0;
    a.head[e] = NONE;
  }
  __syncthreads();
  const uint32_t ng = s_ng;
  if (ng > 1) {
    uint32_t *tmp = U;  // rank sort (ascending launch index)
    for (uint32_t p = tid; p < ng; p += BUILD_NT) {
      uint32_t v = grp[p], r = 0;
      for (uint32_t q = 0; q < ng; ++q) r += grp[q] < v;
      tmp[r] = v;
    }
    __syncthreads();
    for (uint32_t p = tid; p < ng; p += BUILD_NT) grp[p] = tmp[p];
    __syncthreads();
  }
  if (tid == 0) {
    uint32_t acc = 0;
    for (uint32_t p = 0; p < ng; ++p) {
      seg[p] = acc;
      acc += a.stage_cnt[grp[p]];
      goff[p] = a.stage_off[grp[p]];
    }
    seg[ng] = acc;
  }
  __syncthreads();
  if (a.cta_clk && tid == 0) a.cta_clk[10 * j + 3] = gtimer();
  const uint32_t n_ops = seg[ng];
  const uint32_t last_seg = seg[ng - 1];
  const uint32_t Llast = grp[ng - 1];
  const uint32_t n = a.stage_cnt[Llast];
  const bool single_round = n_ops <= OPCAP;
  const bool use_rc = single_round && n <= WCAP && n * (1 + S) <= RCCAP;
  uint32_t *tbl_e = a.tbl + (uint64_t)e * R * g.stride;

  // ---- apply: rounds of up to OPCAP ops, grouped by set ----
  // Each op (fused TOUCH b_p + INSERT b_p -> b_{p+1}) is linked into its set's
  // list through a shared hash keyed by set index (O(ops), independent of R);
  // the owner of a set collects the set's ops, orders them by position (lists
  // are tiny), loads the set into registers, applies them and stores it.
  uint32_t *hk = U, *hh = U + HCAPMAX;          // set key, list head
  uint32_t *opb = U + 2 * HCAPMAX, *onx = opb + OPCAP;
  for (uint32_t r0 = 0; r0 < n_ops; r0 += OPCAP) {
    const uint32_t m = min(OPCAP, n_ops - r0);
    uint32_t hcap = pow2ceil(2 * m);
    if (hcap < 64) hcap = 64;
    for (uint32_t p = tid; p < hcap; p += BUILD_NT) {
      hk[p] = NONE;
      hh[p] = NONE;
    }
    __syncthreads();
    // (1) gather the round's op blocks (coalesced, independent loads)
    for (uint32_t p = tid; p < m; p += BUILD_NT) {
      const uint32_t gp = r0 + p;
      uint32_t lo = 0, hi = ng;  // seg[lo] <= gp < seg[lo+1]
      while (hi - lo > 1) {
        const uint32_t mid = (lo + hi) >> 1;
        if (seg[mid] <= gp) lo = mid;
        else hi = mid;
      }
      const uint64_t base = goff[lo] + (gp - seg[lo]);
      uint32_t b = a.stage_norm[base];
      if (!GUARD(a.st, b < g.W, b)) b = 0;
      opb[p] = b;
      // successor within the same launch: the next op, or past the round's end
      // CLAIM marks "the next op of this round" (never a block id: ids < 2^20)
      onx[p] = (gp + 1 < seg[lo + 1]) ? (p + 1 < m ? (uint32_t)CLAIM : a.stage_norm[base + 1]) : NONE;
    }
    __syncthreads();
    // (2) link each op into its set's list
    for (uint32_t p = tid; p < m; p += BUILD_NT) {
      const uint32_t b = opb[p];
      if (onx[p] == CLAIM) onx[p] = opb[p + 1];
      const uint32_t key = row_of(g, b);
      uint32_t sl = hslot(key, hcap);
      for (;;) {
        const uint32_t old = atomicCAS(&hk[sl], NONE, key);
        if (old == NONE || old == key) break;
        sl = (sl + 1) & (hcap - 1);
      }
      sorted_link(p, sl, hh, U + 2 * HCAPMAX + 2 * OPCAP);
    }
    __syncthreads();
  if (a.cta_clk && tid == 0) a.cta_clk[10 * j + 4] = gtimer();
    uint32_t *lnk = U + 2 * HCAPMAX + 2 * OPCAP;  // per-op next pointer of its set list
    uint32_t nsets = 0;
    for (uint32_t k0 = tid; k0 < hcap; k0 += BUILD_NT * OWN_B) {
      RegSet<MAXA, MAXS> rs[OWN_B];
      uint32_t sid[OWN_B], head[OWN_B];
#pragma unroll
      for (int q = 0; q < OWN_B; ++q) {  // issue every set load of the batch first
        const uint32_t k = k0 + q * BUILD_NT;
        sid[q] = k < hcap ? hk[k] : NONE;
        head[q] = k < hcap ? hh[k] : NONE;
        if (sid[q] != NONE) rs[q].load(tbl_e + (uint64_t)sid[q] * g.stride, A, S);
      }
#pragma unroll
      for (int q = 0; q < OWN_B; ++q) {
        if (sid[q] == NONE) continue;
        ++nsets;
        // the set's ops in position order: repeatedly take the smallest
        // remaining position from the (short) list
        uint32_t last = 0xFFFFFFFFu;
        for (;;) {
          uint32_t best = NONE;
          for (uint32_t x = head[q]; x != NONE; x = lnk[x])
            if ((last == 0xFFFFFFFFu || x > last) && (best == NONE || x < best)) best = x;
          if (best == NONE) break;
          if (!GUARD(a.st, best < m, best)) break;
          rs[q].touch(opb[best], A);
          if (onx[best] != NONE) rs[q].insert0(onx[best], S);
          last = best;
        }
        rs[q].store(tbl_e + (uint64_t)sid[q] * g.stride, A, S);
        if (use_rc) {
          // row cache for the walk: final rows of the latest launch's blocks
          for (uint32_t x = head[q]; x != NONE; x = lnk[x]) {
            if (r0 + x < last_seg) continue;
            const uint32_t i = r0 + x - last_seg;
            if (!GUARD(a.st, i < n && (i + 1) * (1 + S) <= RCCAP, i)) continue;
            rs[q].export_row(opb[x], A, S, rc + i * (1 + S));
          }
        }
      }
    }
    if (nsets) atomicAdd(&s_sets, nsets);
    __syncthreads();
  }
  if (tid == 0) {
    ctr_add(a.st, DUM_CTR_EXEC_BUILT, 1);
    ctr_add(a.st, DUM_CTR_OPS, n_ops);
    ctr_add(a.st, DUM_CTR_SETS, s_sets);
  }
  if (a.cta_clk && tid == 0) a.cta_clk[10 * j + 5] = gtimer();
  // ---- Start / End from the latest launch (D11) ----
  const uint32_t *C = a.stage_norm + a.stage_off[Llast];
  const uint32_t start = C[0], end = C[n - 1];
  if (tid == 0) {
    a.start_end[2 * e] = start;
    a.start_end[2 * e + 1] = end;
  }
  uint32_t *wout = a.walk + (uint64_t)e * g.walk_cap;
  if (n == 1) {  // x == End: the walk is [Start]
    if (tid == 0) {
      wout[0] = start;
      a.walk_len[e] = 1;
      reinterpret_cast<uint2 *>(a.wrun)[(uint64_t)e * g.walk_cap] = make_uint2(start >> 5, 1u << (start & 31));
      a.wrun_len[e] = 1;
      ctr_add(a.st, DUM_CTR_WALK_OUT, 1);
    }
    return;
  }
  // row i of the chain: pointer to its successor list (row cache or table)
  // and its successor count; NONE count = row missing
  auto row_at = [&](uint32_t i, const uint32_t *&sc) -> uint32_t {
    if (use_rc) {
      sc = rc + i * (1 + S) + 1;
      DCHECK(rc[i * (1 + S)] == NONE || rc[i * (1 + S)] <= S, "rc[%u]=%x n=%u e=%u\n", i, rc[i * (1 + S)], n, e);
      return rc[i * (1 + S)];
    }
    const uint32_t x = C[i];
    const uint32_t *set = tbl_e + (uint64_t)row_of(g, x) * g.stride;
    int w = -1;
    for (uint32_t q = 0; q < A; ++q)
      if (w < 0 && __ldcg(set + q * (1 + S)) == x) w = (int)q;
    if (w < 0) return NONE;
    sc = set + w * (1 + S) + 1;
    uint32_t cnt = 0;
    while (cnt < S && __ldcg(sc + cnt) != NONE) ++cnt;
    return cnt;
  };

  // ---- pass A: per chain position i < n-1: row present? stop? successor count ----
  uint32_t *cq;
  // without the row cache, [rc, end of U) is free for the walk's arrays
  const uint32_t free_words = RCCAP + WCAP + apply_union_words(R);
  const uint32_t cq_words = (n + 31) & ~31u;
  if (n <= WCAP) {
    cq = use_rc ? cqs : rc;
  } else if (!use_rc && cq_words + 2 * 1024 <= free_words) {
    cq = rc;
  } else {
    if (tid == 0) {
      const unsigned long long off = atomicAdd(&a.st->pool_big, (unsigned long long)n);
      s_flag = off + n <= a.big_entries * 2 ? 0u : 1u;
      s_tev = (uint32_t)off;
    }
    __syncthreads();
    if (s_flag) {
      if (tid == 0) a.slow_list[atomicAdd(&a.st->n_slow, 1u)] = e;
      return;
    }
    cq = a.big_pool + s_tev;
    __syncthreads();
  }
  if (tid == 0) s_tev = NONE;
  __syncthreads();
  for (uint32_t i = tid; i < n - 1; i += BUILD_NT) {
    const uint32_t *sc = nullptr;
    const uint32_t cnt = row_at(i, sc);
    uint32_t ev = 0;
    if (cnt == NONE) {
      ev = 1;  // row missing: stop, nothing emitted at this step
      cq[i] = 0;
    } else {
      bool hit = false;
      for (uint32_t q = 0; q < cnt; ++q) hit |= sc[q] == end;
      if (hit) ev = 2;                                   // a successor is End: stop after emitting
      else if (cnt == 0 || sc[0] != C[i + 1]) ev = 3;    // speculation violated -> sequential walker
      cq[i] = cnt;
    }
    if (ev) atomicMin(&s_tev, (i << 2) | ev);
  }
  __syncthreads();
  if (a.cta_clk && tid == 0) a.cta_clk[10 * j + 6] = gtimer();
  const uint32_t tev = s_tev;
  if (tev == NONE || (tev & 3) == 3) {
    if (tid == 0) a.slow_list[atomicAdd(&a.st->n_slow, 1u)] = e;
    return;
  }
  const uint32_t t = tev >> 2;
  if (!GUARD(a.st, t + 1 < n, t)) {
    if (tid == 0) a.slow_list[atomicAdd(&a.st->n_slow, 1u)] = e;
    return;
  }
  // ---- pass B: Q positions (qpos[i] = 1 + sum cq[0..i)) in place ----
  uint32_t run = 1;
  for (uint32_t c = 0; c <= t; c += BUILD_NT) {
    const uint32_t i = c + tid;
    const uint32_t v = i <= t ? cq[i] : 0;
    uint32_t tot;
    const uint32_t pre = block_excl_scan(v, ws, &tot);
    if (i <= t) cq[i] = run + pre;
    run += tot;
  }
  if (a.cta_clk && tid == 0) a.cta_clk[10 * j + 7] = gtimer();
  const uint32_t qlen = run;  // |Q|
  if (!GUARD(a.st, qlen <= 1 + (t + 1) * S, qlen)) {
    if (tid == 0) a.slow_list[atomicAdd(&a.st->n_slow, 1u)] = e;
    return;
  }
  // dedupe map block -> min Q position
  uint32_t *qk, *qv;
  const uint32_t qcap = pow2ceil(2 * qlen);
  const bool cq_in_rc = cq == rc;
  if (use_rc && qcap <= QCAP) {
    qk = U;
    qv = qk + qcap;
  } else if (!use_rc && (cq_in_rc ? cq_words : 0) + 2 * qcap <= free_words) {
    qk = rc + (cq_in_rc ? cq_words : 0);
    qv = qk + qcap;
  } else {
    if (tid == 0) {
      const unsigned long long off = atomicAdd(&a.st->pool_big, 2ull * qcap);
      s_flag = off + 2ull * qcap <= a.big_entries * 2 ? 0u : 1u;
      s_tev = (uint32_t)off;
    }
    __syncthreads();
    if (s_flag) {
      if (tid == 0) a.slow_list[atomicAdd(&a.st->n_slow, 1u)] = e;
      return;
    }
    qk = a.big_pool + s_tev;
    qv = qk + qcap;
  }
  for (uint32_t p = tid; p < qcap; p += BUILD_NT) {
    qk[p] = NONE;
    qv[p] = NONE;
  }
  __syncthreads();
  if (tid == 0) hmap_insert_min(qk, qv, qcap, start, 0);
  for (uint32_t i = tid; i <= t; i += BUILD_NT) {
    const uint32_t q0 = cq[i];
    const uint32_t qn = (i < t ? cq[i + 1] : qlen) - q0;
    if (qn == 0) continue;
    const uint32_t *sc = nullptr;
    row_at(i, sc);
    for (uint32_t q = 0; q < qn; ++q) hmap_insert_min(qk, qv, qcap, sc[q], q0 + q);
  }
  __syncthreads();
  if (a.cta_clk && tid == 0) a.cta_clk[10 * j + 8] = gtimer();
  // ---- pass C: ordered compaction of first occurrences ----
  // The kept blocks of each warp step are also grouped by bitmap word into
  // runs (word, mask) for k_predict (any grouping that puts every block in
  // exactly one run will do; runs of one walk are disjoint).
  uint32_t outn = 0;
  uint2 *wrun = reinterpret_cast<uint2 *>(a.wrun) + (uint64_t)e * g.walk_cap;
  if (tid == 0) s_nrun = 0;
  for (uint32_t c = 0; c < qlen; c += BUILD_NT) {
    const uint32_t p = c + tid;
    uint32_t val = NONE, keep = 0;
    if (p < qlen) {
      if (p == 0) {
        val = start;
      } else {
        uint32_t lo = 0, hi = t + 1;  // largest lo with cq[lo] <= p
        while (hi - lo > 1) {
          const uint32_t mid = (lo + hi) >> 1;
          if (cq[mid] <= p) lo = mid;
          else hi = mid;
        }
        const uint32_t *sc = nullptr;
        const uint32_t cnt_lo = row_at(lo, sc);
        val = GUARD(a.st, cnt_lo != NONE && p - cq[lo] < cnt_lo, (lo << 16) | (p - cq[lo])) ? sc[p - cq[lo]] : start;
      }
      keep = hmap_get(qk, qv, qcap, val) == p;
    }
    uint32_t tot;
    const uint32_t pre = block_excl_scan(keep, ws, &tot);
    if (keep && outn + pre < g.walk_cap) wout[outn + pre] = val;
    {
      const uint32_t lane = tid & 31;
      const uint32_t wkey = keep ? val >> 5 : NONE;
      const uint32_t grp = __match_any_sync(0xffffffffu, wkey);
      const uint32_t msk = __reduce_or_sync(grp, keep ? 1u << (val & 31) : 0u);
      const bool lead = keep && lane == (uint32_t)(__ffs(grp) - 1);
      const uint32_t lm = __ballot_sync(0xffffffffu, lead);
      uint32_t rb = 0;
      if (lane == 0 && lm) rb = atomicAdd(&s_nrun, (uint32_t)__popc(lm));
      rb = __shfl_sync(0xffffffffu, rb, 0) + __popc(lm & ((1u << lane) - 1));
      if (lead && rb < g.walk_cap) wrun[rb] = make_uint2(wkey, msk);
    }
    outn += tot;
  }
  __syncthreads();  // every warp's run count is in s_nrun
  if (tid == 0) {
    if (outn > g.walk_cap) set_err(a.st, ERR_ECAPACITY, outn);
    a.walk_len[e] = outn;
    a.wrun_len[e] = s_nrun;
    ctr_add(a.st, DUM_CTR_WALK_ROWS, t + 1);
    ctr_add(a.st, DUM_CTR_WALK_OUT, outn);
    if (a.cta_clk) {
      a.cta_clk[10 * j] = t_begin;
      a.cta_clk[10 * j + 1] = gtimer();
      a.cta_clk[10 * j + 2] = (unsigned long long)n_ops | ((unsigned long long)n << 32);
    }
  }
}

__global__ void k_walk_slow(Geo g, const uint32_t *tbl, const uint32_t *start_end, uint32_t *walk,
                            uint32_t *walk_len, uint32_t *wrun, uint32_t *wrun_len, const uint32_t *slow_list,
                            WalkScratch ws, DevState *st) {
  const uint32_t nslow = *(volatile uint32_t *)&st->n_slow;
  for (uint32_t q = blockIdx.x; q < nslow; q += gridDim.x) {
    const uint32_t e = slow_list[q];
    const uint32_t *tbl_e = tbl + (uint64_t)e * g.R * g.stride;
    uint32_t n = walk_seq(g, tbl_e, start_end[2 * e], start_end[2 * e + 1], NONE, walk + (uint64_t)e * g.walk_cap,
                          g.walk_cap, ws, blockIdx.x);
    if (threadIdx.x == 0) {
      if (n == NONE) {
        set_err(st, ERR_ECAPACITY, g.walk_cap + 1ull);
        n = 0;
      }
      walk_len[e] = n;
    }
    __syncwarp();
    // bitmap runs of the new walk (see pass C of k_apply_walk)
    const uint32_t lane = threadIdx.x & 31;
    const uint32_t *w = walk + (uint64_t)e * g.walk_cap;
    uint2 *out = reinterpret_cast<uint2 *>(wrun) + (uint64_t)e * g.walk_cap;
    const uint32_t len = *(volatile uint32_t *)&walk_len[e];
    uint32_t nr = 0;
    for (uint32_t c = 0; c < len; c += 32) {
      const bool v = c + lane < len;
      const uint32_t b = v ? w[c + lane] : NONE;
      const uint32_t word = v ? b >> 5 : NONE;
      const uint32_t grp = __match_any_sync(0xffffffffu, word);
      const uint32_t mask = __reduce_or_sync(grp, v ? 1u << (b & 31) : 0u);
      const bool lead = v && lane == (uint32_t)(__ffs(grp) - 1);
      const uint32_t lm = __ballot_sync(0xffffffffu, lead);
      if (lead) out[nr + __popc(lm & ((1u << lane) - 1))] = make_uint2(word, mask);
      nr += __popc(lm);
    }
    if (lane == 0) wrun_len[e] = nr;
    __syncwarp();
  }
}

template <int MA, int MS>
static cudaError_t launch_apply(dum_engine *e, const BuildArgs &ba, cudaStream_t s) {
  const size_t smem = (size_t)(2 * GCAP + 1 + RCCAP + WCAP + apply_union_words(ba.g.R)) * 4;
  cudaFuncSetAttribute(k_apply_walk<MA, MS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  cudaFuncSetAttribute(k_apply_walk<MA, MS>, cudaFuncAttributePreferredSharedMemoryCarveout,
                       cudaSharedmemCarveoutMaxShared);
  k_apply_walk<MA, MS><<<3 * ba.n_staged, BUILD_NT, smem, s>>>(ba);
  return cudaGetLastError();
}

cudaError_t launch_build(dum_engine *e, cudaStream_t s) {
  const uint32_t n = e->n_staged;
  if (n == 0) return cudaSuccess;
  {
  TimerScope t(e, DUM_T_BUILD_PREP, s);
  cudaMemsetAsync(e->d_state->cls_cnt, 0, sizeof(e->d_state->cls_cnt), s);
  k_build_prep<<<(n + 255) / 256, 256, 0, s>>>(n, (uint32_t)e->built_launches, e->d_stage_exec, e->d_stage_cnt,
                                                e->d_corr, e->corr_cap, e->d_rec_slot, e->d_head, e->d_next,
                                                e->d_order,
                                                e->d_state);
  }
  // the jump tables depend only on the correlation table, final here
  cudaEventRecord(e->ev_fork, s);
  cudaStreamWaitEvent(e->side, e->ev_fork, 0);
  {
    const cudaError_t je = launch_jump_tables(e, e->side);
    cudaEventRecord(e->ev_join, e->side);
    if (je != cudaSuccess) return je;
  }
  BuildArgs ba;
  ba.g = e->g;
  ba.n_staged = n;
  ba.stage_exec = e->d_stage_exec;
  ba.stage_cnt = e->d_stage_cnt;
  ba.stage_norm = e->d_stage_norm;
  ba.stage_off = e->d_stage_off;
  ba.head = e->d_head;
  ba.next = e->d_next;
  ba.tbl = e->d_tbl;
  ba.start_end = e->d_start_end;
  ba.walk = e->d_walk;
  ba.walk_len = e->d_walk_len;
  ba.big_pool = e->d_big_pool;
  ba.big_entries = e->big_pool_entries;
  ba.slow_list = e->d_slow_list;
  ba.wrun = e->d_wrun;
  ba.wrun_len = e->d_wrun_len;
  ba.order = e->d_order;
  ba.st = e->d_state;
  ba.cta_clk = nullptr;
  static const char *clk_path = getenv("DUM_CTA_CLOCK");
  static unsigned long long *d_clk = nullptr;
  static int clk_calls = 0;
  if (clk_path) {
    if (!d_clk) cudaMalloc(&d_clk, 10ull * 8 * e->stage_launch_cap);
    cudaMemsetAsync(d_clk, 0, 10ull * 8 * n, s);
    ba.cta_clk = d_clk;
  }
  cudaError_t err;
  {
  TimerScope t(e, DUM_T_APPLY_WALK, s);
  if (e->g.A <= 2 && e->g.S <= 4) err = launch_apply<2, 4>(e, ba, s);
  else if (e->g.A == 2 && e->g.S == 8) err = launch_apply<2, 8>(e, ba, s);
  else if (e->g.A == 4 && e->g.S == 4) err = launch_apply<4, 4>(e, ba, s);
  else if (e->g.A <= 4 && e->g.S <= 8) err = launch_apply<4, 8>(e, ba, s);
  else err = launch_apply<32, 32>(e, ba, s);
  }
  if (err != cudaSuccess) return err;
  WalkScratch ws{e->d_walk_seen, e->d_walk_chain, e->d_walk_tmp, e->walk_hash_cap,
                 e->g.walk_cap + e->g.R * e->g.A + 4};
  {
    TimerScope t(e, DUM_T_WALK_SLOW, s);
    k_walk_slow<<<e->n_walk_slots, 32, 0, s>>>(e->g, e->d_tbl, e->d_start_end, e->d_walk, e->d_walk_len,
                                               e->d_wrun, e->d_wrun_len, e->d_slow_list, ws, e->d_state);
  }
  if (clk_path) {
    std::vector<unsigned long long> h(10ull * n);
    cudaStreamSynchronize(s);
    cudaMemcpy(h.data(), d_clk, 8ull * 10 * n, cudaMemcpyDeviceToHost);
    char fn[512];
    snprintf(fn, sizeof fn, "%s.%d", clk_path, clk_calls++);
    if (FILE *f = fopen(fn, "wb")) {
      fwrite(h.data(), 8, h.size(), f);
      fclose(f);
    }
  }
  cudaStreamWaitEvent(s, e->ev_join, 0);
  e->kernel_launches += 3;
  return cudaGetLastError();
}

}  // namespace dum
