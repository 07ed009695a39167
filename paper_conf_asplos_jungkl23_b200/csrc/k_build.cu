// a3 - a6: table build.
//
//  k_build_prep   one thread per staged launch k: upsert the record
//                 (e_{k-4}, e_{k-3}, e_{k-2} -> e_k) into entry e_{k-1} of the
//                 execution ID correlation table (PAPER.md; D5): key claimed
//                 with a 128-bit CAS, successor = max(k<<32 | e_k) ("last
//                 wins"), order = min(k) ("first seen") -- order-independent
//                 (SURVEY P4).  Links the launch into its exec ID's group and
//                 sums the group's operations / latest launch.
//  k_plan         one CTA: the history shift register, and the work lists of
//                 the two persistent kernels below -- one walk item per exec ID
//                 with faults (its group leader), and P apply items per exec ID,
//                 P = ceil(ops / OPP) set partitions (largest groups first).
//  k_apply        persistent; item (e, c of P): applies the block-table
//                 operations of exec ID e whose set lies in partition c
//                 (D7-D10): per fault b_j, INSERT b_j
//                 into row(b_{j-1}) then TOUCH b_j.  Tables of different exec IDs
//                 are independent (P1) and operations on different sets commute
//                 (P2): a CTA owns the sets {s : (s / 32) mod P = c}, selects their
//                 operations in order, groups them by set through a shared hash,
//                 and one thread per set applies the set's operations with the set
//                 held in registers.  Big exec IDs are thereby spread over many
//                 SMs instead of one.
//  k_walk         persistent; one exec ID per item: Start/End, then the walk
//                 cache WALK(e, NONE) (D13) in parallel --
//                 see the comment above the kernel.
//  k_walk_slow    sequential one-warp walker; takes the exec IDs whose walk
//                 the parallel path cannot prove (never on the configs
//                 measured; kept for exactness on any input).
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include "device_util.cuh"
#include "kernels.cuh"
#include "corr.cuh"
#include "predict.cuh"
#include "walk_seq.cuh"

namespace dum {

constexpr uint32_t GCAP = 256;     // launches of one exec ID per build batch
constexpr int PLAN_NT = 256;
constexpr int AP_NT = 256;         // k_apply threads
constexpr uint32_t OPP = 1024;     // target operations per apply partition
constexpr uint32_t PMAX = 64;      // partitions per exec ID (<= R / 32)
constexpr uint32_t AP_OPCAP = 1024;  // selected operations per apply round
constexpr uint32_t AP_SCAN = 2 * AP_NT;  // operations scanned per selection step
constexpr uint32_t AP_HCAP = 2 * AP_OPCAP;
constexpr int WK_NT = 256;         // k_walk threads
constexpr uint32_t WK_RC = 5120;   // shared row-cache words (n (1 + S) <= WK_RC)
constexpr uint32_t WK_CQ = 1024;   // shared chain-position words (n <= WK_CQ)
constexpr uint32_t WK_QCAP = 4096; // shared dedupe-hash capacity (|Q| <= WK_QCAP / 2)

// ---------------------------------------------------------------------------
// k_build_prep
// ---------------------------------------------------------------------------
__global__ void k_build_prep(uint32_t n_staged, const uint32_t *__restrict__ stage_exec,
                             const uint32_t *__restrict__ stage_cnt, CorrSlot *corr, uint32_t corr_cap,
                             uint32_t *rec_slot, uint32_t *head, uint32_t *__restrict__ next,
                             uint32_t *__restrict__ order, uint32_t *e_ops, uint32_t *e_last,
                             unsigned long long *plan_agg, DevState *st) {
  const uint32_t j = blockIdx.x * blockDim.x + threadIdx.x;
  if (j == 0) {
    st->pool_bigb = 0;  // the build's own scratch (the exact predict kernel may run beside it)
    st->n_slow = 0;
    st->n_dd = 0;
    st->n_items = 0;  // k_plan's last chunk writes the list sizes
    st->n_leads = 0;
  }
  if (j >= n_staged) return;
  auto prev = [&](int m) -> uint32_t {
    long jj = (long)j - m;
    return jj >= 0 ? stage_exec[jj] : st->hist[4 + jj];
  };
  if (j < (n_staged + 255) / 256) plan_agg[j] = 0;  // k_plan's look-back slots
  const uint32_t e = stage_exec[j];
  const uint32_t owner = prev(1);
  const bool up = owner != NONE && e != NONE;
  // global launch index of staged launch j: the device-side base of this build
  // (k_plan advances it; the same value in a replayed graph step)
  const uint32_t k0 = *(volatile uint32_t *)&st->k_base;
  if (up) corr_upsert(corr, corr_cap, rec_slot, owner, prev(4), prev(3), prev(2), e, k0 + j, st);
  const uint32_t nup = __popc(__ballot_sync(__activemask(), up));
  if ((threadIdx.x & 31) == __ffs(__activemask()) - 1) ctr_add(st, DUM_CTR_CORR_UPSERTS, nup);
  if (e != NONE && stage_cnt[j] > 0) {
    next[j] = atomicExch(&head[e], j);
    atomicAdd(&e_ops[e], stage_cnt[j]);
    atomicMax(&e_last[e], j);
    // big launches first (k_plan orders the work lists by this class)
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
  // CG: load through L2 only (sets written earlier by this CTA, k_build_exec)
  template <bool CG = false>
  __device__ __forceinline__ void load(const uint32_t *p, uint32_t A, uint32_t S) {
    if (A == MAXA && S == MAXS) {
      // exact geometry: a few 16 B vector loads instead of A(1+S) scalar ones
      const uint4 *p4 = reinterpret_cast<const uint4 *>(p);
      uint4 v[NV];
#pragma unroll
      for (int i = 0; i < NV; ++i) v[i] = CG ? __ldcg(p4 + i) : p4[i];
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
        tag[w] = CG ? __ldcg(p + w * (1 + S)) : p[w * (1 + S)];
#pragma unroll
        for (int j = 0; j < MAXS; ++j)
          if (j < (int)S) sc[w][j] = CG ? __ldcg(p + w * (1 + S) + 1 + j) : p[w * (1 + S) + 1 + j];
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
// k_plan
// ---------------------------------------------------------------------------
// One exec ID with faults in the batch (written by k_plan, read by k_apply / k_walk).
struct LeadDesc {
  uint32_t j, e;                // group leader launch (head of the group list), exec ID
  uint32_t single, n_ops;       // the group is one launch; operations of the group
  uint32_t n_last, pad;         // faults of the latest launch of the group
  unsigned long long off_last;  // its staging offset
};

struct BuildArgs {
  Geo g;
  uint32_t n_staged;
  const uint32_t *stage_exec, *stage_cnt, *stage_norm;
  const uint64_t *stage_off;
  uint32_t *head, *next;
  uint32_t *e_ops, *e_last;    // per exec ID: operations / latest launch of the batch (k_build_prep)
  LeadDesc *desc;              // [n_leads] exec IDs with faults, largest launches first
  uint2 *items;                // [n_items] apply items (leader index, c | P << 16)
  uint32_t *tbl, *start_end, *walk, *walk_len;
  uint32_t *rowc;              // global row cache for walks too long for shared memory
  uint32_t *big_pool;
  uint64_t big_entries;
  uint32_t *slow_list;
  uint32_t *wrun, *wrun_len;   // walk bitmap runs (read by k_predict)
  const uint32_t *order;       // [3][n_staged] faulting launches by size class
  unsigned long long *plan_agg;  // [k_plan CTAs] published chunk totals (flag << 63 | leads << 32 | items)
  DevState *st;
  uint32_t seq_walks;          // DUM_CFG_SEQ_WALKS
  uint32_t *dd_list;           // k_build_exec -> k_walk: walks that need the min-position dedupe (desc indices)
};

__global__ void __launch_bounds__(PLAN_NT) k_plan(BuildArgs a) {
  __shared__ uint32_t ws[PLAN_NT / 32];
  __shared__ uint32_t s_ib, s_lb;
  const uint32_t tid = threadIdx.x;
  if (blockIdx.x == 0 && tid == 0) {
    // history shift register after this batch: the last four exec IDs of
    // (old history ++ staged launches); read by the next k_build_prep only
    uint32_t h[4];
    for (int q = 0; q < 4; ++q) {
      const long jj = (long)a.n_staged - 4 + q;
      h[q] = jj >= 0 ? a.stage_exec[jj] : a.st->hist[4 + jj];
    }
    for (int q = 0; q < 4; ++q) a.st->hist[q] = h[q];
    a.st->k_base += a.n_staged;  // the next build's launch index base (k_build_prep of this build has read it)
  }
  const uint32_t c0 = a.st->cls_cnt[0], c1 = a.st->cls_cnt[1], c2 = a.st->cls_cnt[2];
  const uint32_t tot = c0 + c1 + c2;
  const uint32_t pmax = max(1u, min(PMAX, a.g.R / 32));
  // one chunk of the class-ordered list per CTA; the CTAs reserve their item
  // ranges with one atomic each (chunks of the big classes come first in CTA
  // order, which is all the largest-first scheduling needs)
  {
    const uint32_t x0 = blockIdx.x * PLAN_NT;
    if (x0 >= tot) return;
    const uint32_t x = x0 + tid;
    uint32_t P = 0, j = NONE, e = NONE;
    LeadDesc d;
    if (x < tot) {
      const uint32_t cls = x < c0 ? 0u : x < c0 + c1 ? 1u : 2u;
      const uint32_t ci = x - (cls == 0 ? 0u : cls == 1 ? c0 : c0 + c1);
      j = a.order[cls * a.n_staged + ci];
      e = a.stage_exec[j];
      // the descriptor's loads go out with the leader test (used by leaders only)
      const uint32_t hd = a.head[e], last = a.e_last[e];
      d.j = j;
      d.e = e;
      d.single = a.next[j] == NONE;
      d.n_ops = a.e_ops[e];
      d.n_last = a.stage_cnt[last];
      d.pad = 0;
      d.off_last = a.stage_off[last];
      if (hd == j) P = min(pmax, max(1u, (d.n_ops + OPP - 1) / OPP));
    }
    uint32_t totP, totL;
    const uint32_t ip = block_excl_scan(P, ws, &totP);
    const uint32_t lp = block_excl_scan(P ? 1u : 0u, ws, &totL);
    // offsets in list order (largest launches keep the lowest item / walk
    // indices): publish this chunk's totals, then add up the earlier chunks'
    // (decoupled look-back; CTAs are dispatched in index order, so every
    // earlier chunk is resident or done)
    if (tid == 0)
      atomicExch(&a.plan_agg[blockIdx.x], (1ull << 63) | ((unsigned long long)totL << 32) | totP);
    if (tid < 32) {
      uint32_t bp = 0, bl = 0;
      for (uint32_t q = tid; q < blockIdx.x; q += 32) {
        unsigned long long v;
        do {
          v = *(volatile unsigned long long *)&a.plan_agg[q];
        } while (!(v >> 63));
        bp += (uint32_t)(v & 0xFFFFFFFFull);
        bl += (uint32_t)((v >> 32) & 0x7FFFFFFFull);
      }
#pragma unroll
      for (int o = 16; o; o >>= 1) {
        bp += __shfl_xor_sync(0xffffffffu, bp, o);
        bl += __shfl_xor_sync(0xffffffffu, bl, o);
      }
      if (tid == 0) {
        s_ib = bp;
        s_lb = bl;
        if (x0 + PLAN_NT >= tot) {  // the last chunk: the list sizes
          a.st->n_items = bp + totP;
          a.st->n_leads = bl + totL;
        }
      }
    }
    __syncthreads();
    const uint32_t ibase = s_ib, lbase = s_lb;
    if (P) {
      a.desc[lbase + lp] = d;
      for (uint32_t c = 0; c < P; ++c) a.items[ibase + ip + c] = make_uint2(lbase + lp, c | (P << 16));
    }
  }
}

// ---------------------------------------------------------------------------
// k_apply
// ---------------------------------------------------------------------------
// The launches of exec ID e's group (ascending launch index) into grp, their
// operation offsets into seg and their staging offsets into goff; returns the
// group size.  j is the group's leader (the head of its list).
__device__ __forceinline__ uint32_t load_group(const BuildArgs &a, uint32_t j, uint32_t e, uint32_t *grp,
                                               uint32_t *seg, unsigned long long *goff, uint32_t *tmp,
                                               uint32_t *s_ng, uint32_t nt) {
  const uint32_t tid = threadIdx.x;
  if (tid == 0) {
    uint32_t x = j, n = 0;
    while (x != NONE && n < GCAP) {
      if (!GUARD(a.st, x < a.n_staged && a.stage_exec[x] == e, x)) break;
      grp[n++] = x;
      x = __ldcg(&a.next[x]);
    }
    if (x != NONE) set_err(a.st, ERR_ECAPACITY, GCAP + 1);
    *s_ng = n;
  }
  __syncthreads();
  const uint32_t ng = *s_ng;
  if (ng > 1) {  // rank sort (ascending launch index)
    for (uint32_t p = tid; p < ng; p += nt) {
      uint32_t v = grp[p], r = 0;
      for (uint32_t q = 0; q < ng; ++q) r += grp[q] < v;
      tmp[r] = v;
    }
    __syncthreads();
    for (uint32_t p = tid; p < ng; p += nt) grp[p] = tmp[p];
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
  return ng;
}

template <int MAXA, int MAXS>
__global__ void __launch_bounds__(AP_NT) k_apply(BuildArgs a) {
  constexpr int OWN_B = (MAXA * (1 + MAXS) <= 10) ? 2 : 1;  // sets loaded per owner batch
  __shared__ uint32_t grp[GCAP], seg[GCAP + 1];
  __shared__ unsigned long long goff[GCAP];
  __shared__ uint32_t opb[AP_OPCAP], onx[AP_OPCAP], opos[AP_OPCAP], lnk[AP_OPCAP], sll[AP_OPCAP];
  __shared__ uint32_t hk[AP_HCAP], hh[AP_HCAP];
  __shared__ uint32_t s_ng, s_m, s_nsl;
  const Geo &g = a.g;
  const uint32_t tid = threadIdx.x;
  const uint32_t A = g.A, S = g.S;
  // one CTA per item; the grid is the host's upper bound on the item count
  // persistent: the grid is sized by occupancy, the item count is on the device
  const uint32_t n_items = *(volatile uint32_t *)&a.st->n_items;
  uint32_t nsets = 0;
  for (uint32_t t = blockIdx.x; t < n_items; t += gridDim.x) {
    const uint2 it = a.items[t];
    const uint32_t c = it.y & 0xFFFFu, P = it.y >> 16;
    const LeadDesc d = a.desc[it.x];
    const uint32_t e = d.e;
    uint32_t ng = 1;
    if (d.single) {  // the common case: no list to chase
      if (tid == 0) {
        seg[0] = 0;
        seg[1] = d.n_ops;
        goff[0] = d.off_last;
      }
      __syncthreads();
    } else {
      ng = load_group(a, d.j, e, grp, seg, goff, hk, &s_ng, AP_NT);
    }
    const uint32_t n_ops = seg[ng];
    __syncthreads();  // every thread has read s_ng (load_group)
    if (tid == 0) s_ng = 0;  // from here on: the CTA's set count
    uint32_t *tbl_e = a.tbl + (uint64_t)e * g.R * g.stride;
    uint32_t m = 0;  // selected operations staged in opb / onx / opos (uniform)
    // apply the staged operations: grouped by set through a shared hash, one
    // owner thread per set applies the set's operations in position order
    auto apply_staged = [&]() {
      uint32_t hcap = pow2ceil(2 * m);
      if (hcap < 64) hcap = 64;
      for (uint32_t p = tid; p < hcap; p += AP_NT) {
        hk[p] = NONE;
        hh[p] = NONE;
      }
      if (tid == 0) s_nsl = 0;
      __syncthreads();
      for (uint32_t p = tid; p < m; p += AP_NT) {
        const uint32_t key = row_of(g, opb[p]);
        uint32_t sl = hslot(key, hcap);
        for (;;) {
          const uint32_t old = atomicCAS(&hk[sl], NONE, key);
          if (old == NONE) sll[atomicAdd(&s_nsl, 1u)] = sl;  // a new set: list its slot
          if (old == NONE || old == key) break;
          sl = (sl + 1) & (hcap - 1);
        }
        lnk[p] = atomicExch(&hh[sl], p);
      }
      __syncthreads();
      const uint32_t nsl = s_nsl;
      for (uint32_t k0 = tid; k0 < nsl; k0 += AP_NT * OWN_B) {
        RegSet<MAXA, MAXS> rs[OWN_B];
        uint32_t sid[OWN_B], hd[OWN_B];
#pragma unroll
        for (int q = 0; q < OWN_B; ++q) {  // issue every set load of the batch first
          const uint32_t k = k0 + q * AP_NT;
          sid[q] = NONE;
          hd[q] = NONE;
          if (k < nsl) {
            const uint32_t sl = sll[k];
            sid[q] = hk[sl];
            hd[q] = hh[sl];
            rs[q].load(tbl_e + (uint64_t)sid[q] * g.stride, A, S);
          }
        }
#pragma unroll
        for (int q = 0; q < OWN_B; ++q) {
          if (sid[q] == NONE) continue;
          ++nsets;
          // the set's operations in position order: repeatedly take the
          // smallest remaining position from the (short) list
          uint32_t last = NONE;
          for (;;) {
            uint32_t best = NONE, bpos = NONE;
            for (uint32_t x = hd[q]; x != NONE; x = lnk[x]) {
              const uint32_t px = opos[x];
              if ((last == NONE || px > last) && (bpos == NONE || px < bpos)) {
                best = x;
                bpos = px;
              }
            }
            if (best == NONE) break;
            if (!GUARD(a.st, best < m, best)) break;
            rs[q].touch(opb[best], A);
            if (onx[best] != NONE) rs[q].insert0(onx[best], S);
            last = bpos;
          }
          rs[q].store(tbl_e + (uint64_t)sid[q] * g.stride, A, S);
        }
      }
      __syncthreads();
      m = 0;
      if (tid == 0) s_m = 0;
    };
    if (tid == 0) s_m = 0;
    __syncthreads();
    for (uint32_t g0 = 0; g0 < n_ops; g0 += AP_SCAN) {
      if (m + AP_SCAN > AP_OPCAP) apply_staged();  // a chunk never straddles two rounds
      // ---- select this partition's operations of [g0, g0 + AP_SCAN) ----
      // Per set, the operations must be applied in position order; across sets
      // any order will do, so the selected ones are appended in any order with
      // their position (P > 1), or in place (P == 1).
      constexpr uint32_t U = AP_SCAN / AP_NT;
      uint32_t b[U], nx[U], gp[U];
      bool sel[U];
#pragma unroll
      for (uint32_t u = 0; u < U; ++u) {  // issue the loads first
        gp[u] = g0 + u * AP_NT + tid;
        b[u] = NONE;
        nx[u] = NONE;
        sel[u] = false;
        if (gp[u] < n_ops) {
          uint32_t lo = 0, hi = ng;  // seg[lo] <= gp < seg[lo+1]
          while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (seg[mid] <= gp[u]) lo = mid;
            else hi = mid;
          }
          const uint64_t base = goff[lo] + (gp[u] - seg[lo]);
          b[u] = a.stage_norm[base];
          // INSERT target: the next fault of the same launch
          if (gp[u] + 1 < seg[lo + 1]) nx[u] = a.stage_norm[base + 1];
        }
      }
#pragma unroll
      for (uint32_t u = 0; u < U; ++u) {
        if (gp[u] < n_ops) {
          if (!GUARD(a.st, b[u] < g.W, b[u])) b[u] = 0;
          sel[u] = P == 1 || ((row_of(g, b[u]) >> 5) % P) == c;
        }
        uint32_t slot = m + u * AP_NT + tid;
        if (P != 1) {  // warp-aggregated append
          const uint32_t lane = tid & 31, bal = __ballot_sync(0xffffffffu, sel[u]);
          uint32_t base = 0;
          if (lane == 0 && bal) base = atomicAdd(&s_m, (uint32_t)__popc(bal));
          slot = __shfl_sync(0xffffffffu, base, 0) + __popc(bal & ((1u << lane) - 1));
        }
        if (sel[u]) {
          opb[slot] = b[u];
          onx[slot] = nx[u];
          opos[slot] = gp[u];
        }
      }
      __syncthreads();
      m = P == 1 ? m + min(AP_SCAN, n_ops - g0) : s_m;
    }
    if (m) apply_staged();
    __syncthreads();  // the next item reuses the shared state
  }
  // one global atomic per CTA (a per-thread atomic on one address serialises
  // hundreds of thousands of updates in L2)
  __shared__ uint32_t s_sets;
  if (tid == 0) s_sets = 0;
  __syncthreads();
  nsets = __reduce_add_sync(0xffffffffu, nsets);
  if ((tid & 31) == 0 && nsets) atomicAdd(&s_sets, nsets);
  __syncthreads();
  if (tid == 0 && s_sets) ctr_add(a.st, DUM_CTR_SETS, s_sets);
}

// ---------------------------------------------------------------------------
// k_build_exec: a4 + a5 + a6 of one exec ID per item (persistent, largest
// exec IDs first), fused so that the walk reads the sets its own apply just
// wrote (L2-hot) and one kernel replaces the partitioned apply and the walk.
//  apply  the exec ID's operations (INSERT b_j into row(b_{j-1}), TOUCH b_j;
//         PAPER.md L168, L174, L216; D7-D10) in rounds of BX_RC in position
//         order; per round the operations are linked per set (shared head
//         table over the R sets) and one owner thread applies a set's
//         operations in position order with the set in registers (SURVEY P2:
//         operations on different sets commute).
//  walk   Start/End (D11) and WALK(e, NONE) (L218-L224; D13) as k_walk's fast
//         path: the walk is the prefix C[0 .. t+1] of the latest launch when
//         rows C[0..t] each hold the single successor C[i+1] (see k_walk);
//         any other walk goes to k_walk's exact dedupe (dd_list) or the
//         sequential walker (slow_list).
// ---------------------------------------------------------------------------
constexpr int BX_NT = 256;
constexpr uint32_t BX_RC = 1024;  // operations per apply round

template <int MAXA, int MAXS>
__global__ void __launch_bounds__(BX_NT, 4) k_build_exec(BuildArgs a) {
  extern __shared__ uint32_t bx[];  // set heads [R] | opb | onx | lnk | sll [BX_RC each]
  __shared__ uint32_t grp[GCAP], seg[GCAP + 1];
  __shared__ unsigned long long goff[GCAP];
  __shared__ uint32_t s_ng, s_nsl, s_tev, s_multi, s_nrun, s_sets;
  const Geo &g = a.g;
  const uint32_t tid = threadIdx.x, lane = tid & 31;
  const uint32_t A = g.A, S = g.S, R = g.R;
  uint32_t *shead = bx, *opb = bx + R, *onx = opb + BX_RC, *lnk = onx + BX_RC, *sll = lnk + BX_RC;
  if (blockIdx.x == 0 && tid < 4) a.st->cls_cnt[tid] = 0;  // k_plan has read them; zero for the next build
  for (uint32_t x = tid; x < R; x += BX_NT) shead[x] = NONE;  // kept clean by the owners
  if (tid == 0) s_sets = 0;
  const uint32_t n_leads = *(volatile uint32_t *)&a.st->n_leads;
  uint32_t nsets = 0;
  for (uint32_t li = blockIdx.x; li < n_leads; li += gridDim.x) {
    const LeadDesc d = a.desc[li];
    const uint32_t e = d.e;
    uint32_t ng = 1;
    if (d.single) {  // the common case: no list to chase
      if (tid == 0) {
        seg[0] = 0;
        seg[1] = d.n_ops;
        goff[0] = d.off_last;
        s_nsl = 0;
      }
      __syncthreads();
    } else {
      if (tid == 0) s_nsl = 0;
      ng = load_group(a, d.j, e, grp, seg, goff, sll, &s_ng, BX_NT);
    }
    const uint32_t n_ops = seg[ng];
    uint32_t *tbl_e = a.tbl + (uint64_t)e * R * g.stride;
    // ---- a4: the operations, BX_RC per round (rounds in position order) ----
    for (uint32_t g0 = 0; g0 < n_ops; g0 += BX_RC) {
      const uint32_t m = min(BX_RC, n_ops - g0);
      for (uint32_t p = tid; p < m; p += BX_NT) {
        const uint32_t gp = g0 + p;
        uint32_t lo = 0, hi = ng;  // seg[lo] <= gp < seg[lo+1]
        while (hi - lo > 1) {
          const uint32_t mid = (lo + hi) >> 1;
          if (seg[mid] <= gp) lo = mid;
          else hi = mid;
        }
        const uint64_t base = goff[lo] + (gp - seg[lo]);
        uint32_t b = a.stage_norm[base];
        // INSERT target: the next fault of the same launch
        const uint32_t nx = gp + 1 < seg[lo + 1] ? a.stage_norm[base + 1] : NONE;
        if (!GUARD(a.st, b < g.W, b)) b = 0;
        opb[p] = b;
        onx[p] = nx;
        const uint32_t sx = row_of(g, b);
        const uint32_t old = atomicExch(&shead[sx], p);
        lnk[p] = old;
        if (old == NONE) sll[atomicAdd(&s_nsl, 1u)] = sx;  // a set touched first in this round
      }
      __syncthreads();
      const uint32_t nsl = s_nsl;
      constexpr int OWN = (MAXA * (1 + MAXS) <= 10) ? 2 : 1;  // sets per owner with loads in flight
      for (uint32_t k0 = tid; k0 < nsl; k0 += BX_NT * OWN) {
        RegSet<MAXA, MAXS> rs[OWN];
        uint32_t sx[OWN], hd[OWN];
#pragma unroll
        for (int q = 0; q < OWN; ++q) {
          const uint32_t k = k0 + q * BX_NT;
          sx[q] = k < nsl ? sll[k] : NONE;
          hd[q] = NONE;
          if (sx[q] != NONE) {
            hd[q] = shead[sx[q]];
            rs[q].template load<true>(tbl_e + (uint64_t)sx[q] * g.stride, A, S);
          }
        }
#pragma unroll
        for (int q = 0; q < OWN; ++q) {
          if (sx[q] == NONE) continue;
          ++nsets;
          // the set's operations in position order: repeatedly the smallest
          // remaining position of its (short) list
          uint32_t last = NONE;
          for (;;) {
            uint32_t best = NONE;
            for (uint32_t x = hd[q]; x != NONE; x = lnk[x])
              if ((last == NONE || x > last) && (best == NONE || x < best)) best = x;
            if (best == NONE) break;
            rs[q].touch(opb[best], A);
            if (onx[best] != NONE) rs[q].insert0(onx[best], S);
            last = best;
          }
          rs[q].store(tbl_e + (uint64_t)sx[q] * g.stride, A, S);
          shead[sx[q]] = NONE;
        }
      }
      if (tid == 0) s_nsl = 0;
      __syncthreads();  // the round's sets are written; the next round may link them again
    }
    // ---- a5 + a6: Start/End and the walk of the post-build table ----
    const uint32_t n = d.n_last;
    const uint32_t *C = a.stage_norm + d.off_last;
    const uint32_t start = C[0], end = C[n - 1];
    if (tid == 0) {
      a.start_end[2 * e] = start;
      a.start_end[2 * e + 1] = end;
      ctr_add(a.st, DUM_CTR_EXEC_BUILT, 1);
      ctr_add(a.st, DUM_CTR_OPS, d.n_ops);
      // the group bookkeeping of this batch is consumed (prep and plan are done)
      a.head[e] = NONE;
      a.e_ops[e] = 0;
      a.e_last[e] = 0;
      s_tev = NONE;
      s_nrun = 0;
      s_multi = NONE;
    }
    uint32_t *wout = a.walk + (uint64_t)e * g.walk_cap;
    uint2 *wrun = reinterpret_cast<uint2 *>(a.wrun) + (uint64_t)e * g.walk_cap;
    if (n == 1 || (a.seq_walks && n > 1)) {
      if (tid == 0) {
        if (n == 1) {  // x == End: the walk is [Start]
          wout[0] = start;
          a.walk_len[e] = 1;
          wrun[0] = make_uint2(start >> 5, 1u << (start & 31));
          a.wrun_len[e] = 1;
          ctr_add(a.st, DUM_CTR_WALK_OUT, 1);
          ctr_add(a.st, DUM_CTR_WALK_PREFIX, 1);
        } else {  // DUM_CFG_SEQ_WALKS: the sequential walker builds every walk
          a.slow_list[atomicAdd(&a.st->n_slow, 1u)] = e;
        }
      }
      __syncthreads();
      continue;
    }
    __syncthreads();
    // pass A: rows of C[0 .. n-2] (written above by this CTA: L2) -> stop events
    constexpr int WB = (MAXA * (1 + MAXS) <= 10) ? 2 : 1;  // rows per thread in flight
    for (uint32_t i0 = tid; i0 < n - 1; i0 += BX_NT * WB) {
      uint32_t x[WB], xn[WB];
      RegSet<MAXA, MAXS> rs[WB];
#pragma unroll
      for (int q = 0; q < WB; ++q) {
        const uint32_t i = i0 + q * BX_NT;
        x[q] = i < n - 1 ? C[i] : NONE;
        xn[q] = i < n - 1 ? C[i + 1] : NONE;
      }
#pragma unroll
      for (int q = 0; q < WB; ++q)
        if (x[q] != NONE) rs[q].template load<true>(tbl_e + (uint64_t)row_of(g, x[q]) * g.stride, A, S);
#pragma unroll
      for (int q = 0; q < WB; ++q) {
        if (x[q] == NONE) continue;
        const uint32_t i = i0 + q * BX_NT;
        uint32_t row[1 + MAXS];
        rs[q].export_row(x[q], A, S, row);
        const uint32_t cnt = row[0];
        uint32_t ev = 0;
        if (cnt == NONE) {
          ev = 1;  // row missing: stop, nothing emitted at this step
        } else {
          bool hit = false;
#pragma unroll
          for (int k = 0; k < MAXS; ++k) hit |= (uint32_t)k < cnt && row[1 + k] == end;
          if (hit) ev = 2;                              // a successor is End: stop after emitting
          else if (cnt == 0 || row[1] != xn[q]) ev = 3;  // speculation violated -> sequential walker
          if (cnt > 1) atomicMin(&s_multi, i);
        }
        if (ev) atomicMin(&s_tev, (i << 2) | ev);
      }
    }
    __syncthreads();
    const uint32_t tev = s_tev;
    const uint32_t t = tev >> 2;
    if (tev == NONE || (tev & 3) == 3 || !GUARD(a.st, t + 1 < n, t)) {
      if (tid == 0) a.slow_list[atomicAdd(&a.st->n_slow, 1u)] = e;
    } else if (s_multi <= t) {
      if (tid == 0) a.dd_list[atomicAdd(&a.st->n_dd, 1u)] = li;  // k_walk: min-position dedupe
    } else {
      // fast path: the walk is C[0 .. t] (+ C[t+1] when a successor is End),
      // duplicate-free; written with its bitmap runs for k_predict
      const uint32_t qlen = t + 1 + ((tev & 3) == 2 ? 1u : 0u);
      for (uint32_t c0 = 0; c0 < qlen; c0 += BX_NT) {
        const uint32_t p = c0 + tid;
        const bool keep = p < qlen;
        const uint32_t val = keep ? C[p] : NONE;
        if (keep && p < g.walk_cap) wout[p] = val;
        const uint32_t wkey = keep ? val >> 5 : NONE;
        const uint32_t gm = __match_any_sync(0xffffffffu, wkey);
        const uint32_t msk = __reduce_or_sync(gm, keep ? 1u << (val & 31) : 0u);
        const bool lead = keep && lane == (uint32_t)(__ffs(gm) - 1);
        const uint32_t lm = __ballot_sync(0xffffffffu, lead);
        uint32_t rb = 0;
        if (lane == 0 && lm) rb = atomicAdd(&s_nrun, (uint32_t)__popc(lm));
        rb = __shfl_sync(0xffffffffu, rb, 0) + __popc(lm & ((1u << lane) - 1));
        if (lead && rb < g.walk_cap) wrun[rb] = make_uint2(wkey, msk);
      }
      __syncthreads();
      if (tid == 0) {
        if (qlen > g.walk_cap) set_err(a.st, ERR_ECAPACITY, qlen);
        a.walk_len[e] = qlen;
        a.wrun_len[e] = s_nrun;
        ctr_add(a.st, DUM_CTR_WALK_ROWS, t + 1);
        ctr_add(a.st, DUM_CTR_WALK_OUT, qlen);
        ctr_add(a.st, DUM_CTR_WALK_PREFIX, 1);
      }
    }
    __syncthreads();  // the next item reuses the shared state
  }
  nsets = __reduce_add_sync(0xffffffffu, nsets);
  if (lane == 0 && nsets) atomicAdd(&s_sets, nsets);
  __syncthreads();
  if (tid == 0 && s_sets) ctr_add(a.st, DUM_CTR_SETS, s_sets);
}

// ---------------------------------------------------------------------------
// k_walk
// ---------------------------------------------------------------------------
// Parallel WALK(e, NONE) after the build (D13).  Let C = the latest faulting
// launch of e in this batch (deduplicated, n = |C|); then Start = C[0], End =
// C[n-1] (D11).  After the build, the row of C[i] (if still present) has
// C[i+1] as its MRU successor: INSERT(C[i] -> C[i+1]) was the last operation
// on that row, because C is duplicate-free and no later launch of e is in the
// batch.  C[i+1] is not among the chained nodes C[0..i], so the sequential
// walk's next chain node is exactly C[i+1] until the first i at which the row
// is missing or a successor equals End.  With t that index, the walk is the
// first-occurrence dedupe of
//   Q = [C[0]] ++ succ(row C[0]) ++ ... ++ succ(row C[t])   (row C[t] only if
//                                                            present).
// The speculation is still verified (succ[0] == C[i+1]); any violation sends e
// to the sequential walker.
//
// Pass A reads the rows of C from the table into a row cache (shared memory,
// or a global scratch for long walks); pass B places the rows' successor
// lists in Q; a min-position hash keeps first occurrences; pass C compacts
// them in order and groups them into bitmap runs for k_predict.
template <int MAXA, int MAXS>
__global__ void __launch_bounds__(WK_NT) k_walk(BuildArgs a) {
  extern __shared__ uint32_t sm[];
  __shared__ uint32_t ws[WK_NT / 32];
  __shared__ uint32_t s_tev, s_flag, s_off, s_nrun, s_multi;
  uint32_t *src = sm, *scq = sm + WK_RC, *sqk = scq + WK_CQ;  // row cache | chain positions | hash
  const Geo &g = a.g;
  const uint32_t tid = threadIdx.x;
  const uint32_t A = g.A, S = g.S;
  // one CTA per exec ID; the grid is the host's upper bound (staged launches)
  if (blockIdx.x == 0 && tid < 4) a.st->cls_cnt[tid] = 0;  // k_plan has read them; zero for the next build
  // persistent over the walks k_build_exec could not prove to be a prefix of
  // the latest launch (dd_list), grid sized by occupancy
  const uint32_t n_dd = *(volatile uint32_t *)&a.st->n_dd;
  for (uint32_t xi = blockIdx.x; xi < n_dd; xi += gridDim.x) {
  const uint32_t li = a.dd_list[xi];
  do {  // (breaks = the early ends of the walk)
    const LeadDesc d = a.desc[li];
    const uint32_t e = d.e;
    const uint32_t n = d.n_last;
    const uint64_t off = d.off_last;
    const uint32_t *C = a.stage_norm + off;
    const uint32_t start = C[0], end = C[n - 1];
    if (tid == 0) {
      a.start_end[2 * e] = start;
      a.start_end[2 * e + 1] = end;
      ctr_add(a.st, DUM_CTR_EXEC_BUILT, 1);
      ctr_add(a.st, DUM_CTR_OPS, d.n_ops);
      // the group bookkeeping of this batch is consumed (prep, plan and apply are done)
      a.head[e] = NONE;
      a.e_ops[e] = 0;
      a.e_last[e] = 0;
      s_tev = NONE;
      s_nrun = 0;
      s_multi = NONE;
    }
    uint32_t *wout = a.walk + (uint64_t)e * g.walk_cap;
    uint2 *wrun = reinterpret_cast<uint2 *>(a.wrun) + (uint64_t)e * g.walk_cap;
    if (a.seq_walks && n > 1) {  // DUM_CFG_SEQ_WALKS: the sequential walker builds every walk
      if (tid == 0) a.slow_list[atomicAdd(&a.st->n_slow, 1u)] = e;
      break;
    }
    if (n == 1) {  // x == End: the walk is [Start]
      if (tid == 0) {
        wout[0] = start;
        a.walk_len[e] = 1;
        wrun[0] = make_uint2(start >> 5, 1u << (start & 31));
        a.wrun_len[e] = 1;
        ctr_add(a.st, DUM_CTR_WALK_OUT, 1);
        ctr_add(a.st, DUM_CTR_WALK_PREFIX, 1);
      }
      break;
    }
    // ---- scratch: shared memory, else the global pools ----
    const uint32_t rw = 1 + S;
    uint32_t *rc = n * rw <= WK_RC ? src : a.rowc + off * rw;
    uint32_t *cq = scq;
    if (n > WK_CQ) {
      if (tid == 0) {
        const unsigned long long o = atomicAdd(&a.st->pool_bigb, (unsigned long long)n);
        s_flag = o + n <= a.big_entries * 2 ? 0u : 1u;
        s_off = (uint32_t)o;
      }
      __syncthreads();
      if (s_flag) {
        if (tid == 0) a.slow_list[atomicAdd(&a.st->n_slow, 1u)] = e;
        break;
      }
      cq = a.big_pool + s_off;
    }
    __syncthreads();
    // ---- pass A: rows of C[0 .. n-2] -> row cache; stop events ----
    const uint32_t *tbl_e = a.tbl + (uint64_t)e * g.R * g.stride;
    constexpr int WB = (MAXA * (1 + MAXS) <= 10) ? 4 : 1;  // rows per thread in flight
    for (uint32_t i0 = tid; i0 < n - 1; i0 += WK_NT * WB) {
      uint32_t x[WB], xn[WB];
      RegSet<MAXA, MAXS> rs[WB];
#pragma unroll
      for (int q = 0; q < WB; ++q) {  // issue every load of the batch first
        const uint32_t i = i0 + q * WK_NT;
        x[q] = i < n - 1 ? C[i] : NONE;
        xn[q] = i < n - 1 ? C[i + 1] : NONE;
      }
#pragma unroll
      for (int q = 0; q < WB; ++q)
        if (x[q] != NONE) rs[q].load(tbl_e + (uint64_t)row_of(g, x[q]) * g.stride, A, S);
#pragma unroll
      for (int q = 0; q < WB; ++q) {
        if (x[q] == NONE) continue;
        const uint32_t i = i0 + q * WK_NT;
        uint32_t *row = rc + i * rw;
        rs[q].export_row(x[q], A, S, row);
        const uint32_t cnt = row[0];
        uint32_t ev = 0;
        if (cnt == NONE) {
          ev = 1;  // row missing: stop, nothing emitted at this step
          cq[i] = 0;
        } else {
          bool hit = false;
          for (uint32_t k = 0; k < cnt; ++k) hit |= row[1 + k] == end;
          if (hit) ev = 2;                              // a successor is End: stop after emitting
          else if (cnt == 0 || row[1] != xn[q]) ev = 3;  // speculation violated -> sequential walker
          cq[i] = cnt;
          if (cnt > 1) atomicMin(&s_multi, i);
        }
        if (ev) atomicMin(&s_tev, (i << 2) | ev);
      }
    }
    __syncthreads();
    const uint32_t tev = s_tev;
    const uint32_t t = tev >> 2;
    if (tev == NONE || (tev & 3) == 3 || !GUARD(a.st, t + 1 < n, t)) {
      if (tid == 0) a.slow_list[atomicAdd(&a.st->n_slow, 1u)] = e;
      break;
    }
    if (s_multi > t) {
      // ---- fast path: rows C[0..t] have the single successor C[i+1], so Q =
      // C[0 .. t+1] (t+1 only when a successor is End), duplicate-free ----
      const uint32_t qlen = t + 1 + ((tev & 3) == 2 ? 1u : 0u);
      constexpr uint32_t FB = 4;  // steps with their loads in flight together
      for (uint32_t c00 = 0; c00 < qlen; c00 += WK_NT * FB) {
       uint32_t vals[FB];
#pragma unroll
       for (uint32_t u = 0; u < FB; ++u) {
         const uint32_t p = c00 + u * WK_NT + tid;
         vals[u] = p < qlen ? C[p] : NONE;
       }
#pragma unroll
       for (uint32_t u = 0; u < FB; ++u) {
        const uint32_t c0 = c00 + u * WK_NT;
        if (c0 >= qlen) break;  // uniform
        const uint32_t p = c0 + tid;
        const bool keep = p < qlen;
        const uint32_t val = vals[u];
        if (keep && p < g.walk_cap) wout[p] = val;
        const uint32_t lane = tid & 31;
        const uint32_t wkey = keep ? val >> 5 : NONE;
        const uint32_t gm = __match_any_sync(0xffffffffu, wkey);
        const uint32_t msk = __reduce_or_sync(gm, keep ? 1u << (val & 31) : 0u);
        const bool lead = keep && lane == (uint32_t)(__ffs(gm) - 1);
        const uint32_t lm = __ballot_sync(0xffffffffu, lead);
        uint32_t rb = 0;
        if (lane == 0 && lm) rb = atomicAdd(&s_nrun, (uint32_t)__popc(lm));
        rb = __shfl_sync(0xffffffffu, rb, 0) + __popc(lm & ((1u << lane) - 1));
        if (lead && rb < g.walk_cap) wrun[rb] = make_uint2(wkey, msk);
       }
      }
      __syncthreads();
      if (tid == 0) {
        if (qlen > g.walk_cap) set_err(a.st, ERR_ECAPACITY, qlen);
        a.walk_len[e] = qlen;
        a.wrun_len[e] = s_nrun;
        ctr_add(a.st, DUM_CTR_WALK_ROWS, t + 1);
        ctr_add(a.st, DUM_CTR_WALK_OUT, qlen);
        ctr_add(a.st, DUM_CTR_WALK_PREFIX, 1);
      }
      break;
    }
    // ---- pass B: Q positions (qpos[i] = 1 + sum cq[0..i)) in place ----
    uint32_t run = 1;
    for (uint32_t c0 = 0; c0 <= t; c0 += WK_NT) {
      const uint32_t i = c0 + tid;
      const uint32_t v = i <= t ? cq[i] : 0;
      uint32_t tot;
      const uint32_t pre = block_excl_scan(v, ws, &tot);
      if (i <= t) cq[i] = run + pre;
      run += tot;
    }
    const uint32_t qlen = run;  // |Q|
    if (!GUARD(a.st, qlen <= 1 + (t + 1) * S, qlen)) {
      if (tid == 0) a.slow_list[atomicAdd(&a.st->n_slow, 1u)] = e;
      break;
    }
    // ---- dedupe map block -> min Q position ----
    const uint32_t qcap = pow2ceil(2 * qlen);
    uint32_t *qk = sqk;
    if (qcap > WK_QCAP) {
      if (tid == 0) {
        const unsigned long long o = atomicAdd(&a.st->pool_bigb, 2ull * qcap);
        s_flag = o + 2ull * qcap <= a.big_entries * 2 ? 0u : 1u;
        s_off = (uint32_t)o;
      }
      __syncthreads();
      if (s_flag) {
        if (tid == 0) a.slow_list[atomicAdd(&a.st->n_slow, 1u)] = e;
        break;
      }
      qk = a.big_pool + s_off;
    }
    uint32_t *qv = qk + qcap;
    for (uint32_t p = tid; p < qcap; p += WK_NT) {
      qk[p] = NONE;
      qv[p] = NONE;
    }
    __syncthreads();
    if (tid == 0) hmap_insert_min(qk, qv, qcap, start, 0);
    for (uint32_t i = tid; i <= t; i += WK_NT) {
      const uint32_t q0 = cq[i];
      const uint32_t qn = (i < t ? cq[i + 1] : qlen) - q0;
      const uint32_t *sc = rc + i * rw + 1;
      for (uint32_t q = 0; q < qn; ++q) hmap_insert_min(qk, qv, qcap, sc[q], q0 + q);
    }
    __syncthreads();
    // ---- pass C: ordered compaction of first occurrences + bitmap runs ----
    // The kept blocks of each warp step are grouped by bitmap word into runs
    // (word, mask) for k_predict (any grouping that puts every block in exactly
    // one run will do; runs of one walk are disjoint).
    uint32_t outn = 0;
    for (uint32_t c0 = 0; c0 < qlen; c0 += WK_NT) {
      const uint32_t p = c0 + tid;
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
          const uint32_t *row = rc + lo * rw;
          val = GUARD(a.st, row[0] != NONE && p - cq[lo] < row[0], (lo << 16) | (p - cq[lo])) ? row[1 + p - cq[lo]]
                                                                                            : start;
        }
        keep = hmap_get(qk, qv, qcap, val) == p;
      }
      uint32_t tot;
      const uint32_t pre = block_excl_scan(keep, ws, &tot);
      if (keep && outn + pre < g.walk_cap) wout[outn + pre] = val;
      {
        const uint32_t lane = tid & 31;
        const uint32_t wkey = keep ? val >> 5 : NONE;
        const uint32_t gm = __match_any_sync(0xffffffffu, wkey);
        const uint32_t msk = __reduce_or_sync(gm, keep ? 1u << (val & 31) : 0u);
        const bool lead = keep && lane == (uint32_t)(__ffs(gm) - 1);
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
      ctr_add(a.st, DUM_CTR_WALK_DEDUPE, 1);
    }
  } while (false);
  __syncthreads();  // the next item reuses the shared state
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
      ctr_add(st, DUM_CTR_WALK_SLOW, 1);
    }
    __syncwarp();
    // bitmap runs of the new walk (see pass C of k_walk)
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
static cudaError_t launch_apply_walk(dum_engine *e, const BuildArgs &ba, cudaStream_t s) {
  const size_t wsmem = (size_t)(WK_RC + WK_CQ + 2 * WK_QCAP) * 4;
  const size_t bsmem = (size_t)(e->g.R + 4 * BX_RC) * 4;
  // the attributes are per device and function: raised by every engine on its own device;
  // persistent grids: resident CTAs per SM x SMs (the item counts are on the device)
  if (!e->build_smem) {
    cudaFuncSetAttribute(k_walk<MA, MS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)wsmem);
    cudaFuncSetAttribute(k_build_exec<MA, MS>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)bsmem);
    e->build_smem = (int)std::max(wsmem, bsmem);
    int dev = 0, sms = 148, nb = 1, nw = 1;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_build_exec<MA, MS>, BX_NT, bsmem);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nw, k_walk<MA, MS>, WK_NT, wsmem);
    e->apply_grid = (uint32_t)std::max(1, nb * sms);
    e->walk_grid = (uint32_t)std::max(1, std::min(nw * sms, 2 * sms));
  }
  {
    TimerScope t(e, DUM_T_APPLY_WALK, s);
    k_build_exec<MA, MS><<<std::min(ba.n_staged, e->apply_grid), BX_NT, bsmem, s>>>(ba);
  }
  // the sequential walks (slow list) on the third side stream, beside the
  // parallel ones (dedupe list): disjoint exec IDs, separate scratch
  cudaEventRecord(e->ev_wslow_fork, s);
  cudaStreamWaitEvent(e->side3, e->ev_wslow_fork, 0);
  {
    WalkScratch ws{e->d_walk_seen, e->d_walk_chain, e->d_walk_tmp, e->walk_hash_cap,
                   e->g.walk_cap + e->g.R * e->g.A + 4};
    TimerScope t(e, DUM_T_WALK_SLOW, e->side3);
    k_walk_slow<<<e->n_walk_slots, 32, 0, e->side3>>>(e->g, e->d_tbl, e->d_start_end, ba.walk, ba.walk_len, ba.wrun,
                                                     ba.wrun_len, e->d_slow_list, ws, e->d_state);
  }
  cudaEventRecord(e->ev_wslow, e->side3);
  {
    TimerScope t(e, DUM_T_WALK, s);
    k_walk<MA, MS><<<std::min(ba.n_staged, e->walk_grid), WK_NT, wsmem, s>>>(ba);  // dd_list only
  }
  cudaStreamWaitEvent(s, e->ev_wslow, 0);
  return cudaGetLastError();
}

static BuildArgs build_args(dum_engine *e, uint32_t n) {
  BuildArgs ba;
  ba.g = e->g;
  ba.n_staged = n;
  ba.stage_exec = e->d_stage_exec;
  ba.stage_cnt = e->d_stage_cnt;
  ba.stage_norm = e->d_stage_norm;
  ba.stage_off = e->d_stage_off;
  ba.head = e->d_head;
  ba.next = e->d_next;
  ba.e_ops = e->d_e_ops;
  ba.e_last = e->d_e_last;
  ba.desc = reinterpret_cast<LeadDesc *>(e->d_lead);
  ba.items = reinterpret_cast<uint2 *>(e->d_items);
  ba.tbl = e->d_tbl;
  ba.start_end = e->d_start_end;
  ba.walk = e->d_walk_n;  // staged: k_walk_commit publishes them (the build may run beside predict)
  ba.walk_len = e->d_walk_len_n;
  ba.rowc = e->d_rowc;
  ba.big_pool = e->d_big_pool_b;
  ba.big_entries = e->big_pool_entries;
  ba.slow_list = e->d_slow_list;
  ba.wrun = e->d_wrun_n;
  ba.wrun_len = e->d_wrun_len_n;
  ba.order = e->d_order;
  ba.plan_agg = reinterpret_cast<unsigned long long *>(e->d_plan_agg);
  ba.st = e->d_state;
  ba.seq_walks = (e->cfg.flags & DUM_CFG_SEQ_WALKS) ? 1u : 0u;
  ba.dd_list = e->d_dd_list;
  return ba;
}

// The published walks of the exec IDs a build rebuilt: the build writes them
// to the staging arrays (d_*_n) -- possibly while the predict kernels of the
// same step still read the live walk cache -- and this copies them over once
// predict is done.  A CTA per rebuilt exec ID (the build's leads).
__global__ void __launch_bounds__(256) k_walk_commit(const LeadDesc *__restrict__ desc, const DevState *st,
                                                     uint32_t walk_cap, const uint32_t *__restrict__ walk_n,
                                                     const uint32_t *__restrict__ len_n,
                                                     const uint2 *__restrict__ wrun_n,
                                                     const uint32_t *__restrict__ rlen_n, uint32_t *walk,
                                                     uint32_t *len, uint2 *wrun, uint32_t *rlen) {
  const uint32_t n_leads = *(volatile const uint32_t *)&st->n_leads;
  for (uint32_t li = blockIdx.x; li < n_leads; li += gridDim.x) {
    const uint32_t e = desc[li].e;
    const uint32_t L = len_n[e], RL = rlen_n[e];
    const uint64_t r0 = (uint64_t)e * walk_cap;  // rows are 32 B aligned (walk_cap % 8 == 0)
    const uint4 *ws = reinterpret_cast<const uint4 *>(walk_n + r0);
    uint4 *wd = reinterpret_cast<uint4 *>(walk + r0);
    for (uint32_t i = threadIdx.x; i < (L + 3) / 4; i += blockDim.x) wd[i] = __ldcs(ws + i);
    const uint4 *rs = reinterpret_cast<const uint4 *>(wrun_n + r0);
    uint4 *rd = reinterpret_cast<uint4 *>(wrun + r0);
    for (uint32_t i = threadIdx.x; i < (RL + 1) / 2; i += blockDim.x) rd[i] = __ldcs(rs + i);
    if (threadIdx.x == 0) {
      len[e] = L;
      rlen[e] = RL;
    }
  }
}

cudaError_t launch_walk_commit(dum_engine *e, cudaStream_t s) {
  TimerScope t(e, DUM_T_COMMIT, s);
  k_walk_commit<<<std::max<uint32_t>(1, std::min<uint32_t>(e->g.Emax, 148 * 8)), 256, 0, s>>>(
      reinterpret_cast<const LeadDesc *>(e->d_lead), e->d_state, e->g.walk_cap, e->d_walk_n, e->d_walk_len_n,
      reinterpret_cast<const uint2 *>(e->d_wrun_n), e->d_wrun_len_n, e->d_walk, e->d_walk_len,
      reinterpret_cast<uint2 *>(e->d_wrun), e->d_wrun_len);
  e->commit_stale = false;
  e->kernel_launches += 1;
  return cudaGetLastError();
}

// The build of the n staged launches into the staging walk arrays: the head
// (correlation upserts + work lists, k_build_prep / k_plan; the jump tables
// forked to the side stream), the table apply + walks (k_build_exec, k_walk)
// and the sequential walks (k_walk_slow), all on `s`.  Everything it writes
// is read by the next predict only through k_chain (corr / jump, already
// read) or after k_walk_commit (walks), so it may run beside this step's
// predict kernels (D12 holds: predict reads the walks of the last build).
static cudaError_t build_body(dum_engine *e, const BuildArgs &ba, cudaStream_t s) {
  const uint32_t n = ba.n_staged;
  {
    TimerScope t(e, DUM_T_BUILD_PREP, s);
    k_build_prep<<<(n + 255) / 256, 256, 0, s>>>(n, e->d_stage_exec, e->d_stage_cnt,
                                                  e->d_corr, e->corr_cap, e->d_rec_slot, e->d_head, e->d_next,
                                                  e->d_order, e->d_e_ops, e->d_e_last, ba.plan_agg, e->d_state);
    k_plan<<<(n + PLAN_NT - 1) / PLAN_NT, PLAN_NT, 0, s>>>(ba);
  }
  // the jump tables depend only on the correlation table, final here; a
  // captured step leaves them to the start of the next step (beside its
  // ingest) instead of joining them at its end
  cudaError_t err = cudaSuccess;
  if (e->capturing) {
    e->jump_stale = true;
  } else {
    cudaEventRecord(e->ev_fork, s);
    cudaStreamWaitEvent(e->side, e->ev_fork, 0);
    err = launch_jump_tables(e, e->side);
    cudaEventRecord(e->ev_join, e->side);
    e->jump_stale = false;
    if (err != cudaSuccess) return err;
  }
  if (e->g.A <= 2 && e->g.S <= 4) err = launch_apply_walk<2, 4>(e, ba, s);
  else if (e->g.A == 2 && e->g.S == 8) err = launch_apply_walk<2, 8>(e, ba, s);
  else if (e->g.A == 4 && e->g.S == 4) err = launch_apply_walk<4, 4>(e, ba, s);
  else if (e->g.A <= 4 && e->g.S <= 8) err = launch_apply_walk<4, 8>(e, ba, s);
  else err = launch_apply_walk<32, 32>(e, ba, s);
  if (err != cudaSuccess) return err;
  e->kernel_launches += 4;
  return cudaGetLastError();
}

// dum_step: the build of the n staged launches, issued by launch_predict right
// after k_chain (the last reader of the correlation and jump tables) on a
// high-priority side stream beside the predict kernels; launch_build (after
// predict) waits for it and publishes the walks.
cudaError_t launch_build_head(dum_engine *e, uint32_t n, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  cudaEventRecord(e->ev_fork4, s);
  cudaStreamWaitEvent(e->side4, e->ev_fork4, 0);
  const BuildArgs ba = build_args(e, n);
  const cudaError_t err = build_body(e, ba, e->side4);
  cudaEventRecord(e->ev_bhead, e->side4);
  e->bhead_pending = true;
  return err;
}

cudaError_t launch_build(dum_engine *e, cudaStream_t s) {
  const uint32_t n = e->n_staged;
  if (n == 0) return cudaSuccess;
  if (e->commit_inflight && !e->capturing) {  // the last commit still reads the staging arrays
    cudaStreamWaitEvent(s, e->ev_commit, 0);
    e->commit_inflight = false;
  }
  if (!e->capturing) {  // (a captured step joins its side streams before it ends)
    cudaStreamWaitEvent(s, e->ev_join, 0);  // the previous build's jump tables read corr
    cudaStreamWaitEvent(s, e->ev_widx, 0);  // the previous build's walk index reads the walk cache
  }
  if (e->bhead_pending) {  // built beside the predict kernels (launch_build_head)
    cudaStreamWaitEvent(s, e->ev_bhead, 0);
    e->bhead_pending = false;
  } else {
    // the staging arrays still hold the last replayed build's unpublished walks
    if (!e->capturing && e->commit_stale) {
      const cudaError_t ce = launch_walk_commit(e, s);
      if (ce != cudaSuccess) return ce;
    }
    const BuildArgs ba = build_args(e, n);
    const cudaError_t be = build_body(e, ba, s);
    if (be != cudaSuccess) return be;
  }
  if (e->capturing && !e->fast_windows) {
    // a captured step publishes its walks at the start of the next step, beside
    // its ingest (before k_chain, their first reader)
    e->commit_stale = true;
  } else if (!e->capturing && !e->fast_windows) {
    // publish the rebuilt walks beside the next step's residency load and
    // ingest (side stream): their readers -- the next predict, the next build
    // (staging) -- wait for ev_commit
    cudaEventRecord(e->ev_fork4, s);
    cudaStreamWaitEvent(e->side4, e->ev_fork4, 0);
    const cudaError_t ce = launch_walk_commit(e, e->side4);
    if (ce != cudaSuccess) return ce;
    cudaEventRecord(e->ev_commit, e->side4);
    e->commit_inflight = true;
  } else {  // publish the rebuilt walks (the walk index below reads them)
    const cudaError_t ce = launch_walk_commit(e, s);
    if (ce != cudaSuccess) return ce;
  }
  if (e->capturing) {
    // a captured step builds the walk index at the start of the next step,
    // beside its ingest (dum_step graph); the next uncaptured predict does it
    e->widx_stale = true;
  } else {
    const cudaError_t we = launch_walk_index(e, s);  // k_window.cu: conflicts between the new walks
    if (we != cudaSuccess) return we;
  }
  // no join here: the jump tables keep building on the side stream, past the
  // end of this call; the next reader of the correlation table (predict's
  // k_chain, the next build, reset) waits for ev_join
  e->kernel_launches += 1;
  return cudaGetLastError();
}

}  // namespace dum
