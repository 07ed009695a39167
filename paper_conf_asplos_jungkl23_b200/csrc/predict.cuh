// Shared definitions of the prefetch-window kernels (k_predict.cu: k_chain and
// the exact kernel k_predict; k_window.cu: the conflict-free fast path).
#pragma once
#include "device_util.cuh"
#include "kernels.cuh"
#include "select_tail.cuh"

namespace dum {

constexpr uint32_t MAXN = 128;      // degree_n limit
constexpr int NQCLS = 5;            // window-size classes of k_chain's query order
constexpr uint32_t HOLD_MAX = 64;   // walk index: holders recorded per block
constexpr uint32_t CONF_MAX = 64;   // walk index: conflicting exec IDs recorded per walk
constexpr uint32_t CHUNK_B = 128;   // window blocks per copy chunk (one warp: 4 coalesced steps)
constexpr int COPY_NT = 256;        // k_copy_fast threads
constexpr int WSEL_NT = 256;        // k_select_fast threads
constexpr int WSEL_IT = 8;          // k_select_fast: log entries per thread per selection chunk
constexpr uint32_t POS_WORDS = 1024;  // k_window position bitmap: log positions [head, head + 32768)

struct PredArgs {
  Geo g;
  const dum_query *q;
  uint32_t nq;
  uint32_t select;       // a8 fused (dum_predict_select)
  uint32_t chain_bitset; // k_chain tests conflicts against a shared bitset of the chain
  const CorrSlot *corr;
  uint32_t corr_cap;
  const uint32_t *jump;  // [levels][corr_cap]
  const uint32_t *walk, *walk_len;
  const uint32_t *wrun, *wrun_len;  // walk bitmap runs (k_walk pass C / k_walk_slow)
  const uint32_t *anchor_pool;
  const uint64_t *anchor_range;
  uint32_t *pairs;
  uint64_t cap;
  uint64_t *range;
  uint32_t *kern_off, *chain;
  DevState *st;
  uint32_t nwords;  // bitmap words
  // walk index (k_window.cu): conflicts per walk; residency facts per walk
  const uint32_t *conf, *conf_n;
  const uint32_t *wnr, *wnres, *respos;
  const uint32_t *inact_bits;  // the LRM log's inactive entries by position from head (k_log_bits), or null
  // per-query scratch written by k_chain
  uint32_t *qkern;  // [nq][N+1]
  uint32_t *qloff;  // [nq][N+2]
  uint32_t *qeoff;  // [nq][N+2] run-entry offsets of the window's lists
  uint32_t *qgoff;  // [nq][N+2] 128-block copy-chunk offsets of the window's lists
  uint32_t *qnk;    // [nq]
  uint32_t *qrank;  // [nq] class << 24 | rank within the class
  uint32_t *qperm;  // [2 NQCLS][nq] class lists of k_chain: fast classes, then the exact-path ones
  uint32_t *qroff;    // [nq][N+2] prefix of the lists' resident blocks (fast queries, select)
  uint32_t *qneed;    // [nq] victims to find (fast queries, select)
  unsigned long long *qvb;  // [nq][2] reserved write-back / invalidate offsets (fast queries, select)
  unsigned long long *chunk_map;  // [chunk_cap] copy chunks of the fast queries (k_chain -> k_copy_fast)
  uint64_t chunk_cap;
  unsigned long long *qbase;  // [nq]
  uint32_t *big_pool;         // scratch for the exact slow path
  uint64_t big_entries;
  SelectOut so;     // fused a8 outputs (SELECT only)
  uint64_t *needed;             // pair-pool size after every reservation (k_chain's last CTA), or null
};

// Stream the window's lists (cached walks, no anchor) as (block, exec) pairs:
// flat over the window's 128-block chunks (chunks never straddle lists);
// warp-uniform chunk lookup, lane-consecutive 4 B loads and 8 B streaming
// stores, two chunks in flight per warp.  List d goes to pairs[base +
// oofs[d] ...].  Called by the warps cw = 0 .. ncw-1 of a group.
__device__ __forceinline__ void copy_window_lists(const PredArgs &a, const uint32_t *kern, const uint32_t *loff,
                                                  const uint32_t *goff, uint32_t nk, unsigned long long base,
                                                  uint32_t cw, uint32_t ncw, const uint32_t *oofs,
                                                  const uint32_t *skip) {
  constexpr uint32_t UN = 2;
  const uint32_t lane = threadIdx.x & 31;
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
        const uint32_t *lst = a.walk + (uint64_t)kern[lo] * a.g.walk_cap;
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
}

cudaError_t launch_walk_index(dum_engine *e, cudaStream_t s);
cudaError_t launch_walk_res(dum_engine *e, cudaStream_t s);
cudaError_t launch_window(dum_engine *e, const PredArgs &a, bool select, cudaStream_t s);

}  // namespace dum
