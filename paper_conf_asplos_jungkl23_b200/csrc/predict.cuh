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
constexpr int WSEL_NT = 256;        // k_window_fast threads
constexpr uint32_t POS_WORDS = 1024;  // k_window position bitmap: log positions [head, head + 32768)

struct PredArgs {
  Geo g;
  const dum_query *q;
  uint32_t nq;
  uint32_t select;       // a8 fused (dum_predict_select)
  uint32_t chain_bitset; // k_chain tests conflicts against a shared bitset of the chain
  uint32_t fast;         // DUM_CFG_FAST_WINDOWS: conflict-free windows take k_window_fast
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
  // k_window_fast: per fast query (class order, like qperm) a 48 B record
  //   {qi, nk, need, nw}, {-, ok, -, -}, {wb base, inv base}
  uint4 *selrec;
  uint32_t lrm_cap;  // LRM log entries allocated (k_window_fast clamps its bulk loads to it)
  uint4 *chunk_map;  // [chunk_cap] copy chunks of the fast queries (k_chain -> k_copy_fast):
                    // {exec ID, first list entry, pair slot lo 32, pair slot hi 16 | entries << 16}
  uint64_t chunk_cap;
  unsigned long long *qbase;  // [nq]
  uint32_t *big_pool;         // scratch for the exact slow path
  uint64_t big_entries;
  SelectOut so;     // fused a8 outputs (SELECT only)
  uint64_t *needed;             // pair-pool size after every reservation (k_chain's last CTA), or null
};

cudaError_t launch_walk_index(dum_engine *e, cudaStream_t s);
cudaError_t launch_walk_res(dum_engine *e, cudaStream_t s);
cudaError_t launch_window(dum_engine *e, const PredArgs &a, bool select, cudaStream_t s);

}  // namespace dum
