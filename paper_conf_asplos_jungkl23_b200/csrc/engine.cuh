// Internal definitions of libdeepum_b200.so (not part of the C-ABI).
//
// HBM layout:
//   exec map     open-addressing u64 keys / u32 ids / u32 min-position, pow2
//                capacity >= 2 * max_exec_ids (+1 slot for the sentinel key)
//   exec_hash    u64[max_exec_ids]   hash of exec ID e (canonical dump)
//   corr         CorrSlot[corr_cap]  32 B: key {owner e, h1, h2, h3} (16 B,
//                claimed with a 128-bit CAS), max(k<<32|succ), min(k)
//   tbl          u32[E][R][stride]   set = A ways x (tag, S succ), MRU first,
//                                    NONE-padded; stride = A(1+S) rounded up to
//                                    a 32 B sector
//   start_end    u32[E][2]
//   walk         u32[E][walk_cap], walk_len u32[E]
//   walk runs    (word, mask) u32x2[E][walk_cap], wrun_len u32[E]: the walk
//                as bitmap words, consecutive blocks of one 32-block word merged
//   residency    frame_of u32[W], stamp_of u32[W], block_of u32[C],
//                free bitmap u32[C/32], inactive bitmap u32[W/32],
//                LRM log (blk u32, stamp u32)[log_cap] ordered by stamp
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>
#include <vector>

#include "../../include/deepum_b200.h"

namespace dum {

// enumerators (not constexpr variables) so that device code never odr-uses them
enum : uint32_t { NONE = 0xFFFFFFFFu, PENDING = 0xFFFFFFFEu, CLAIM = 0xFFFFFFFDu, CLAIM_DST = 0xFFFFFFFCu };
enum : unsigned long long { EMPTY64 = 0xFFFFFFFFFFFFFFFFull };

// sticky device error bits
enum : uint32_t {
  ERR_EINVAL = 1u,
  ERR_ECAPACITY = 2u,
};

struct __align__(32) CorrSlot {
  uint32_t key[4];      // owner, h1, h2, h3 ; owner == NONE -> empty
  unsigned long long last;   // max over observations of (k << 32 | succ)
  unsigned long long first;  // min over observations of k
};

// Device-resident engine scalars (one struct in device memory).
struct DevState {
  uint32_t E;                 // exec IDs assigned
  uint32_t hist[4];           // last four exec IDs applied by build, oldest first
  uint32_t err;               // sticky ERR_* bits
  unsigned long long needed;  // largest capacity a failed call required
  unsigned long long pool_pairs;   // predict output bump pointer
  unsigned long long pool_wb, pool_inv;
  unsigned long long pool_anchor;  // anchored-walk scratch bump pointer
  unsigned long long pool_big;     // exact-predict global hash scratch bump pointer (d_big_pool)
  unsigned long long pool_bigb;    // build-walk global hash scratch bump pointer (d_big_pool_b)
  unsigned long long pool_chunks;  // predict: k_copy_fast chunk-map bump pointer
  uint32_t sel_queue;         // predict: k_window_fast selection-item queue head
  unsigned long long copy_queue;  // predict: k_window_fast copy-chunk queue head
  uint32_t n_slow;            // exec IDs queued for the sequential walk
  uint32_t n_pend;            // record: launches with a hash first seen in the batch (k_ingest -> k_exec_assign)
  uint32_t free_count;        // free HBM frames
  uint32_t mig_counter;       // next migration stamp (D19)
  uint32_t lrm_head, lrm_tail;// LRM log [head, tail)
  uint32_t n_resident;
  uint32_t corr_used;
  uint32_t mig_ok;            // last migrate validated
  uint32_t mig_n;             // blocks moved by the last migrate
  uint32_t log_dirty;         // LRM log may hold entries of evicted blocks
  uint32_t dbg_line, dbg_val; // first failed internal guard (GUARD macro)
  uint32_t cls_cnt[4];        // build: faulting launches per size class
  uint32_t q_cls[16];         // predict: queries per (fast/exact, window-size) class (k_chain)
  uint32_t n_fast;            // predict: queries answered by k_window (the first n_fast of qperm)
  uint32_t chain_done;        // predict: k_chain CTAs finished
  uint32_t n_items, n_leads;  // build: k_apply items / exec IDs with faults (k_plan)
  uint32_t n_dd;              // build: walks left to k_walk's dedupe (k_build_exec)
  uint32_t counting;          // ctr_add is live (dum_set_counting)
  uint32_t k_base;            // global launch index of the next build's first staged launch
  unsigned long long ctr[DUM_NCOUNTERS];  // work counters (instrumentation)
};

struct Geo {
  uint32_t R, A, S, N, W, C, Emax;
  uint32_t row_index;
  uint32_t set_u32;     // A * (1 + S)
  uint32_t stride;      // set stride in u32 (multiple of 8)
  uint32_t walk_cap;    // per-exec walk capacity
};

__host__ __device__ inline uint32_t fmix32(uint32_t h) {
  h ^= h >> 16;
  h *= 0x85ebca6bu;
  h ^= h >> 13;
  h *= 0xc2b2ae35u;
  h ^= h >> 16;
  return h;
}
__host__ __device__ inline uint64_t fmix64(uint64_t k) {
  k ^= k >> 33;
  k *= 0xff51afd7ed558ccdull;
  k ^= k >> 33;
  k *= 0xc4ceb9fe1a85ec53ull;
  k ^= k >> 33;
  return k;
}
__host__ __device__ inline uint32_t row_of(const Geo &g, uint32_t b) {
  return (g.row_index ? fmix32(b) : b) & (g.R - 1);
}

__device__ __forceinline__ void ctr_add(DevState *st, int c, unsigned long long v) {
#ifdef __CUDA_ARCH__
  // `counting` only changes between calls (dum_set_counting synchronizes): a
  // read-only-cache load, no L2 round trip per call site
  if (v && __ldg(&st->counting)) atomicAdd(&st->ctr[c], v);
#endif
}

}  // namespace dum

struct dum_engine;
namespace dum {
// RAII event pair around a kernel launch when timing is enabled.
struct TimerScope {
  dum_engine *e;
  int id;
  cudaStream_t s;
  cudaEvent_t b;
  TimerScope(dum_engine *e_, int id_, cudaStream_t s_);
  ~TimerScope();
};
}  // namespace dum

struct dum_engine {
  dum_config cfg;
  dum::Geo g;
  int device;
  // exec map
  uint32_t exec_cap;   // pow2; slot exec_cap is the sentinel-key slot
  unsigned long long *d_exec_keys;
  uint32_t *d_exec_vals, *d_exec_minpos;
  uint64_t *d_exec_hash;
  // corr
  uint32_t corr_cap;
  dum::CorrSlot *d_corr;
  uint32_t *d_rec_slot;   // [corr_cap] slots of the records in insertion order
  uint32_t *d_jump;       // [jump_levels][corr_cap] J_k = next^(2^k) over record slots (k_jump.cu)
  uint32_t jump_levels;
  cudaStream_t side;      // jump-table build runs here, overlapping the block-table apply
  cudaEvent_t ev_fork, ev_join;
  // block tables / walk cache
  uint32_t *d_tbl, *d_start_end, *d_walk, *d_walk_len;
  uint32_t *d_wrun, *d_wrun_len;   // walk as (word, mask) runs (k_walk / k_walk_slow)
  // staging
  uint32_t stage_launch_cap;
  uint64_t stage_fault_cap;
  uint64_t *d_in_hash, *d_in_off;   // host-pointer inputs are uploaded here (on rec_s), two sets
  // record_faults runs on its own stream so that the next batch's ingest
  // overlaps the current build; the staging arrays alternate between two sets
  cudaStream_t rec_s;
  cudaEvent_t ev_rec, ev_s_now, ev_stage_free[2];
  int stage_set;
  void *stage_base[6];              // the two-set allocations behind d_stage_*
  uint32_t *d_in_faults;
  uint64_t *d_stage_hash;
  uint32_t *d_stage_norm, *d_stage_cnt, *d_stage_exec, *d_stage_slot;
  uint32_t *d_pend;       // [stage_launch_cap] launches queued for k_exec_assign
  uint64_t *d_stage_off;  // offset of launch j's records in d_stage_norm
  uint32_t n_staged;
  uint64_t staged_faults;
  uint64_t launches;      // recorded since reset (global launch index base)
  uint64_t built_launches;
  // build scratch
  uint32_t *d_head, *d_next, *d_slow_list, *d_order;
  uint32_t *d_dd_list;           // k_build_exec -> k_walk: walks needing the dedupe
  uint32_t *d_e_ops, *d_e_last;  // per exec ID: group operations / latest launch of the batch
  uint64_t *d_plan_agg;          // k_plan look-back slots (one per 256 staged launches)
  uint32_t *d_lead;              // exec IDs with faults of the batch (k_build.cu LeadDesc, 32 B each)
  uint32_t *d_items;             // apply items, u32 pairs (leader index, partition | P << 16)
  uint64_t items_cap;
  uint32_t *d_rowc;              // walk row cache for long walks: (1 + S) u32 per staged record
  uint32_t *d_big_pool;   // u32 pairs for large-window hash tables (exact predict)
  uint32_t *d_big_pool_b; // the same for the build's large walks (the build may run beside predict)
  // the build writes the walks of the exec IDs it rebuilds here, beside the
  // predict kernels that read the live walk cache; k_walk_commit copies them
  // into the live arrays once predict is done (D12)
  uint32_t *d_walk_n, *d_walk_len_n, *d_wrun_n, *d_wrun_len_n;
  uint32_t *d_ingest_pool;  // the ingest's own global hash region (it may run concurrently with a build)
  uint64_t big_pool_entries;
  // walk scratch for the sequential walker (per CTA slot)
  uint32_t n_walk_slots;
  uint32_t walk_hash_cap; // pow2 per table
  uint32_t *d_walk_seen, *d_walk_chain, *d_walk_tmp, *d_walk_out;
  // predict anchored walks
  uint32_t *d_anchor_pool;
  uint64_t anchor_pool_entries;
  uint64_t *d_anchor_range;   // per query (begin, len)
  uint32_t anchor_range_cap;  // max queries per predict call
  uint32_t *d_qkern, *d_qloff, *d_qeoff, *d_qgoff, *d_qnk;
  uint32_t *d_qrank, *d_qperm;  // window-size class rank per query; predict CTA order (largest first)  // per-query chain scratch (k_chain -> k_predict)
  unsigned long long *d_qbase;
  // walk index (k_window.cu): holders per block, conflicts per walk (build
  // end); residency facts per walk (predict time); fast/exact split
  uint32_t *d_bcnt, *d_bhold;   // [W], [W][HOLD_MAX]
  uint32_t *d_conf, *d_conf_n;  // [Emax][CONF_MAX], [Emax] (NONE = not recorded)
  uint32_t *d_wnr, *d_wnres;    // [Emax] walk blocks without / with a frame
  uint32_t *d_respos;           // [Emax][walk_cap] log positions of the latter
  uint32_t *d_log_bits;         // [lrm_cap / 32 + 1] inactive log entries by position from head (k_log_bits)
  uint32_t *d_qroff, *d_qneed;  // [max queries][N+2], [max queries] (k_chain -> k_window)
  unsigned long long *d_qvb;    // [max queries][2] victim-range bases (k_chain -> k_window)
  uint4 *d_selrec;  // [NQCLS][max queries][3] k_window_fast selection records, k_chain's class order
  uint4 *d_chunk_map;  // [chunk_cap] copy chunks of the fast queries' windows: {exec, first, dst lo, dst hi | n << 16}
  uint64_t chunk_cap;
  cudaStream_t side2;           // exact-path predict kernel beside the fast path
  cudaEvent_t ev_fork2, ev_join2;
  cudaStream_t side3;           // walk index (build end)
  cudaStream_t side4;           // dum_step: the build's head (k_build_prep, k_plan) beside the predict kernels
  cudaEvent_t ev_fork4, ev_bhead;
  cudaEvent_t ev_wslow_fork, ev_wslow;  // the build's sequential walks beside its parallel ones (third side stream)
  uint32_t bhead_n;             // dum_step: launches whose build head launch_predict issues after k_chain
  bool bhead_pending;           // the head was issued early: launch_build waits for ev_bhead
  bool fast_windows;            // DUM_CFG_FAST_WINDOWS
  cudaEvent_t ev_widx;
  // dum_step: exec IDs [last 3 of the previous step | this batch] and the batch's queries
  uint32_t *d_step_exec;
  dum_query *d_step_q;
  // closed-loop replay scratch (k_sim.cu, allocated by the first dum_simulate)
  bool sim_ready;
  uint32_t sim_acc_cap;
  uint64_t sim_pair_cap;
  uint32_t *sim_acc_bits, *sim_faults, *sim_pairs, *sim_wb, *sim_inv, *sim_pf;
  uint64_t *sim_foff, *sim_ranges;
  dum_query *sim_q;
  // residency
  uint32_t *d_frame_of, *d_stamp_of, *d_block_of, *d_free_bits, *d_inactive_bits, *d_res_bits;
  uint32_t *d_lrm_blk, *d_lrm_stamp;   // LRM log: block | inactive << 31, migration stamp
  uint32_t *d_logpos;                  // log position of each resident block
  uint32_t lrm_cap;
  uint32_t *d_mig_frames;     // destination frames of the last migrate
  uint32_t *d_mig_src;        // source frames (D2D)
  uint32_t *d_mig_blocks;     // blocks of the last migrate
  uint32_t mig_cap;
  // data plane
  char *host_arena, *host_arena_dev, *frame_pool;
  // state
  dum::DevState *d_state;
  dum::DevState *h_state;     // pinned mirror for dum_sync / stats
  std::string last_error;
  uint64_t kernel_launches;
  // per-kernel event timing
  bool timing;
  struct TimedLaunch {
    int id;
    cudaEvent_t a, b;
  };
  std::vector<TimedLaunch> pending;
  std::vector<cudaEvent_t> event_pool;
  double t_ms[DUM_NTIMERS];
  uint64_t t_cnt[DUM_NTIMERS];
  int predict_smem, select_smem, build_smem, ingest_smem;
  uint32_t apply_grid, walk_grid;  // persistent build grids (occupancy x SMs), set on first build
  uint32_t copy_grid, sel_grid;  // persistent predict grids (k_window.cu)
  int chain_smem;                  // k_chain dynamic smem attribute applied
  int bulk_smem;                   // k_copy_bulk dynamic smem attribute applied
  uint32_t copy_sms;               // copy kernels: SMs' worth of CTAs (0 = all; dum_set_copy_sms)
  // dum_step as a replayed CUDA graph (dum_set_step_graphs)
  bool graph_steps, capturing, step_warm;
  cudaStream_t graph_s;        // the step graphs are captured and replayed here
  cudaEvent_t ev_graph, ev_wres;
  bool wres_pending;           // dum_step issued the walk residency facts beside the ingest
  bool cap_events_ready;
  bool widx_stale;             // the walk index lags the last (replayed) build
  bool jump_stale;             // the jump tables lag the last (captured / replayed) build
  bool commit_stale;           // the walks of the last (captured / replayed) build are not yet published
  cudaEvent_t ev_commit;       // an uncaptured build's walk commit (side stream); its readers wait for it
  bool commit_inflight;        // ev_commit not yet waited for by predict
  cudaEvent_t cap_ev[12];       // the fork / join events of a step-graph capture (graph edges only)
  struct StepGraph {
    uint64_t key[12];
    cudaGraphExec_t exec;
  };
  std::vector<StepGraph> step_graphs;  // dynamic smem attributes applied (per engine / device)
};

// this staging set's upload buffers for host-pointer / step inputs
inline uint64_t *in_hash(const dum_engine *e) { return e->d_in_hash + (uint64_t)e->stage_set * e->stage_launch_cap; }
inline uint64_t *in_off(const dum_engine *e) {
  return e->d_in_off + (uint64_t)e->stage_set * (e->stage_launch_cap + 1ull);
}
inline uint32_t *in_faults(const dum_engine *e) { return e->d_in_faults + (uint64_t)e->stage_set * e->stage_fault_cap; }
