/*
 * include/deepum_b200.h -- C-ABI of the B200-native DeepUM correlation-prefetch
 * and tensor-migration engine (libdeepum_b200.so).
 *
 * The five calls of the hot path follow the paper's statement of the problem
 * (DeepUM, Jung, Kim and Lee, ASPLOS '23; "P:Lnnn" = /root/reference/PAPER.md
 * line nnn):
 *
 *   dum_record_faults     a1+a2  fault records grouped per kernel launch, the
 *                                launch's exec ID from the hash of its name and
 *                                arguments (P:L124 step 2)
 *   dum_build_tables      a3-a6  execution ID correlation table (P:L176,
 *                                P:L208-L210), per-exec-ID set-associative UM
 *                                block correlation tables with Start/End
 *                                (P:L164-L174), walk cache
 *   dum_predict_prefetch  a7     chained prefetch window of the current kernel
 *                                plus the next N predicted kernels, as
 *                                (block, exec ID) commands
 *   dum_select_evictions  a8     pre-eviction victims: least recently migrated
 *                                and not in the window; split into write-back
 *                                and invalidate by PT-block inactivity
 *
 *   dum_migrate_blocks    a9     batched 2 MiB block moves between pinned host
 *                                memory and HBM (P:L124 steps 4-7), plus
 *                                HBM->HBM compaction
 *
 * Semantics where the paper is silent follow the readings D1-D22 listed in
 * DESIGN.md ("Readings").  Every state-changing call is bit-exact with the
 * sequential CPU oracle in oracle/ (tests/test_gpu_parity.py).
 *
 * Conventions (all calls):
 *   - Return 0 (DUM_OK) or a negative DUM_E* code; dum_last_error() has text.
 *   - All calls are asynchronous and stream-ordered on the given CUDA stream
 *     (cudaStream_t passed as dum_stream_t), except dum_create, dum_destroy,
 *     dum_dump_state, dum_sync, dum_get_stats, dum_read_counters,
 *     dum_read_timing and dum_migrate_blocks with method 2 (copy engines:
 *     the frame plan is read back to the host before the copies are
 *     issued), which synchronize.
 *   - Ownership: the caller owns every input/output buffer and must keep it
 *     valid until the stream work completes; the engine owns all tables,
 *     residency state and scratch (device memory on cfg.device).
 *   - Pointers are device pointers unless a call says otherwise.  With
 *     DUM_HOST_PTRS, dum_record_faults copies host inputs to the device itself.
 *   - Errors detected on the device (a block id >= max_blocks, an exceeded
 *     capacity) are sticky; dum_sync() returns them (and the required capacity
 *     through *needed).  Outputs of a call that raised DUM_ECAPACITY on the
 *     device are unspecified.
 *   - Identifiers: UM block ids are uint32 in [0, max_blocks) (block =
 *     (va - um_base) >> 21, D1); exec IDs are dense uint32 from 0 in
 *     first-seen order (D3); DUM_NONE = 0xFFFFFFFF marks absence.
 *   - Thread safety: one engine per host thread; engines share nothing.
 */
#ifndef DEEPUM_B200_H
#define DEEPUM_B200_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct dum_engine dum_engine;
typedef struct CUstream_st *dum_stream_t; /* == cudaStream_t */

#define DUM_NONE 0xFFFFFFFFu
#define DUM_BLOCK_BYTES (2ull << 20) /* 4 KB x 512 pages */

enum {
  DUM_OK = 0,
  DUM_EINVAL = -1,    /* bad geometry / argument / alignment / block id */
  DUM_ECAPACITY = -2, /* an output or engine capacity is too small */
  DUM_ENOMEM = -3,
  DUM_ECUDA = -4,
  DUM_ESTATE = -5     /* call not valid in the engine's current state */
};

/* flags */
#define DUM_HOST_PTRS 0x1u /* dum_record_faults: inputs are host pointers */
#define DUM_INPUTS_READY 0x2u /* dum_record_faults: the device inputs do not depend on work
                                 queued on `stream` (the ingest may start before it) */

typedef struct {
  /* UM block correlation table geometry, Table 6;
   * default Config9 = 2048 rows, 2-way, 4 successors.
   * num_rows: power of two <= 8192; assoc <= 32; num_succs <= 32. */
  uint32_t num_rows, assoc, num_succs;
  /* degree of prefetching N: window = current + next N kernels (P:L224,
   * P:L465; default 32) */
  uint32_t degree_n;           /* <= 128 */
  uint32_t max_blocks;         /* W: block-id space; <= 2^20 (window bitmaps) */
  uint32_t max_exec_ids;       /* table capacity; DUM_ECAPACITY beyond */
  uint32_t hbm_frames;         /* C: HBM capacity in 2 MiB frames */
  uint32_t row_index;          /* 0 = low bits b & (R-1) (D7), 1 = fmix32 */
  uint32_t max_batch_launches; /* staging capacity between build calls (0 = 65536) */
  uint64_t max_batch_faults;   /* staging capacity in fault records (0 = 16 Mi) */
  uint32_t corr_capacity;      /* exec-correlation records (0 = 16 * max_exec_ids) */
  int device;                  /* CUDA device ordinal */
  /* Data plane (optional; NULL = metadata-only engine, migrate -> DUM_ESTATE):
   * host_arena: pinned (cudaHostAlloc / cudaHostRegister) host memory holding
   *             block b at byte offset b * 2 MiB, max_blocks blocks;
   * frame_pool: device memory holding frame f at f * 2 MiB, hbm_frames frames. */
  void *host_arena;
  uint64_t host_arena_bytes;
  void *frame_pool;
  uint64_t frame_pool_bytes;
  /* DUM_CFG_* bits (0 = production). */
  uint32_t flags;
} dum_config;

/* dum_config.flags: build every walk with the sequential one-warp walker
 * (the literal PAPER.md L218-L224 loop) instead of the parallel k_walk --
 * a verification mode: both must give identical walk caches. */
#define DUM_CFG_SEQ_WALKS 0x1u
/* dum_config.flags: answer the windows whose kernels' walks share no block
 * on the fast path (walk index at build end, per-walk residency facts, the
 * persistent copy + staged-selection kernel k_window_fast) and only the rest
 * on the exact kernel.  Without it (the default) every query takes the exact
 * kernel k_predict, one CTA per query, and the walk index is not built.  Both
 * give identical outputs; the default is the faster one on the G workload
 * (DESIGN.md 7). */
#define DUM_CFG_FAST_WINDOWS 0x2u

/* Fill *cfg with the defaults (Config9, N = 32). */
void dum_config_default(dum_config *cfg);

int dum_create(const dum_config *cfg, dum_engine **out);
int dum_destroy(dum_engine *eng);
/* Clear exec map, correlation tables, block tables, walk cache, history,
 * staging, residency (all frames free, no inactive blocks). Keeps allocations. */
int dum_reset(dum_engine *eng, dum_stream_t stream);

/* ---- a1 + a2 ------------------------------------------------------------
 * Stage one batch of whole kernel launches.  Launch i has hash launch_hash[i]
 * ("hash value of the kernel's name and arguments") and the fault
 * records fault_block[launch_off[i] .. launch_off[i+1]) (block ids, in fault
 * order, duplicates allowed).  Requires launch_off[0] == 0 and
 * launch_off[n_launch] == n_fault.  Records are normalised to the first
 * occurrence of each block per launch (P:L124 step 2; D2).  Exec IDs: same
 * hash -> same ID, else the next dense ID in first-seen order (D3);
 * written to out_exec[i] if out_exec != NULL (device).  Staged launches are
 * applied by the next dum_build_tables.  With DUM_HOST_PTRS the launch
 * offsets are validated on the host (DUM_EINVAL); block ids >= max_blocks are
 * detected on the device for both kinds of pointers (sticky DUM_EINVAL from
 * dum_sync; the offending records are dropped); so are device-side launch
 * offsets that are not monotone or run past n_fault (sticky DUM_EINVAL, the
 * launch is dropped).  DUM_HOST_PTRS uploads run on the engine's ingest stream
 * into a single upload buffer, in order with the ingest kernels that read it
 * (the ingest of this batch may overlap the build of the previous one), and
 * `stream` waits for the ingest: pinned host inputs must stay unmodified until
 * the call's work on `stream` has completed, exactly like device inputs
 * (pageable inputs are staged by the CUDA runtime before the call returns). */
int dum_record_faults(dum_engine *eng, const uint64_t *launch_hash, const uint64_t *launch_off,
                      uint32_t n_launch, const uint32_t *fault_block, uint64_t n_fault,
                      uint32_t *out_exec, uint32_t flags, dum_stream_t stream);

/* ---- a3 - a6 ------------------------------------------------------------
 * Apply every staged launch, in order:
 *  a3  record (e_{k-4}, e_{k-3}, e_{k-2} -> e_k) in entry e_{k-1} of the
 *      execution ID correlation table (D4, D5);
 *  a4  per normalised fault b_j of launch k (exec e): INSERT b_j as the MRU
 *      successor in the row of b_{j-1}, then TOUCH b_j (allocate / make MRU)
 *      in block table e (D7-D10);
 *  a5  Start/End of e = first/last normalised fault of e's latest faulting
 *      launch (D11);
 *  a6  rebuild the walk cache WALK(e, NONE) of every exec ID touched
 *      (D13). */
int dum_build_tables(dum_engine *eng, dum_stream_t stream);

/* A prefetch query: the kernel running now (exec), the three exec IDs that ran
 * before it (hist[0] oldest; DUM_NONE allowed, D4), the faulted block the walk
 * starts from (anchor) or DUM_NONE for a kernel-transition query that starts at
 * Start (D14), and the degree n <= cfg.degree_n (D15). */
typedef struct {
  uint32_t exec;
  uint32_t hist[3];
  uint32_t anchor;
  uint32_t n;
} dum_query;

/* Build transition queries for launches first..n_seq-1 of an exec-ID sequence
 * (device array exec_seq[0..n_seq)): q[i-first] = {exec_seq[i],
 * exec_seq[i-3..i-1] (DUM_NONE before 0), DUM_NONE, degree}. */
int dum_make_queries(dum_engine *eng, const uint32_t *exec_seq, uint32_t n_seq, uint32_t first,
                     uint32_t degree, dum_query *out, dum_stream_t stream);

/* ---- a6 + a7 ------------------------------------------------------------
 * For each query q (device array): chain up to q.n next-kernel predictions
 * through the execution ID correlation table (D16), then
 * concatenate WALK(exec, anchor) and WALK(e_d, NONE) of each predicted kernel,
 * keeping the first occurrence of every block (D17).  Reads the state left by
 * the last dum_build_tables.
 *   out_pairs      pool of (block, exec) uint32 pairs, out_cap_pairs entries;
 *   out_range      2 * n_query uint64: query i's pairs are
 *                  out_pairs[2*out_range[2i] .. 2*out_range[2i+1]) -- each query
 *                  owns a contiguous range; ranges are disjoint but not ordered;
 *   out_kern_off   n_query * (degree_n + 2) uint32 or NULL: kern_off[0] = 0,
 *                  kern_off[d+1] = pairs emitted after kernel d (padded);
 *   out_chain      n_query * (degree_n + 1) uint32 or NULL: the predicted
 *                  kernels (DUM_NONE padded);
 *   out_needed     device uint64 or NULL: pool entries the call required. */
int dum_predict_prefetch(dum_engine *eng, const dum_query *queries, uint32_t n_query, uint32_t *out_pairs,
                         uint64_t out_cap_pairs, uint64_t *out_range, uint32_t *out_kern_off,
                         uint32_t *out_chain, uint64_t *out_needed, dum_stream_t stream);

/* ---- a8 -----------------------------------------------------------------
 * Pre-eviction selection per query window (D18-D20): need =
 * max(0, #window blocks without a frame - #free frames); victims = the first
 * `need` resident blocks in least-recently-migrated order that are neither in
 * the window nor the anchor.  Victims whose UM block is inactive (P:L285,
 * dum_mark_inactive) go to out_invalidate, the rest to out_writeback, both in
 * LRM order.  query_range/pairs as produced by dum_predict_prefetch; anchors
 * are read from queries[i].anchor (queries may be NULL: no anchors).
 *   out_range: 4 * n_query uint64 = {wb_begin, wb_end, inv_begin, inv_end}
 *   out_needed: device uint64 or NULL (entries required per pool). */
int dum_select_evictions(dum_engine *eng, const uint64_t *query_range, const uint32_t *pairs,
                         uint32_t n_query, const dum_query *queries, uint32_t *out_writeback,
                         uint32_t *out_invalidate, uint64_t out_cap, uint64_t *out_range,
                         uint64_t *out_needed, dum_stream_t stream);

/* ---- a7 + a8 fused ------------------------------------------------------
 * dum_predict_prefetch followed by dum_select_evictions on the same windows,
 * in one kernel: the window set built for the prefetch list is reused for the
 * victim search instead of being re-read from HBM.  Outputs and semantics are
 * exactly those of the two calls (same arguments, same layouts). */
int dum_predict_select(dum_engine *eng, const dum_query *queries, uint32_t n_query, uint32_t *out_pairs,
                       uint64_t out_cap_pairs, uint64_t *out_range, uint32_t *out_kern_off, uint32_t *out_chain,
                       uint64_t *out_needed, uint32_t *out_writeback, uint32_t *out_invalidate, uint64_t sel_cap,
                       uint64_t *sel_range, uint64_t *sel_needed, dum_stream_t stream);

/* ---- one step ------------------------------------------------------------
 * The whole hot path of one batch in one call (SURVEY 8d schedule):
 * dum_record_faults(batch, flags: DUM_HOST_PTRS / DUM_INPUTS_READY) -> one
 * transition query per launch of the batch ({its exec ID, the three exec IDs
 * before it -- across steps --, DUM_NONE, degree}) -> dum_predict_select on the
 * state built by the previous steps -> dum_build_tables(batch).  Outputs and
 * their layouts are dum_predict_select's, one query per launch in launch
 * order.  The engine keeps the last three exec IDs of the previous step
 * (DUM_NONE after dum_reset).  Requires no batch staged by dum_record_faults.
 * The build of the batch runs beside the predict kernels (side stream, issued
 * after the chain step); its rebuilt walks are published after predict, so
 * predict sees the tables and walks of the previous steps only (D12). */
int dum_step(dum_engine *eng, const uint64_t *launch_hash, const uint64_t *launch_off, uint32_t n_launch,
             const uint32_t *fault_block, uint64_t n_fault, uint32_t flags, uint32_t degree, uint32_t *out_pairs,
             uint64_t out_cap_pairs, uint64_t *out_range, uint32_t *out_kern_off, uint32_t *out_chain,
             uint64_t *out_needed, uint32_t *out_writeback, uint32_t *out_invalidate, uint64_t sel_cap,
             uint64_t *sel_range, uint64_t *sel_needed, dum_stream_t stream);

/* dum_step as a replayed CUDA graph (enable != 0): the batch is copied into
 * the engine's upload buffers, then the whole step replays as one graph (one
 * per batch size x staging set x output buffers, captured on first use; every
 * value a step changes lives on the device).  Outputs must keep their
 * addresses between the steps of one graph.  A captured build leaves its
 * jump tables and the publishing of its walks to the start of the next step
 * (or to the next predict / build / dum_dump_state call). */
int dum_set_step_graphs(dum_engine *eng, int enable);

/* Mark UM blocks as belonging to inactive (inactive != 0) or active PyTorch
 * blocks (D20: a block is invalidatable iff every PT block overlapping
 * it is inactive -- the caller resolves overlap). */
int dum_mark_inactive(dum_engine *eng, const uint32_t *blocks, uint32_t n, int inactive,
                      dum_stream_t stream);

/* Replace the residency with a snapshot: lrm_blocks[i] resident in frame i with
 * migration stamp i (oldest first); frames n_resident.. free. */
int dum_load_residency(dum_engine *eng, const uint32_t *lrm_blocks, uint32_t n_resident,
                       dum_stream_t stream);

/* ---- a9 -----------------------------------------------------------------
 * DUM_H2D:        blocks (non-resident) get the lowest free frames in list
 *                 order (D21), are copied host -> HBM and stamped (D19).
 * DUM_D2H:        resident blocks are copied HBM -> host and freed.
 * DUM_INVALIDATE: resident blocks are freed without a copy.
 * DUM_D2D:        blocks_or_src == NULL: compaction -- the resident blocks in
 *                 the highest frames move into the lowest free frames until
 *                 the free frames form a contiguous tail; otherwise block
 *                 blocks_or_src[i] moves to the free frame dst_frames[i].
 * method: 0 = auto (SM copy kernel), 1 = SM copy kernel (16 B vector loads /
 *         stores, host memory through its mapped address), 2 = copy engines
 *         (one cudaMemcpyAsync per run contiguous on both sides; synchronizes:
 *         the frame plan is read back first), 3 = TMA bulk copies
 *         (cp.async.bulk global -> shared -> global, 32 KiB tiles, one CTA per
 *         SM).
 * Invalid lists (duplicates, wrong residency, not enough free frames) set a
 * sticky DUM_EINVAL / DUM_ECAPACITY and move nothing. */
typedef enum { DUM_H2D = 0, DUM_D2H = 1, DUM_INVALIDATE = 2, DUM_D2D = 3 } dum_dir;
int dum_migrate_blocks(dum_engine *eng, dum_dir dir, const uint32_t *blocks_or_src, const uint32_t *dst_frames,
                       uint32_t n, uint32_t method, dum_stream_t stream);
/* The copy kernels (methods 0, 1, 3) of this engine use at most n_sms SMs'
 * worth of CTAs (0 = every SM, the default): two engines whose copies run
 * concurrently -- write-back on one, fetch on another -- each take a share
 * instead of queueing behind each other.  No synchronization. */
int dum_set_copy_sms(dum_engine *eng, uint32_t n_sms);

/* ---- closed-loop replay ------------------------------
 * dum_simulate replays launches 0 .. n_launch-1 (launch k has hash
 * launch_hash[k] and accesses the blocks acc_blk[acc_off[k % n_kernels] ..
 * acc_off[k % n_kernels + 1]), per launch and in order, through the paper's
 * loop: faults = accesses without a frame (first
 * occurrence, D2) -> dum_record_faults -> demand eviction when the faults
 * exceed the free frames (least recently migrated blocks the launch does not
 * access, D22; inactive ones invalidated with DUM_SIM_INVALIDATE) and H2D of
 * the faults -> dum_build_tables -> (DUM_SIM_PREFETCH) the transition query of
 * the next launch (its exec ID if its hash is known, the last three exec IDs
 * as history, degree n) -> (DUM_SIM_PREEVICT) pre-eviction of the window's
 * victims (L236-L243) -> H2D of the window's non-resident prefix that fits the
 * free frames (L156-L158); without DUM_SIM_PREEVICT every non-resident window
 * block is prefetched and the driver evicts the least recently migrated
 * blocks, window or not, for those beyond the free frames (L236-L238; the
 * evictions are reported as pre_wb / pre_inv).  Every step runs in this library's kernels, list
 * sizes stay on the device.  Without a data plane the migrations move the
 * residency only (metadata-only engine: B/G scale); with one the bytes move.
 * Per-launch statistics go to stats[k] (device).  launch_hash, acc_blk, stats:
 * device; acc_off: HOST (n_kernels + 1 entries, <= 8192 accesses per launch).
 * Requires an empty staging area (call after dum_build_tables). */
typedef struct {
  uint32_t faults;      /* demand faults of the launch (blocks migrated on demand) */
  uint32_t demand_wb;   /* demand-path victims written back */
  uint32_t demand_inv;  /* demand-path victims invalidated (D20) */
  uint32_t pre_wb;      /* pre-evicted (prefetch only: driver-evicted) blocks written back */
  uint32_t pre_inv;     /* pre-evicted (prefetch only: driver-evicted) blocks invalidated */
  uint32_t prefetched;  /* window blocks migrated ahead of use */
} dum_sim_stats;
#define DUM_SIM_PREFETCH 0x1u   /* query + prefetch the window (else naive UM: demand only) */
#define DUM_SIM_PREEVICT 0x2u   /* pre-evict for the window */
#define DUM_SIM_INVALIDATE 0x4u /* inactive victims are invalidated, not written back (L285) */
int dum_simulate(dum_engine *eng, const uint64_t *launch_hash, uint32_t n_launch, const uint64_t *acc_off,
                 const uint32_t *acc_blk, uint32_t n_kernels, uint32_t degree, uint32_t flags,
                 dum_sim_stats *stats, dum_stream_t stream);

/* 64-bit position-weighted checksums (sum_w word_w * (2w+1) mod 2^64) of 2 MiB
 * blocks: where = 0 -> HBM frames ids[i]; 1 -> host-arena blocks ids[i]. */
int dum_block_checksums(dum_engine *eng, int where, const uint32_t *ids, uint32_t n, uint64_t *out,
                        dum_stream_t stream);

/* ---- inspection ---------------------------------------------------------
 * Canonical state dump (identical byte format to
 * the oracle's).  `what` is a bitwise OR of DUM_DUMP_*.  Synchronizes.  If cap
 * is too small nothing is written, *needed holds the size and DUM_ECAPACITY is
 * returned. */
#define DUM_DUMP_EXEC 1u
#define DUM_DUMP_CORR 2u
#define DUM_DUMP_BLK 4u
#define DUM_DUMP_WALK 8u
#define DUM_DUMP_RES 16u
#define DUM_DUMP_HIST 32u
int dum_dump_state(dum_engine *eng, uint32_t what, void *host_buf, uint64_t cap, uint64_t *needed);

/* Synchronize `stream`, then return the sticky device error (clearing it) and
 * the largest capacity a failed call required (*needed, may be NULL). */
int dum_sync(dum_engine *eng, dum_stream_t stream, uint64_t *needed);

typedef struct {
  uint32_t num_exec;        /* exec IDs assigned */
  uint32_t corr_records;    /* execution-correlation records */
  uint32_t free_frames;
  uint32_t staged_launches; /* recorded, not yet built */
  uint64_t launches;        /* launches recorded since reset */
  uint64_t staged_faults;
  uint32_t slow_walks;      /* walks that took the sequential fallback in the last build */
  uint32_t n_resident;
  uint32_t guard_line;      /* first failed internal consistency guard (0 = none) */
  uint32_t guard_val;
} dum_stats;
/* Synchronizes. */
int dum_get_stats(dum_engine *eng, dum_stats *out);

/* ---- instrumentation (bench / profiling; not needed for correctness) ------
 * Work counters accumulated on the device by the kernels (one atomic per CTA);
 * the bench derives each kernel's algorithmic bytes from them (DESIGN.md
 * "Roofline accounting").  Reading synchronizes the device. */
enum {
  DUM_CTR_RAW_RECORDS = 0,  /* fault records ingested                    */
  DUM_CTR_NORM_RECORDS,     /* after first-occurrence dedupe             */
  DUM_CTR_LAUNCHES,         /* launches ingested                         */
  DUM_CTR_CORR_UPSERTS,     /* exec-correlation upserts                  */
  DUM_CTR_EXEC_BUILT,       /* exec IDs whose block table was updated    */
  DUM_CTR_OPS,              /* fused INSERT+TOUCH ops applied            */
  DUM_CTR_SETS,             /* (exec, set) pairs read-modified-written   */
  DUM_CTR_WALK_ROWS,        /* rows read by walk rebuilds                */
  DUM_CTR_WALK_OUT,         /* walk-cache entries written                */
  DUM_CTR_QUERIES,          /* prefetch queries answered                 */
  DUM_CTR_CHAIN,            /* kernels in predicted windows              */
  DUM_CTR_GATHERED,         /* walk-list entries gathered by predict     */
  DUM_CTR_EMITTED,          /* (block, exec) pairs emitted               */
  DUM_CTR_SEL_WINDOW,       /* window entries read by select             */
  DUM_CTR_SEL_SCANNED,      /* LRM-log entries scanned by select         */
  DUM_CTR_SEL_VICTIMS,      /* victims selected                          */
  DUM_CTR_MIG_BLOCKS,       /* 2 MiB blocks copied                       */
  DUM_CTR_RUNS,             /* walk bitmap runs inserted by predict      */
  /* which code path answered each unit of work (tests assert every path is
   * exercised; the bench reports them) */
  DUM_CTR_Q_NODUP,          /* predict queries: window-bitmap path, no duplicate found    */
  DUM_CTR_Q_DUP,            /* predict queries: duplicate path (occurrence lists)         */
  DUM_CTR_Q_FALLBACK,       /* predict queries: min-position hash over every element      */
  DUM_CTR_WALK_PREFIX,      /* walks proved to be a prefix of the latest launch           */
  DUM_CTR_WALK_DEDUPE,      /* walks built by the parallel min-position dedupe            */
  DUM_CTR_WALK_SLOW,        /* walks built by the sequential walker                       */
  DUM_CTR_Q_FAST,           /* predict queries: conflict-free window (no bitmap)          */
  DUM_CTR_ANCHOR_WALKS,     /* fault-anchored walks (WALK(e, anchor))                     */
  DUM_CTR_INGEST_DUP,       /* launches whose records held duplicates                     */
  DUM_CTR_Q_SLOW,           /* predict queries sent to the exact (bitmap) kernel          */
  DUM_CTR_FAST_EMITTED,     /* pairs emitted by the fast path (= walk entries it gathered)      */
  DUM_CTR_FAST_SCANNED,     /* LRM-log entries scanned by the fast path's selection             */
  DUM_CTR_FAST_VICTIMS,     /* victims selected by the fast path                                */
  DUM_CTR_SLOW_CONFLICT,    /* exact path: two walks of the chain share a block            */
  DUM_CTR_SLOW_UNRECORDED,  /* exact path: a walk's conflicts were too many to record      */
  DUM_CTR_SLOW_SPAN,        /* exact path: the selection could pass the position bitmap   */
  DUM_CTR_SLOW_ANCHOR,      /* exact path: fault-anchored query                            */
  DUM_CTR_FAST_DIRTY,       /* fast selections over a log with stale entries               */
  DUM_NCOUNTERS = 40
};
/* Counters accumulate only while counting is on (the default); the bench turns
 * it off for its timed region (no instrumentation atomics there). */
int dum_set_counting(dum_engine *eng, int enable);
int dum_read_counters(dum_engine *eng, uint64_t out[DUM_NCOUNTERS], int reset);

/* Per-kernel CUDA-event timing on the launching stream (off by default).
 * dum_read_timing synchronizes and returns the summed milliseconds and launch
 * counts per kernel since the last reset. */
enum {
  DUM_T_INGEST = 0,
  DUM_T_EXEC_ASSIGN,
  DUM_T_BUILD_PREP,
  DUM_T_APPLY_WALK,
  DUM_T_WALK_SLOW,
  DUM_T_MAKE_QUERIES,
  DUM_T_ANCHOR_WALK,
  DUM_T_PREDICT,
  DUM_T_SELECT,
  DUM_T_MIG_PLAN,
  DUM_T_COPY,
  DUM_T_RESIDENCY,
  DUM_T_CHAIN,
  DUM_T_JUMP,         /* jump tables over the correlation table (side stream, in dum_build_tables) */
  DUM_T_WALK,         /* parallel walk-cache rebuild (in dum_build_tables) */
  DUM_T_EXACT,        /* exact-path predict kernel k_predict (the fast path runs beside it on a side stream) */
  DUM_T_WALK_INDEX,   /* walk index: holders per block, conflicts per walk (build end) */
  DUM_T_WALK_RES,     /* residency facts per walk (predict) */
  DUM_T_SELECT_FAST,  /* fast path with selection: k_window_fast (pairs + selection, one persistent kernel) */
  DUM_T_COMMIT,       /* k_walk_commit: the rebuilt walks published after predict (dum_build_tables) */
  DUM_NTIMERS = 24
};
int dum_set_timing(dum_engine *eng, int enable);
int dum_read_timing(dum_engine *eng, double ms[DUM_NTIMERS], uint64_t count[DUM_NTIMERS], int reset);
/* The same timed regions as a timeline: synchronizes, then for each region
 * recorded since the last dum_read_timing / dum_read_timeline (in issue order,
 * at most cap) writes its timer id and its start / end in ms relative to the
 * first region's start; returns the number written (>= 0) or a negative
 * DUM_* code.  The regions are consumed (and added to dum_read_timing's sums). */
int dum_read_timeline(dum_engine *eng, int cap, int *ids, float *t0, float *t1);

const char *dum_last_error(const dum_engine *eng);

/* Number of the library's own kernel launches issued so far (for bench
 * launch counting). */
uint64_t dum_kernel_launches(const dum_engine *eng);

/* Memory kind of a pointer as this library's CUDA runtime sees it
 * (cudaMemoryType: 0 unregistered host, 1 pinned host, 2 device, 3 managed;
 * -1 on error).  DUM_HOST_PTRS inputs should be pinned (1) for asynchronous
 * full-bandwidth copies. */
int dum_host_ptr_kind(const void *ptr);

#ifdef __cplusplus
}
#endif
#endif /* DEEPUM_B200_H */
