// libdeepum_b200.so: the C-ABI (include/deepum_b200.h) and the host engine that
// owns the device state, validates calls and launches the kernels of
// k_record.cu, k_build.cu, k_predict.cu, k_select.cu and k_migrate.cu in stream
// order.  Every step of the hot path runs in those kernels; this file only
// allocates, validates, launches, and (for dum_dump_state) canonicalises a
// device snapshot for inspection.
#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <vector>

#include "device_util.cuh"
#include "kernels.cuh"
#include "predict.cuh"
#include "select_tail.cuh"

using namespace dum;

namespace {

__global__ void k_fill_u32(uint32_t *p, uint64_t n, uint32_t v) {
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = v;
}

__global__ void k_init_corr(CorrSlot *c, uint32_t n) {
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    c[i].key[0] = c[i].key[1] = c[i].key[2] = c[i].key[3] = NONE;
    c[i].last = 0;
    c[i].first = ~0ull;
  }
}

__global__ void k_init_state(DevState *st) {
  st->E = 0;
  for (int q = 0; q < 4; ++q) st->hist[q] = NONE;
  st->err = 0;
  st->needed = 0;
  st->pool_pairs = st->pool_wb = st->pool_inv = st->pool_anchor = st->pool_big = st->pool_chunks = 0;
  st->pool_bigb = 0;
  st->sel_queue = 0;
  st->copy_queue = 0;
  st->chain_done = 0;
  for (int c = 0; c < 16; ++c) st->q_cls[c] = 0;
  st->n_fast = 0;
  st->n_dd = 0;
  st->n_slow = 0;
  st->n_pend = 0;
  st->n_items = st->n_leads = 0;
  for (int c = 0; c < 4; ++c) st->cls_cnt[c] = 0;
  st->corr_used = 0;
  st->mig_ok = 0;
  st->mig_n = 0;
  st->dbg_line = st->dbg_val = 0;
  for (int c = 0; c < DUM_NCOUNTERS; ++c) st->ctr[c] = 0;
  st->counting = 1;
  st->k_base = 0;
}

uint32_t pow2ceil_h(uint64_t x) {
  uint64_t p = 1;
  while (p < x) p <<= 1;
  return (uint32_t)p;
}

int fail(dum_engine *e, int code, const char *msg) {
  if (e) e->last_error = msg;
  return code;
}

int cuda_fail(dum_engine *e, cudaError_t err, const char *where) {
  if (e) {
    e->last_error = std::string(where) + ": " + cudaGetErrorString(err);
  }
  return DUM_ECUDA;
}

#define CK(call)                                  \
  do {                                            \
    cudaError_t _e = (call);                      \
    if (_e != cudaSuccess) return cuda_fail(e, _e, #call); \
  } while (0)

template <class T>
cudaError_t dmalloc(T **p, uint64_t count) {
  return cudaMalloc((void **)p, std::max<uint64_t>(count, 1) * sizeof(T));
}

cudaError_t fill(uint32_t *p, uint64_t n, uint32_t v, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  uint64_t blocks = std::min<uint64_t>((n + 255) / 256, 4096);
  k_fill_u32<<<(unsigned)blocks, 256, 0, s>>>(p, n, v);
  return cudaGetLastError();
}

int reset_state(dum_engine *e, cudaStream_t s) {
  const Geo &g = e->g;
  if (e->ev_commit) CK(cudaStreamWaitEvent(s, e->ev_commit, 0));  // a walk commit still copying
  e->commit_inflight = false;
  e->commit_stale = false;  // (the walks are cleared below)
  e->jump_stale = false;
  if (e->ev_join) CK(cudaStreamWaitEvent(s, e->ev_join, 0));  // jump tables still building on the side stream
  if (e->ev_join2) CK(cudaStreamWaitEvent(s, e->ev_join2, 0));  // exact-path predict kernel
  if (e->ev_widx) CK(cudaStreamWaitEvent(s, e->ev_widx, 0));    // walk index
  if (e->ev_rec) CK(cudaStreamWaitEvent(s, e->ev_rec, 0));    // record work on the ingest stream
  CK(fill((uint32_t *)e->d_exec_keys, 2ull * (e->exec_cap + 1), NONE, s));
  CK(cudaMemsetAsync(e->d_exec_keys + e->exec_cap, 0, 8, s));  // sentinel slot: absent
  CK(fill(e->d_exec_vals, e->exec_cap + 1, PENDING, s));
  CK(fill(e->d_exec_minpos, e->exec_cap + 1, NONE, s));
  k_init_corr<<<1024, 256, 0, s>>>(e->d_corr, e->corr_cap);
  CK(cudaGetLastError());
  CK(fill(e->d_tbl, (uint64_t)g.Emax * g.R * g.stride, NONE, s));
  CK(fill(e->d_start_end, 2ull * g.Emax, NONE, s));
  CK(cudaMemsetAsync(e->d_walk_len, 0, 4ull * g.Emax, s));
  CK(cudaMemsetAsync(e->d_wrun_len, 0, 4ull * g.Emax, s));
  CK(cudaMemsetAsync(e->d_conf_n, 0, 4ull * g.Emax, s));  // no walks: no conflicts
  CK(fill(e->d_step_exec, 3, NONE, s));  // dum_step: no history
  CK(cudaMemsetAsync(e->d_bcnt, 0, 4ull * g.W, s));
  CK(fill(e->d_head, g.Emax, NONE, s));
  CK(cudaMemsetAsync(e->d_e_ops, 0, 4ull * g.Emax, s));
  CK(cudaMemsetAsync(e->d_e_last, 0, 4ull * g.Emax, s));
  k_init_state<<<1, 1, 0, s>>>(e->d_state);
  CK(cudaGetLastError());
  CK(launch_reset_residency(e, s));
  // the ingest stream waits for the reset: a following dum_record_faults with
  // DUM_HOST_PTRS / DUM_INPUTS_READY does not order itself after `s`
  CK(cudaEventRecord(e->ev_s_now, s));
  CK(cudaStreamWaitEvent(e->rec_s, e->ev_s_now, 0));
  e->n_staged = 0;
  e->staged_faults = 0;
  e->launches = 0;
  e->built_launches = 0;
  e->kernel_launches += 8;
  return DUM_OK;
}

void free_all(dum_engine *e) {
  void *ptrs[] = {e->d_exec_keys, e->d_exec_vals, e->d_exec_minpos, e->d_exec_hash, e->d_corr, e->d_tbl,
                  e->d_start_end, e->d_walk, e->d_walk_len, e->d_walk_n, e->d_walk_len_n, e->d_wrun_n,
                  e->d_wrun_len_n, e->d_in_hash, e->d_in_off, e->d_in_faults,
                  e->stage_base[0], e->stage_base[1], e->stage_base[2], e->stage_base[3], e->stage_base[4],
                  e->stage_base[5], e->d_head, e->d_next, e->d_order, e->d_slow_list,
                  e->d_e_ops, e->d_e_last, e->d_pend, e->d_plan_agg, e->d_lead, e->d_items, e->d_rowc, e->d_big_pool, e->d_big_pool_b, e->d_ingest_pool, e->d_walk_seen,
                  e->d_walk_chain, e->d_walk_tmp, e->d_walk_out, e->d_anchor_pool, e->d_anchor_range,
                  e->d_frame_of, e->d_stamp_of, e->d_block_of, e->d_free_bits, e->d_inactive_bits, e->d_res_bits, e->d_logpos, e->d_lrm_blk,
                  e->d_lrm_stamp, e->d_mig_frames, e->d_mig_src, e->d_mig_blocks, e->d_state, e->d_qkern,
                  e->d_qloff, e->d_qnk, e->d_qbase, e->d_rec_slot, e->d_jump, e->d_wrun, e->d_wrun_len, e->d_qeoff, e->d_qgoff, e->d_qrank, e->d_qperm,
                  e->d_bcnt, e->d_bhold, e->d_conf, e->d_conf_n, e->d_wnr, e->d_wnres, e->d_respos, e->d_qroff, e->d_qneed, e->d_qvb, e->d_chunk_map, e->d_selrec, e->d_dd_list, e->d_log_bits,
                  e->sim_acc_bits, e->sim_faults, e->sim_pairs, e->sim_wb, e->sim_inv, e->sim_pf, e->sim_foff,
                  e->sim_ranges, e->sim_q, e->d_step_exec, e->d_step_q};
  for (void *p : ptrs)
    if (p) cudaFree(p);
  if (e->ev_fork) cudaEventDestroy(e->ev_fork);
  if (e->ev_join) cudaEventDestroy(e->ev_join);
  if (e->side) cudaStreamDestroy(e->side);
  if (e->side2) cudaStreamDestroy(e->side2);
  if (e->graph_s) cudaStreamDestroy(e->graph_s);
  if (e->ev_graph) cudaEventDestroy(e->ev_graph);
  if (e->ev_wres) cudaEventDestroy(e->ev_wres);
  if (e->cap_events_ready)
    for (int i = 0; i < 8; ++i)
      if (e->cap_ev[i]) cudaEventDestroy(e->cap_ev[i]);
  if (e->side3) cudaStreamDestroy(e->side3);
  if (e->side4) cudaStreamDestroy(e->side4);
  if (e->ev_fork4) cudaEventDestroy(e->ev_fork4);
  if (e->ev_bhead) cudaEventDestroy(e->ev_bhead);
  if (e->ev_commit) cudaEventDestroy(e->ev_commit);
  if (e->ev_wslow_fork) cudaEventDestroy(e->ev_wslow_fork);
  if (e->ev_wslow) cudaEventDestroy(e->ev_wslow);
  if (e->ev_widx) cudaEventDestroy(e->ev_widx);
  if (e->ev_fork2) cudaEventDestroy(e->ev_fork2);
  if (e->ev_join2) cudaEventDestroy(e->ev_join2);
  if (e->rec_s) cudaStreamDestroy(e->rec_s);
  if (e->ev_rec) cudaEventDestroy(e->ev_rec);
  if (e->ev_s_now) cudaEventDestroy(e->ev_s_now);
  for (int b = 0; b < 2; ++b)
    if (e->ev_stage_free[b]) cudaEventDestroy(e->ev_stage_free[b]);
  if (e->h_state) cudaFreeHost(e->h_state);
  for (auto &t : e->pending) {
    cudaEventDestroy(t.a);
    cudaEventDestroy(t.b);
  }
  for (auto ev : e->event_pool) cudaEventDestroy(ev);
  for (auto &g : e->step_graphs) cudaGraphExecDestroy(g.exec);
  e->step_graphs.clear();
}

cudaEvent_t get_event(dum_engine *e) {
  if (!e->event_pool.empty()) {
    cudaEvent_t ev = e->event_pool.back();
    e->event_pool.pop_back();
    return ev;
  }
  cudaEvent_t ev = nullptr;
  cudaEventCreate(&ev);
  return ev;
}

}  // namespace

namespace dum {
TimerScope::TimerScope(dum_engine *e_, int id_, cudaStream_t s_) : e(e_), id(id_), s(s_), b(nullptr) {
  if (!e->timing || e->capturing) return;
  cudaEvent_t a = get_event(e);
  b = get_event(e);
  cudaEventRecord(a, s);
  e->pending.push_back({id, a, b});
}
TimerScope::~TimerScope() {
  if (b) cudaEventRecord(b, s);
}
}  // namespace dum

extern "C" {

void dum_config_default(dum_config *c) {
  std::memset(c, 0, sizeof(*c));
  c->num_rows = 2048;  // Config9
  c->assoc = 2;
  c->num_succs = 4;
  c->degree_n = 32;
  c->max_blocks = 1u << 16;
  c->max_exec_ids = 8192;
  c->hbm_frames = 1024;
  c->row_index = 0;
  c->device = 0;
}

int dum_create(const dum_config *cfg, dum_engine **out) {
  if (!cfg || !out) return DUM_EINVAL;
  *out = nullptr;
  const uint32_t R = cfg->num_rows, A = cfg->assoc, S = cfg->num_succs;
  if (R == 0 || (R & (R - 1)) || R > 8192 || A == 0 || A > 32 || S == 0 || S > 32 || cfg->degree_n > 128 ||
      cfg->max_blocks == 0 || cfg->max_blocks > (1u << 20) || cfg->max_exec_ids == 0 || cfg->hbm_frames == 0 ||
      cfg->row_index > 1)
    return DUM_EINVAL;
  dum_engine *e = new (std::nothrow) dum_engine();
  if (!e) return DUM_ENOMEM;
  e->cfg = *cfg;
  e->fast_windows = (cfg->flags & DUM_CFG_FAST_WINDOWS) != 0;
  e->device = cfg->device;
  e->timing = false;
  for (int i = 0; i < DUM_NTIMERS; ++i) {
    e->t_ms[i] = 0;
    e->t_cnt[i] = 0;
  }
  Geo &g = e->g;
  g.R = R;
  g.A = A;
  g.S = S;
  g.N = cfg->degree_n;
  g.W = cfg->max_blocks;
  g.C = cfg->hbm_frames;
  g.Emax = cfg->max_exec_ids;
  g.row_index = cfg->row_index;
  g.set_u32 = A * (1 + S);
  g.stride = (g.set_u32 + 7) / 8 * 8;  // 32 B sectors
  // a walk has at most 1 + S(RA + 1) blocks; rounded up to 8 so that every
  // walk (and its run list) starts 32 B aligned (vector loads in k_predict)
  g.walk_cap = (1 + S * (R * A + 1) + 7) / 8 * 8;
  if (cudaSetDevice(cfg->device) != cudaSuccess) {
    delete e;
    return DUM_ECUDA;
  }
  e->exec_cap = std::max<uint32_t>(64, pow2ceil_h(2ull * g.Emax));
  const uint64_t corr_records = cfg->corr_capacity ? cfg->corr_capacity : 16ull * g.Emax;
  e->corr_cap = pow2ceil_h(2 * corr_records);
  e->jump_levels = 1;
  while ((1u << e->jump_levels) < g.N) ++e->jump_levels;  // d <= N - 1 needs bits 0..levels-1
  e->stage_launch_cap = cfg->max_batch_launches ? cfg->max_batch_launches : 65536;
  e->stage_fault_cap = cfg->max_batch_faults ? cfg->max_batch_faults : (16ull << 20);
  e->big_pool_entries = 4 * e->stage_fault_cap;
  e->n_walk_slots = 64;
  e->walk_hash_cap = pow2ceil_h(2ull * g.walk_cap);
  e->anchor_range_cap = 1u << 16;
  e->anchor_pool_entries = 16ull << 20;
  e->lrm_cap = 4 * g.C + 1024;
  e->mig_cap = g.C + 32;
  const uint64_t tmp_cap = g.walk_cap + (uint64_t)g.R * g.A + 4;
  cudaError_t err = cudaSuccess;
  auto A_ = [&](cudaError_t x) {
    if (err == cudaSuccess) err = x;
  };
  A_(dmalloc(&e->d_exec_keys, e->exec_cap + 1));
  A_(dmalloc(&e->d_exec_vals, e->exec_cap + 1));
  A_(dmalloc(&e->d_exec_minpos, e->exec_cap + 1));
  A_(dmalloc(&e->d_exec_hash, g.Emax));
  A_(dmalloc(&e->d_corr, e->corr_cap));
  A_(dmalloc(&e->d_rec_slot, e->corr_cap));
  A_(dmalloc(&e->d_jump, (uint64_t)e->jump_levels * e->corr_cap));
  {
    // jump tables (k_jump.cu) overlap the block-table apply/walk here.  Normal
    // priority: a high-priority side stream stalled the main stream by
    // ~100 us per step when steps are issued back to back (measured in round 1)
    A_(cudaStreamCreateWithFlags(&e->side, cudaStreamNonBlocking));
  }
  A_(cudaStreamCreateWithFlags(&e->side2, cudaStreamNonBlocking));
  A_(cudaStreamCreateWithFlags(&e->graph_s, cudaStreamNonBlocking));
  A_(cudaEventCreateWithFlags(&e->ev_graph, cudaEventDisableTiming));
  A_(cudaEventCreateWithFlags(&e->ev_wres, cudaEventDisableTiming));
  {  // the walk index runs here beside the next step's ingest and gates its k_chain:
     // high priority, so that its CTAs are dispatched first
    int lo = 0, hi = 0;
    cudaDeviceGetStreamPriorityRange(&lo, &hi);
    A_(cudaStreamCreateWithPriority(&e->side3, cudaStreamNonBlocking, hi));
  }
  {  // the build head beside the exact predict kernel: its few CTAs are dispatched first
    int lo = 0, hi = 0;
    cudaDeviceGetStreamPriorityRange(&lo, &hi);
    A_(cudaStreamCreateWithPriority(&e->side4, cudaStreamNonBlocking, hi));
  }
  A_(cudaEventCreateWithFlags(&e->ev_fork4, cudaEventDisableTiming));
  A_(cudaEventCreateWithFlags(&e->ev_bhead, cudaEventDisableTiming));
  A_(cudaEventCreateWithFlags(&e->ev_commit, cudaEventDisableTiming));
  A_(cudaEventCreateWithFlags(&e->ev_wslow_fork, cudaEventDisableTiming));
  A_(cudaEventCreateWithFlags(&e->ev_wslow, cudaEventDisableTiming));
  A_(cudaEventCreateWithFlags(&e->ev_widx, cudaEventDisableTiming));
  A_(cudaEventCreateWithFlags(&e->ev_fork2, cudaEventDisableTiming));
  A_(cudaEventCreateWithFlags(&e->ev_join2, cudaEventDisableTiming));
  A_(cudaEventCreateWithFlags(&e->ev_fork, cudaEventDisableTiming));
  A_(cudaEventCreateWithFlags(&e->ev_join, cudaEventDisableTiming));
  A_(dmalloc(&e->d_tbl, (uint64_t)g.Emax * g.R * g.stride));
  A_(dmalloc(&e->d_start_end, 2ull * g.Emax));
  A_(dmalloc(&e->d_walk, (uint64_t)g.Emax * g.walk_cap));
  A_(dmalloc(&e->d_walk_len, g.Emax));
  A_(dmalloc(&e->d_wrun, 2ull * g.Emax * g.walk_cap));
  A_(dmalloc(&e->d_wrun_len, g.Emax));
  A_(dmalloc(&e->d_walk_n, (uint64_t)g.Emax * g.walk_cap));
  A_(dmalloc(&e->d_walk_len_n, g.Emax));
  A_(dmalloc(&e->d_wrun_n, 2ull * g.Emax * g.walk_cap));
  A_(dmalloc(&e->d_wrun_len_n, g.Emax));
  // host-pointer inputs are uploaded here on the ingest stream (in order with
  // the ingest that reads them), one buffer per staging set: the upload of
  // batch i+1 overlaps the work on batch i
  A_(dmalloc(&e->d_in_hash, 2ull * e->stage_launch_cap));
  A_(dmalloc(&e->d_in_off, 2ull * (e->stage_launch_cap + 1ull)));
  A_(dmalloc(&e->d_in_faults, 2ull * e->stage_fault_cap));
  A_(cudaStreamCreateWithFlags(&e->rec_s, cudaStreamNonBlocking));
  A_(cudaEventCreateWithFlags(&e->ev_rec, cudaEventDisableTiming));
  A_(cudaEventCreateWithFlags(&e->ev_s_now, cudaEventDisableTiming));
  for (int b = 0; b < 2; ++b) A_(cudaEventCreateWithFlags(&e->ev_stage_free[b], cudaEventDisableTiming));
  A_(dmalloc(&e->d_stage_hash, 2ull * e->stage_launch_cap));
  A_(dmalloc(&e->d_stage_norm, 2ull * e->stage_fault_cap));
  A_(dmalloc(&e->d_stage_cnt, 2ull * e->stage_launch_cap));
  A_(dmalloc(&e->d_stage_exec, 2ull * e->stage_launch_cap));
  A_(dmalloc(&e->d_stage_slot, 2ull * e->stage_launch_cap));
  A_(dmalloc(&e->d_pend, e->stage_launch_cap));
  A_(dmalloc(&e->d_stage_off, 2ull * e->stage_launch_cap));
  e->stage_base[0] = e->d_stage_hash;
  e->stage_base[1] = e->d_stage_norm;
  e->stage_base[2] = e->d_stage_cnt;
  e->stage_base[3] = e->d_stage_exec;
  e->stage_base[4] = e->d_stage_slot;
  e->stage_base[5] = e->d_stage_off;
  e->stage_set = 0;
  A_(dmalloc(&e->d_head, g.Emax));
  A_(dmalloc(&e->d_next, e->stage_launch_cap));
  A_(dmalloc(&e->d_order, 3ull * e->stage_launch_cap));
  A_(dmalloc(&e->d_slow_list, e->stage_launch_cap));
  A_(dmalloc(&e->d_dd_list, e->stage_launch_cap));
  A_(dmalloc(&e->d_step_exec, 3ull + e->stage_launch_cap));
  A_(dmalloc(&e->d_step_q, e->stage_launch_cap));
  A_(dmalloc(&e->d_e_ops, g.Emax));
  A_(dmalloc(&e->d_e_last, g.Emax));
  A_(dmalloc(&e->d_lead, 8ull * e->stage_launch_cap));
  A_(dmalloc(&e->d_plan_agg, e->stage_launch_cap / 256 + 1));  // k_build.cu LeadDesc (32 B)
  // apply items: sum over groups of ceil(ops / 256) <= launches + faults / 256
  e->items_cap = e->stage_launch_cap + e->stage_fault_cap / 256 + 1;
  A_(dmalloc(&e->d_items, 2 * e->items_cap));
  A_(dmalloc(&e->d_rowc, e->stage_fault_cap * (1ull + g.S)));
  A_(dmalloc(&e->d_big_pool, 2 * e->big_pool_entries));
  A_(dmalloc(&e->d_big_pool_b, 2 * e->big_pool_entries));
  A_(dmalloc(&e->d_ingest_pool, 2 * e->big_pool_entries));
  A_(dmalloc(&e->d_walk_seen, (uint64_t)e->n_walk_slots * e->walk_hash_cap));
  A_(dmalloc(&e->d_walk_chain, (uint64_t)e->n_walk_slots * e->walk_hash_cap));
  A_(dmalloc(&e->d_walk_tmp, (uint64_t)e->n_walk_slots * tmp_cap));
  A_(dmalloc(&e->d_walk_out, (uint64_t)e->n_walk_slots * g.walk_cap));
  A_(dmalloc(&e->d_anchor_pool, e->anchor_pool_entries));
  A_(dmalloc(&e->d_anchor_range, 2ull * e->anchor_range_cap));
  A_(dmalloc(&e->d_qkern, (uint64_t)e->anchor_range_cap * (g.N + 1)));
  A_(dmalloc(&e->d_qloff, (uint64_t)e->anchor_range_cap * (g.N + 2)));
  A_(dmalloc(&e->d_qeoff, (uint64_t)e->anchor_range_cap * (g.N + 2)));
  A_(dmalloc(&e->d_qgoff, (uint64_t)e->anchor_range_cap * (g.N + 2)));
  A_(dmalloc(&e->d_qrank, e->anchor_range_cap));
  A_(dmalloc(&e->d_qperm, 10ull * e->anchor_range_cap));  // k_chain's class lists (2 NQCLS x queries)
  A_(dmalloc(&e->d_qnk, e->anchor_range_cap));
  A_(dmalloc(&e->d_qbase, e->anchor_range_cap));
  A_(dmalloc(&e->d_bcnt, g.W));
  A_(dmalloc(&e->d_bhold, (uint64_t)g.W * HOLD_MAX));
  A_(dmalloc(&e->d_conf, (uint64_t)g.Emax * CONF_MAX));
  A_(dmalloc(&e->d_conf_n, g.Emax));
  A_(dmalloc(&e->d_wnr, g.Emax));
  A_(dmalloc(&e->d_wnres, g.Emax));
  A_(dmalloc(&e->d_respos, (uint64_t)g.Emax * g.walk_cap));
  // lrm_cap / 32 + 1 (lrm_cap = 4 C + 1024), + slack: k_window_fast bulk-loads whole 16 B
  A_(dmalloc(&e->d_log_bits, 4 * g.C / 32 + 1024 / 32 + 8));
  A_(dmalloc(&e->d_qroff, (uint64_t)e->anchor_range_cap * (g.N + 2)));
  A_(dmalloc(&e->d_qneed, e->anchor_range_cap));
  A_(dmalloc(&e->d_qvb, 2ull * e->anchor_range_cap));
  // copy chunks of one predict call <= out_cap_pairs / 128 + queries x (N + 1); grown by
  // launch_predict when a call's bound exceeds it
  e->chunk_cap = 1u << 20;
  A_(dmalloc(&e->d_chunk_map, e->chunk_cap));
  A_(dmalloc(&e->d_selrec, 3ull * NQCLS * e->anchor_range_cap));
  A_(dmalloc(&e->d_frame_of, g.W));
  A_(dmalloc(&e->d_stamp_of, g.W));
  A_(dmalloc(&e->d_block_of, g.C));
  A_(dmalloc(&e->d_free_bits, (g.C + 31) / 32));
  A_(dmalloc(&e->d_inactive_bits, (g.W + 31) / 32));
  A_(dmalloc(&e->d_res_bits, (g.W + 31) / 32));
  A_(dmalloc(&e->d_lrm_blk, e->lrm_cap));
  A_(dmalloc(&e->d_logpos, g.W));
  A_(dmalloc(&e->d_lrm_stamp, e->lrm_cap));
  A_(dmalloc(&e->d_mig_frames, e->mig_cap));
  A_(dmalloc(&e->d_mig_src, e->mig_cap));
  A_(dmalloc(&e->d_mig_blocks, e->mig_cap));
  A_(dmalloc(&e->d_state, 1));
  A_(cudaMemset(e->d_state, 0, sizeof(DevState)));
  A_(cudaMallocHost((void **)&e->h_state, sizeof(DevState)));
  if (err != cudaSuccess) {
    free_all(e);
    delete e;
    return err == cudaErrorMemoryAllocation ? DUM_ENOMEM : DUM_ECUDA;
  }
  // walker scratch starts empty (NONE) and is kept empty by the walkers
  fill(e->d_walk_seen, (uint64_t)e->n_walk_slots * e->walk_hash_cap, NONE, 0);
  fill(e->d_walk_chain, (uint64_t)e->n_walk_slots * e->walk_hash_cap, NONE, 0);
  fill(e->d_walk_tmp, (uint64_t)e->n_walk_slots * tmp_cap, NONE, 0);
  if (cfg->host_arena) {
    if (cfg->host_arena_bytes < (uint64_t)g.W * DUM_BLOCK_BYTES) {
      free_all(e);
      delete e;
      return DUM_EINVAL;
    }
    void *dp = nullptr;
    if (cudaHostGetDevicePointer(&dp, cfg->host_arena, 0) != cudaSuccess) {
      cudaGetLastError();
      free_all(e);
      delete e;
      return DUM_EINVAL;  // not pinned / not mapped
    }
    e->host_arena = (char *)cfg->host_arena;
    e->host_arena_dev = (char *)dp;
  }
  if (cfg->frame_pool) {
    if (cfg->frame_pool_bytes < (uint64_t)g.C * DUM_BLOCK_BYTES) {
      free_all(e);
      delete e;
      return DUM_EINVAL;
    }
    e->frame_pool = (char *)cfg->frame_pool;
  }
  int rc = reset_state(e, 0);
  if (rc == DUM_OK && cudaDeviceSynchronize() != cudaSuccess) rc = DUM_ECUDA;
  if (rc != DUM_OK) {
    free_all(e);
    delete e;
    return rc;
  }
  *out = e;
  return DUM_OK;
}

int dum_destroy(dum_engine *e) {
  if (!e) return DUM_EINVAL;
  cudaSetDevice(e->device);
  cudaDeviceSynchronize();
  free_all(e);
  delete e;
  return DUM_OK;
}

int dum_reset(dum_engine *e, dum_stream_t stream) {
  if (!e) return DUM_EINVAL;
  cudaSetDevice(e->device);
  return reset_state(e, (cudaStream_t)stream);
}

int dum_record_faults(dum_engine *e, const uint64_t *launch_hash, const uint64_t *launch_off, uint32_t n_launch,
                      const uint32_t *fault_block, uint64_t n_fault, uint32_t *out_exec, uint32_t flags,
                      dum_stream_t stream) {
  if (!e) return DUM_EINVAL;
  if (n_launch == 0) return DUM_OK;
  if (!launch_hash || !launch_off || (n_fault && !fault_block)) return fail(e, DUM_EINVAL, "null input");
  if ((uint64_t)e->n_staged + n_launch > e->stage_launch_cap || e->staged_faults + n_fault > e->stage_fault_cap)
    return fail(e, DUM_ECAPACITY, "staging capacity exceeded: call dum_build_tables or raise max_batch_*");
  if (e->launches + n_launch > 0xFFFFFFFFull) return fail(e, DUM_ECAPACITY, "launch counter exceeds 2^32");
  cudaSetDevice(e->device);
  cudaStream_t s = (cudaStream_t)stream;
  cudaStream_t r = e->rec_s;
  const uint64_t *h = launch_hash, *o = launch_off;
  const uint32_t *f = fault_block;
  if (flags & DUM_HOST_PTRS) {
    if (launch_off[0] != 0 || launch_off[n_launch] != n_fault) return fail(e, DUM_EINVAL, "batch not launch-aligned");
    for (uint32_t i = 0; i < n_launch; ++i)
      if (launch_off[i + 1] < launch_off[i]) return fail(e, DUM_EINVAL, "launch_off not monotone");
    // block ids are checked on the device, as for device pointers (a host pass
    // over the records would read them from DRAM a second time)
  } else if ((reinterpret_cast<uintptr_t>(launch_hash) | reinterpret_cast<uintptr_t>(launch_off)) & 7 ||
             reinterpret_cast<uintptr_t>(fault_block) & 3) {
    return fail(e, DUM_EINVAL, "unaligned pointer");
  }
  // The batch is ingested on the engine's record stream: it waits for the
  // build that last read this staging set (two batches ago), and -- unless
  // the inputs come from the host or the caller declares them ready -- for
  // the work already queued on `stream`; `stream` then waits for the
  // ingest.  The ingest of batch i+1 thereby overlaps the build of batch i
  // (the paper's fault-handling and table-update threads run concurrently,
  // P:L140-L158).
  if (!(flags & (DUM_HOST_PTRS | DUM_INPUTS_READY))) {
    CK(cudaEventRecord(e->ev_s_now, s));
    CK(cudaStreamWaitEvent(r, e->ev_s_now, 0));
  }
  CK(cudaStreamWaitEvent(r, e->ev_stage_free[e->stage_set], 0));
  if (flags & DUM_HOST_PTRS) {
    uint64_t *dh = in_hash(e);
    uint64_t *doff = in_off(e);
    uint32_t *df = in_faults(e);
    CK(cudaMemcpyAsync(dh, launch_hash, 8ull * n_launch, cudaMemcpyHostToDevice, r));
    CK(cudaMemcpyAsync(doff, launch_off, 8ull * (n_launch + 1), cudaMemcpyHostToDevice, r));
    if (n_fault) CK(cudaMemcpyAsync(df, fault_block, 4ull * n_fault, cudaMemcpyHostToDevice, r));
    h = dh;
    o = doff;
    f = df;
  }
  CK(launch_record(e, h, o, n_launch, f, n_fault, out_exec, r));
  CK(cudaEventRecord(e->ev_rec, r));
  CK(cudaStreamWaitEvent(s, e->ev_rec, 0));
  e->n_staged += n_launch;
  e->staged_faults += n_fault;
  e->launches += n_launch;
  return DUM_OK;
}

int dum_build_tables(dum_engine *e, dum_stream_t stream) {
  if (!e) return DUM_EINVAL;
  cudaSetDevice(e->device);
  if (e->n_staged) {
    CK(cudaStreamWaitEvent((cudaStream_t)stream, e->ev_rec, 0));
    CK(launch_build(e, (cudaStream_t)stream));
    // this staging set is free once the build has run; the next batch goes to the other set
    CK(cudaEventRecord(e->ev_stage_free[e->stage_set], (cudaStream_t)stream));
    e->stage_set ^= 1;
    const uint64_t L = e->stage_launch_cap, F = e->stage_fault_cap, k = (uint64_t)e->stage_set;
    e->d_stage_hash = static_cast<uint64_t *>(e->stage_base[0]) + k * L;
    e->d_stage_norm = static_cast<uint32_t *>(e->stage_base[1]) + k * F;
    e->d_stage_cnt = static_cast<uint32_t *>(e->stage_base[2]) + k * L;
    e->d_stage_exec = static_cast<uint32_t *>(e->stage_base[3]) + k * L;
    e->d_stage_slot = static_cast<uint32_t *>(e->stage_base[4]) + k * L;
    e->d_stage_off = static_cast<uint64_t *>(e->stage_base[5]) + k * L;
  }
  e->n_staged = 0;
  e->staged_faults = 0;
  e->built_launches = e->launches;
  return DUM_OK;
}

__global__ void k_step_shift(uint32_t *ex, uint32_t n) {
  // the last three exec IDs of [previous three | batch] become the next step's history
  if (threadIdx.x == 0) {
    const uint32_t a = ex[n], b = ex[n + 1], c = ex[n + 2];
    ex[0] = a;
    ex[1] = b;
    ex[2] = c;
  }
}

// The selection's per-walk residency facts depend only on the residency and
// the walks of the previous build: issued on the second side stream so that
// they overlap the ingest of the step; launch_predict joins them.
static cudaError_t fork_walk_res(dum_engine *e, cudaStream_t s) {
  cudaError_t err;
  if ((err = cudaEventRecord(e->ev_fork2, s)) != cudaSuccess) return err;
  if ((err = cudaStreamWaitEvent(e->side2, e->ev_fork2, 0)) != cudaSuccess) return err;
  if ((err = launch_walk_res(e, e->side2)) != cudaSuccess) return err;
  if ((err = cudaEventRecord(e->ev_wres, e->side2)) != cudaSuccess) return err;
  e->wres_pending = true;
  return cudaSuccess;
}

// dum_step as one CUDA graph per (batch size, staging set, outputs): the
// inputs go to the engine's fixed upload buffers outside the graph, then the
// whole step -- ingest, queries, predict + select, build, history shift, every
// side-stream fork joined -- replays with one cudaGraphLaunch.  The values a
// step changes (launch index base, pools, counts) live on the device.
static int step_graph(dum_engine *e, const uint64_t *launch_hash, const uint64_t *launch_off, uint32_t n_launch,
                      const uint32_t *fault_block, uint64_t n_fault, uint32_t flags, uint32_t degree,
                      uint32_t *out_pairs, uint64_t out_cap_pairs, uint64_t *out_range, uint32_t *out_kern_off,
                      uint32_t *out_chain, uint64_t *out_needed, uint32_t *out_writeback, uint32_t *out_invalidate,
                      uint64_t sel_cap, uint64_t *sel_range, uint64_t *sel_needed, cudaStream_t s) {
  if (!launch_hash || !launch_off || (n_fault && !fault_block) || !out_range || !sel_range)
    return fail(e, DUM_EINVAL, "null argument");
  if (n_launch > e->stage_launch_cap || n_fault > e->stage_fault_cap)
    return fail(e, DUM_ECAPACITY, "staging capacity exceeded: raise max_batch_*");
  if (e->launches + n_launch > 0xFFFFFFFFull) return fail(e, DUM_ECAPACITY, "launch counter exceeds 2^32");
  if (reinterpret_cast<uintptr_t>(out_pairs) & 7) return fail(e, DUM_EINVAL, "out_pairs must be 8-byte aligned");
  cudaSetDevice(e->device);
  const cudaMemcpyKind kind = (flags & DUM_HOST_PTRS) ? cudaMemcpyHostToDevice : cudaMemcpyDeviceToDevice;
  if (flags & DUM_HOST_PTRS) {
    if (launch_off[0] != 0 || launch_off[n_launch] != n_fault) return fail(e, DUM_EINVAL, "batch not launch-aligned");
    for (uint32_t i = 0; i < n_launch; ++i)
      if (launch_off[i + 1] < launch_off[i]) return fail(e, DUM_EINVAL, "launch_off not monotone");
  }
  // the batch into this staging set's upload buffers, on the record stream:
  // after the replay that last read them (two steps ago) -- and, for device
  // inputs, after the caller's stream -- so that it overlaps the previous step
  cudaStream_t caller = s;
  const int set = e->stage_set;
  CK(cudaEventRecord(e->ev_s_now, caller));
  if (!(flags & DUM_HOST_PTRS)) CK(cudaStreamWaitEvent(e->rec_s, e->ev_s_now, 0));
  CK(cudaStreamWaitEvent(e->rec_s, e->ev_stage_free[set], 0));
  CK(cudaMemcpyAsync(in_hash(e), launch_hash, 8ull * n_launch, kind, e->rec_s));
  CK(cudaMemcpyAsync(in_off(e), launch_off, 8ull * (n_launch + 1), kind, e->rec_s));
  if (n_fault) CK(cudaMemcpyAsync(in_faults(e), fault_block, 4ull * n_fault, kind, e->rec_s));
  CK(cudaEventRecord(e->ev_rec, e->rec_s));
  // the graph runs on the engine's own (capturable, non-blocking) stream, ordered
  // after the caller's stream (and the upload) and before it again
  s = e->graph_s;
  CK(cudaStreamWaitEvent(s, e->ev_s_now, 0));
  // side-stream work of an earlier uncaptured call (jump tables, walk index,
  // predict's side kernels) is finished before the graph starts
  CK(cudaStreamWaitEvent(s, e->ev_join, 0));
  CK(cudaStreamWaitEvent(s, e->ev_widx, 0));
  CK(cudaStreamWaitEvent(s, e->ev_join2, 0));
  CK(cudaStreamWaitEvent(s, e->ev_rec, 0));
  if (e->commit_inflight) {  // an uncaptured build's walk commit (side stream)
    CK(cudaStreamWaitEvent(s, e->ev_commit, 0));
    e->commit_inflight = false;
  }
  const uint64_t key[12] = {n_launch, (uint64_t)e->stage_set, degree, (uint64_t)out_pairs, out_cap_pairs,
                            (uint64_t)out_range, (uint64_t)out_kern_off, (uint64_t)out_chain, (uint64_t)out_needed,
                            (uint64_t)out_writeback ^ ((uint64_t)out_invalidate << 1), sel_cap,
                            (uint64_t)sel_range ^ ((uint64_t)sel_needed << 1)};
  cudaGraphExec_t exec = nullptr;
  for (auto &g : e->step_graphs)
    if (std::memcmp(g.key, key, sizeof key) == 0) exec = g.exec;
  if (!exec) {
    // the chunk map of this output capacity is grown before the capture
    const uint64_t bound = out_cap_pairs / CHUNK_B + (uint64_t)n_launch * (e->g.N + 1) + 1;
    if (bound > e->chunk_cap) {
      CK(cudaDeviceSynchronize());
      CK(cudaFree(e->d_chunk_map));
      e->d_chunk_map = nullptr;
      CK(cudaMalloc((void **)&e->d_chunk_map, 16 * bound));
      e->chunk_cap = bound;
    }
    SelectOut so = make_select_out(e, out_writeback, out_invalidate, sel_cap, sel_range);
    cudaGraph_t graph = nullptr;
    // fork / join events recorded inside a capture become graph edges and may
    // not be waited on outside it: the capture uses its own set
    cudaEvent_t *evs[] = {&e->ev_fork, &e->ev_join, &e->ev_fork2, &e->ev_join2, &e->ev_widx,
                          &e->ev_wres, &e->ev_fork4, &e->ev_bhead, &e->ev_wslow_fork, &e->ev_wslow};
    constexpr int NEV = sizeof(evs) / sizeof(evs[0]);
    if (!e->cap_events_ready) {
      for (int i = 0; i < NEV; ++i) CK(cudaEventCreateWithFlags(&e->cap_ev[i], cudaEventDisableTiming));
      e->cap_events_ready = true;
    }
    cudaEvent_t real[NEV];
    for (int i = 0; i < NEV; ++i) {
      real[i] = *evs[i];
      *evs[i] = e->cap_ev[i];
    }
    e->capturing = true;
    const uint32_t ns0 = e->n_staged;
    const uint64_t sf0 = e->staged_faults;
    e->n_staged = 0;
    e->staged_faults = 0;
    // an error left by an earlier uncaptured launch is not this capture's
    const cudaError_t pending = cudaGetLastError();
    if (pending != cudaSuccess) {
      e->last_error = std::string("pending before a dum_step capture: ") + cudaGetErrorString(pending);
      return DUM_ECUDA;
    }
    const char *stage = "begin capture";
    cudaError_t err = cudaStreamBeginCapture(s, cudaStreamCaptureModeThreadLocal);
    // the previous step's walk index (a replayed build leaves it to this step),
    // beside the residency facts and the ingest
    if (err == cudaSuccess && (stage = "jump tables", true)) {
      // the previous build's jump tables (a captured build leaves them to the
      // next step), on the side stream beside the ingest; k_chain joins them
      cudaEventRecord(e->ev_fork, s);
      cudaStreamWaitEvent(e->side, e->ev_fork, 0);
      err = launch_jump_tables(e, e->side);
      // ... and its walks (exact windows: k_chain is their first reader; a
      // fast-window build published them itself, for the walk index)
      if (err == cudaSuccess && !e->fast_windows) err = launch_walk_commit(e, e->side);
      cudaEventRecord(e->ev_join, e->side);
    }
    if (err == cudaSuccess && (stage = "walk index", true)) err = launch_walk_index(e, s);
    if (err == cudaSuccess && (stage = "walk residency", true)) err = fork_walk_res(e, s);
    if (err == cudaSuccess && (stage = "record", true))
      err = launch_record(e, in_hash(e), in_off(e), n_launch, in_faults(e), e->stage_fault_cap,
                          e->d_step_exec + 3, s);
    if (err == cudaSuccess && (stage = "queries", true))
      err = launch_make_queries(e, e->d_step_exec, 3 + n_launch, 3, degree, e->d_step_q, s);
    e->bhead_n = n_launch;  // the build goes beside the predict kernels
    if (err == cudaSuccess && (stage = "predict + build", true))
      err = launch_predict(e, e->d_step_q, n_launch, out_pairs, out_cap_pairs, out_range, out_kern_off, out_chain,
                           out_needed, &so, sel_needed, s);
    e->bhead_n = 0;
    e->n_staged = n_launch;
    e->staged_faults = e->stage_fault_cap;
    if (err == cudaSuccess && (stage = "build commit", true)) err = launch_build(e, s);
    if (err == cudaSuccess) {
      k_step_shift<<<1, 32, 0, s>>>(e->d_step_exec, n_launch);
      // every side stream joins the step: the next replay may start at once
      cudaStreamWaitEvent(s, e->ev_join, 0);
      cudaStreamWaitEvent(s, e->ev_widx, 0);
      err = cudaGetLastError();
    }
    const cudaError_t err2 = cudaStreamEndCapture(s, &graph);
    e->capturing = false;
    for (int i = 0; i < NEV; ++i) *evs[i] = real[i];
    e->n_staged = ns0;
    e->staged_faults = sf0;
    if (err == cudaSuccess) err = err2;
    if (err == cudaSuccess) err = cudaGraphInstantiate(&exec, graph, cudaGraphInstantiateFlagUseNodePriority);
    if (graph) cudaGraphDestroy(graph);
    if (err != cudaSuccess) {
      // not capturable here: say so once, drop to the one-call path for good
      cudaGetLastError();
      fprintf(stderr, "libdeepum_b200: dum_step graph capture failed at %s (%s); steps run uncaptured\n", stage,
              cudaGetErrorString(err));
      e->graph_steps = false;
      e->wres_pending = false;
      e->last_error = std::string("dum_step graph capture: ") + cudaGetErrorString(err);
      CK(cudaEventRecord(e->ev_graph, s));
      CK(cudaStreamWaitEvent(caller, e->ev_graph, 0));
      return DUM_ECUDA;
    }
    dum_engine::StepGraph sg;
    std::memcpy(sg.key, key, sizeof key);
    sg.exec = exec;
    e->step_graphs.push_back(sg);
  }
  CK(cudaGraphLaunch(exec, s));
  e->widx_stale = true;  // the replayed build's walk index is built by the next step
  e->jump_stale = true;  // and so are its jump tables
  e->commit_stale = !e->fast_windows;  // and, with exact windows, the publishing of its walks
  CK(cudaEventRecord(e->ev_graph, s));
  CK(cudaEventRecord(e->ev_stage_free[set], s));  // this set's staging and upload buffers are free again
  CK(cudaStreamWaitEvent(caller, e->ev_graph, 0));
  // host bookkeeping of the replayed step (as dum_record_faults + dum_build_tables)
  e->launches += n_launch;
  e->built_launches = e->launches;
  e->stage_set ^= 1;
  const uint64_t L = e->stage_launch_cap, F = e->stage_fault_cap, k = (uint64_t)e->stage_set;
  e->d_stage_hash = static_cast<uint64_t *>(e->stage_base[0]) + k * L;
  e->d_stage_norm = static_cast<uint32_t *>(e->stage_base[1]) + k * F;
  e->d_stage_cnt = static_cast<uint32_t *>(e->stage_base[2]) + k * L;
  e->d_stage_exec = static_cast<uint32_t *>(e->stage_base[3]) + k * L;
  e->d_stage_slot = static_cast<uint32_t *>(e->stage_base[4]) + k * L;
  e->d_stage_off = static_cast<uint64_t *>(e->stage_base[5]) + k * L;
  e->kernel_launches += 40;  // approximate node count of a step graph
  return DUM_OK;
}

int dum_set_step_graphs(dum_engine *e, int enable) {
  if (!e) return DUM_EINVAL;
  e->graph_steps = enable != 0;
  return DUM_OK;
}

int dum_step(dum_engine *e, const uint64_t *launch_hash, const uint64_t *launch_off, uint32_t n_launch,
             const uint32_t *fault_block, uint64_t n_fault, uint32_t flags, uint32_t degree, uint32_t *out_pairs,
             uint64_t out_cap_pairs, uint64_t *out_range, uint32_t *out_kern_off, uint32_t *out_chain,
             uint64_t *out_needed, uint32_t *out_writeback, uint32_t *out_invalidate, uint64_t sel_cap,
             uint64_t *sel_range, uint64_t *sel_needed, dum_stream_t stream) {
  if (!e) return DUM_EINVAL;
  if (n_launch == 0) return DUM_OK;
  if (e->n_staged) return fail(e, DUM_ESTATE, "dum_step: a batch is already staged (call dum_build_tables)");
  if (n_launch > e->anchor_range_cap) return fail(e, DUM_EINVAL, "too many launches in one step (max 65536)");
  // graph mode: the first step of a shape runs uncaptured (first-use attribute /
  // occupancy queries of the launchers are not capturable), later ones replay
  if (e->graph_steps && e->step_warm) {
    const int rc = step_graph(e, launch_hash, launch_off, n_launch, fault_block, n_fault, flags, degree, out_pairs,
                              out_cap_pairs, out_range, out_kern_off, out_chain, out_needed, out_writeback,
                              out_invalidate, sel_cap, sel_range, sel_needed, (cudaStream_t)stream);
    if (rc != DUM_ECUDA || e->graph_steps) return rc;  // (a failed capture turned graph mode off: run it below)
  }
  e->step_warm = e->graph_steps;
  cudaSetDevice(e->device);
  CK(fork_walk_res(e, (cudaStream_t)stream));
  int rc = dum_record_faults(e, launch_hash, launch_off, n_launch, fault_block, n_fault, e->d_step_exec + 3, flags,
                             stream);
  if (rc) return rc;
  cudaStream_t s = (cudaStream_t)stream;
  CK(launch_make_queries(e, e->d_step_exec, 3 + n_launch, 3, degree, e->d_step_q, s));
  e->bhead_n = e->n_staged;  // the build's head goes beside the predict kernels
  rc = dum_predict_select(e, e->d_step_q, n_launch, out_pairs, out_cap_pairs, out_range, out_kern_off, out_chain,
                          out_needed, out_writeback, out_invalidate, sel_cap, sel_range, sel_needed, stream);
  e->bhead_n = 0;
  if (rc) {
    e->bhead_pending = false;
    return rc;
  }
  rc = dum_build_tables(e, stream);
  if (rc) return rc;
  k_step_shift<<<1, 32, 0, s>>>(e->d_step_exec, n_launch);
  e->kernel_launches += 1;
  CK(cudaGetLastError());
  return DUM_OK;
}

int dum_make_queries(dum_engine *e, const uint32_t *exec_seq, uint32_t n_seq, uint32_t first, uint32_t degree,
                     dum_query *out, dum_stream_t stream) {
  if (!e || (!exec_seq && n_seq) || (!out && first < n_seq)) return DUM_EINVAL;
  cudaSetDevice(e->device);
  CK(launch_make_queries(e, exec_seq, n_seq, first, degree, out, (cudaStream_t)stream));
  return DUM_OK;
}

int dum_predict_prefetch(dum_engine *e, const dum_query *q, uint32_t n_query, uint32_t *out_pairs,
                         uint64_t out_cap_pairs, uint64_t *out_range, uint32_t *out_kern_off, uint32_t *out_chain,
                         uint64_t *out_needed, dum_stream_t stream) {
  if (!e) return DUM_EINVAL;
  if (n_query == 0) return DUM_OK;
  if (!q || !out_range || (!out_pairs && out_cap_pairs)) return fail(e, DUM_EINVAL, "null argument");
  if (n_query > e->anchor_range_cap) return fail(e, DUM_EINVAL, "too many queries in one call (max 65536)");
  if (reinterpret_cast<uintptr_t>(out_pairs) & 7) return fail(e, DUM_EINVAL, "out_pairs must be 8-byte aligned");
  cudaSetDevice(e->device);
  CK(launch_predict(e, q, n_query, out_pairs, out_cap_pairs, out_range, out_kern_off, out_chain, out_needed,
                    nullptr, nullptr, (cudaStream_t)stream));
  return DUM_OK;
}

int dum_predict_select(dum_engine *e, const dum_query *q, uint32_t n_query, uint32_t *out_pairs,
                       uint64_t out_cap_pairs, uint64_t *out_range, uint32_t *out_kern_off, uint32_t *out_chain,
                       uint64_t *out_needed, uint32_t *out_writeback, uint32_t *out_invalidate, uint64_t sel_cap,
                       uint64_t *sel_range, uint64_t *sel_needed, dum_stream_t stream) {
  if (!e) return DUM_EINVAL;
  if (n_query == 0) return DUM_OK;
  if (!q || !out_range || !sel_range || (!out_pairs && out_cap_pairs)) return fail(e, DUM_EINVAL, "null argument");
  if (n_query > e->anchor_range_cap) return fail(e, DUM_EINVAL, "too many queries in one call (max 65536)");
  if (reinterpret_cast<uintptr_t>(out_pairs) & 7) return fail(e, DUM_EINVAL, "out_pairs must be 8-byte aligned");
  cudaSetDevice(e->device);
  SelectOut so = make_select_out(e, out_writeback, out_invalidate, sel_cap, sel_range);
  CK(launch_predict(e, q, n_query, out_pairs, out_cap_pairs, out_range, out_kern_off, out_chain, out_needed, &so,
                    sel_needed, (cudaStream_t)stream));
  return DUM_OK;
}

int dum_select_evictions(dum_engine *e, const uint64_t *query_range, const uint32_t *pairs, uint32_t n_query,
                         const dum_query *queries, uint32_t *out_writeback, uint32_t *out_invalidate,
                         uint64_t out_cap, uint64_t *out_range, uint64_t *out_needed, dum_stream_t stream) {
  if (!e) return DUM_EINVAL;
  if (n_query == 0) return DUM_OK;
  if (!query_range || !out_range) return fail(e, DUM_EINVAL, "null argument");
  cudaSetDevice(e->device);
  CK(launch_select(e, query_range, pairs, n_query, queries, out_writeback, out_invalidate, out_cap, out_range,
                   out_needed, (cudaStream_t)stream));
  return DUM_OK;
}

int dum_simulate(dum_engine *e, const uint64_t *launch_hash, uint32_t n_launch, const uint64_t *acc_off,
                 const uint32_t *acc_blk, uint32_t n_kernels, uint32_t degree, uint32_t flags, dum_sim_stats *stats,
                 dum_stream_t stream) {
  if (!e) return DUM_EINVAL;
  if (n_launch == 0) return DUM_OK;
  if (!launch_hash || !acc_off || !acc_blk || !stats || n_kernels == 0 || flags > 7)
    return fail(e, DUM_EINVAL, "null argument / bad flags");
  if (e->n_staged) return fail(e, DUM_ESTATE, "dum_simulate needs an empty staging area (call dum_build_tables)");
  for (uint32_t j = 0; j < n_kernels; ++j)
    if (acc_off[j + 1] < acc_off[j] || acc_off[j + 1] - acc_off[j] > 8192)
      return fail(e, DUM_EINVAL, "acc_off not monotone or a launch with more than 8192 accesses");
  if (e->launches + n_launch > 0xFFFFFFFFull) return fail(e, DUM_ECAPACITY, "launch counter exceeds 2^32");
  cudaSetDevice(e->device);
  cudaStream_t s = (cudaStream_t)stream;
  // the ingest stream's pending work (a record call before) is ordered before the loop
  CK(cudaStreamWaitEvent(s, e->ev_rec, 0));
  CK(launch_simulate(e, launch_hash, n_launch, acc_off, acc_blk, n_kernels, degree, flags, stats, s));
  return DUM_OK;
}

int dum_mark_inactive(dum_engine *e, const uint32_t *blocks, uint32_t n, int inactive, dum_stream_t stream) {
  if (!e || (n && !blocks)) return DUM_EINVAL;
  cudaSetDevice(e->device);
  CK(launch_mark_inactive(e, blocks, n, inactive, (cudaStream_t)stream));
  return DUM_OK;
}

int dum_load_residency(dum_engine *e, const uint32_t *lrm_blocks, uint32_t n_resident, dum_stream_t stream) {
  if (!e || (n_resident && !lrm_blocks)) return DUM_EINVAL;
  if (n_resident > e->g.C) return fail(e, DUM_ECAPACITY, "more resident blocks than frames");
  cudaSetDevice(e->device);
  CK(launch_load_residency(e, lrm_blocks, n_resident, (cudaStream_t)stream));
  return DUM_OK;
}

int dum_migrate_blocks(dum_engine *e, dum_dir dir, const uint32_t *blocks_or_src, const uint32_t *dst_frames,
                       uint32_t n, uint32_t method, dum_stream_t stream) {
  if (!e) return DUM_EINVAL;
  if ((int)dir < 0 || (int)dir > 3 || method > 3) return fail(e, DUM_EINVAL, "bad direction or method");
  if (n > e->g.C) return fail(e, DUM_EINVAL, "list longer than the frame count");
  if (dir != DUM_D2D && n && !blocks_or_src) return fail(e, DUM_EINVAL, "null block list");
  if (dir == DUM_D2D && blocks_or_src && !dst_frames) return fail(e, DUM_EINVAL, "D2D needs dst_frames");
  if (dir != DUM_INVALIDATE && (!e->frame_pool || (dir != DUM_D2D && !e->host_arena)))
    return fail(e, DUM_ESTATE, "metadata-only engine: no host arena / frame pool configured");
  if (n == 0 && !(dir == DUM_D2D && !blocks_or_src)) return DUM_OK;
  cudaSetDevice(e->device);
  CK(launch_migrate(e, (int)dir, blocks_or_src, dst_frames, n, method, (cudaStream_t)stream));
  return DUM_OK;
}

int dum_block_checksums(dum_engine *e, int where, const uint32_t *ids, uint32_t n, uint64_t *out,
                        dum_stream_t stream) {
  if (!e || (n && (!ids || !out))) return DUM_EINVAL;
  if ((where == 0 && !e->frame_pool) || (where == 1 && !e->host_arena) || where < 0 || where > 1)
    return fail(e, DUM_ESTATE, "no such arena");
  cudaSetDevice(e->device);
  CK(launch_checksums(e, where, ids, n, out, (cudaStream_t)stream));
  return DUM_OK;
}

int dum_sync(dum_engine *e, dum_stream_t stream, uint64_t *needed) {
  if (!e) return DUM_EINVAL;
  cudaSetDevice(e->device);
  CK(cudaStreamSynchronize((cudaStream_t)stream));
  CK(cudaMemcpy(e->h_state, e->d_state, sizeof(DevState), cudaMemcpyDeviceToHost));
  const uint32_t err = e->h_state->err;
  if (needed) *needed = e->h_state->needed;
  if (err) {
    CK(cudaMemset(&e->d_state->err, 0, 4));
    CK(cudaMemset(&e->d_state->needed, 0, 8));
    if (err & ERR_EINVAL) return fail(e, DUM_EINVAL, "device-side validation failed (block id / list / alignment)");
    return fail(e, DUM_ECAPACITY, "device-side capacity exceeded (see *needed)");
  }
  return DUM_OK;
}

int dum_get_stats(dum_engine *e, dum_stats *out) {
  if (!e || !out) return DUM_EINVAL;
  cudaSetDevice(e->device);
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(e->h_state, e->d_state, sizeof(DevState), cudaMemcpyDeviceToHost));
  out->num_exec = e->h_state->E;
  out->corr_records = e->h_state->corr_used;
  out->free_frames = e->h_state->free_count;
  out->staged_launches = e->n_staged;
  out->launches = e->launches;
  out->staged_faults = e->staged_faults;
  out->slow_walks = e->h_state->n_slow;
  out->n_resident = e->h_state->n_resident;
  out->guard_line = e->h_state->dbg_line;
  out->guard_val = e->h_state->dbg_val;
  return DUM_OK;
}

const char *dum_last_error(const dum_engine *e) { return e ? e->last_error.c_str() : "null engine"; }

int dum_read_counters(dum_engine *e, uint64_t out[DUM_NCOUNTERS], int reset) {
  if (!e || !out) return DUM_EINVAL;
  cudaSetDevice(e->device);
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(out, e->d_state->ctr, sizeof(uint64_t) * DUM_NCOUNTERS, cudaMemcpyDeviceToHost));
  if (reset) CK(cudaMemset(e->d_state->ctr, 0, sizeof(uint64_t) * DUM_NCOUNTERS));
  return DUM_OK;
}

int dum_set_copy_sms(dum_engine *e, uint32_t n_sms) {
  if (!e) return DUM_EINVAL;
  e->copy_sms = n_sms;
  return DUM_OK;
}

int dum_set_counting(dum_engine *e, int enable) {
  if (!e) return DUM_EINVAL;
  cudaSetDevice(e->device);
  const uint32_t v = enable ? 1u : 0u;
  // stream-ordered with the caller's legacy default stream and every engine stream (a plain store)
  CK(cudaDeviceSynchronize());
  CK(cudaMemcpy(&e->d_state->counting, &v, 4, cudaMemcpyHostToDevice));
  return DUM_OK;
}

int dum_set_timing(dum_engine *e, int enable) {
  if (!e) return DUM_EINVAL;
  e->timing = enable != 0;
  return DUM_OK;
}

int dum_read_timing(dum_engine *e, double ms[DUM_NTIMERS], uint64_t count[DUM_NTIMERS], int reset) {
  if (!e) return DUM_EINVAL;
  cudaSetDevice(e->device);
  CK(cudaDeviceSynchronize());
  for (auto &t : e->pending) {
    float x = 0.f;
    CK(cudaEventElapsedTime(&x, t.a, t.b));
    e->t_ms[t.id] += x;
    e->t_cnt[t.id] += 1;
    e->event_pool.push_back(t.a);
    e->event_pool.push_back(t.b);
  }
  e->pending.clear();
  for (int i = 0; i < DUM_NTIMERS; ++i) {
    if (ms) ms[i] = e->t_ms[i];
    if (count) count[i] = e->t_cnt[i];
    if (reset) {
      e->t_ms[i] = 0;
      e->t_cnt[i] = 0;
    }
  }
  return DUM_OK;
}

int dum_read_timeline(dum_engine *e, int cap, int *ids, float *t0, float *t1) {
  if (!e || cap < 0 || (cap && (!ids || !t0 || !t1))) return DUM_EINVAL;
  cudaSetDevice(e->device);
  CK(cudaDeviceSynchronize());
  int n = 0;
  for (auto &t : e->pending) {
    float x = 0.f, a = 0.f, b = 0.f;
    CK(cudaEventElapsedTime(&x, t.a, t.b));
    CK(cudaEventElapsedTime(&a, e->pending[0].a, t.a));
    CK(cudaEventElapsedTime(&b, e->pending[0].a, t.b));
    e->t_ms[t.id] += x;
    e->t_cnt[t.id] += 1;
    if (n < cap) {
      ids[n] = t.id;
      t0[n] = a;
      t1[n] = b;
      ++n;
    }
  }
  for (auto &t : e->pending) {
    e->event_pool.push_back(t.a);
    e->event_pool.push_back(t.b);
  }
  e->pending.clear();
  return n;
}

uint64_t dum_kernel_launches(const dum_engine *e) { return e ? e->kernel_launches : 0; }

int dum_host_ptr_kind(const void *p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return -1;
  }
  return (int)a.type;
}

// ---------------------------------------------------------------------------
// canonical dump (host-side canonicalisation of a device snapshot)
// ---------------------------------------------------------------------------
static void put32(std::vector<uint8_t> &o, uint32_t v) {
  const size_t n = o.size();
  o.resize(n + 4);
  std::memcpy(o.data() + n, &v, 4);
}
static void put64(std::vector<uint8_t> &o, uint64_t v) {
  const size_t n = o.size();
  o.resize(n + 8);
  std::memcpy(o.data() + n, &v, 8);
}

int dum_dump_state(dum_engine *e, uint32_t what, void *host_buf, uint64_t cap, uint64_t *needed) {
  if (!e) return DUM_EINVAL;
  cudaSetDevice(e->device);
  if (e->commit_stale) CK(launch_walk_commit(e, e->graph_s));  // the last replayed build's walks
  CK(cudaDeviceSynchronize());
  DevState st;
  CK(cudaMemcpy(&st, e->d_state, sizeof(st), cudaMemcpyDeviceToHost));
  const Geo &g = e->g;
  const uint32_t E = st.E;
  std::vector<uint8_t> o;
  if (what & DUM_DUMP_EXEC) {
    std::vector<uint64_t> h(E);
    if (E) CK(cudaMemcpy(h.data(), e->d_exec_hash, 8ull * E, cudaMemcpyDeviceToHost));
    put32(o, E);
    for (auto x : h) put64(o, x);
  }
  if (what & DUM_DUMP_CORR) {
    std::vector<CorrSlot> c(e->corr_cap);
    CK(cudaMemcpy(c.data(), e->d_corr, sizeof(CorrSlot) * e->corr_cap, cudaMemcpyDeviceToHost));
    std::vector<std::vector<const CorrSlot *>> per(E);
    for (auto &sl : c)
      if (sl.key[0] != NONE && sl.key[0] < E) per[sl.key[0]].push_back(&sl);
    for (uint32_t x = 0; x < E; ++x) {
      auto &v = per[x];
      std::sort(v.begin(), v.end(), [](const CorrSlot *a, const CorrSlot *b) { return a->first < b->first; });
      put32(o, (uint32_t)v.size());
      for (auto *sl : v) {
        put32(o, sl->key[1]);
        put32(o, sl->key[2]);
        put32(o, sl->key[3]);
        put32(o, (uint32_t)(sl->last & 0xFFFFFFFFull));
      }
    }
  }
  if (what & DUM_DUMP_BLK) {
    std::vector<uint32_t> t((uint64_t)g.R * g.stride), se(2ull * std::max<uint32_t>(E, 1));
    if (E) CK(cudaMemcpy(se.data(), e->d_start_end, 8ull * E, cudaMemcpyDeviceToHost));
    for (uint32_t x = 0; x < E; ++x) {
      CK(cudaMemcpy(t.data(), e->d_tbl + (uint64_t)x * g.R * g.stride, 4ull * g.R * g.stride,
                    cudaMemcpyDeviceToHost));
      const size_t n = o.size();
      o.resize(n + 4ull * g.R * g.set_u32);
      uint8_t *dst = o.data() + n;
      for (uint32_t r = 0; r < g.R; ++r) std::memcpy(dst + 4ull * r * g.set_u32, &t[(uint64_t)r * g.stride], 4ull * g.set_u32);
      put32(o, se[2 * x]);
      put32(o, se[2 * x + 1]);
    }
  }
  if (what & DUM_DUMP_WALK) {
    std::vector<uint32_t> len(std::max<uint32_t>(E, 1));
    if (E) CK(cudaMemcpy(len.data(), e->d_walk_len, 4ull * E, cudaMemcpyDeviceToHost));
    std::vector<uint32_t> w;
    for (uint32_t x = 0; x < E; ++x) {
      w.resize(len[x]);
      if (len[x])
        CK(cudaMemcpy(w.data(), e->d_walk + (uint64_t)x * g.walk_cap, 4ull * len[x], cudaMemcpyDeviceToHost));
      put32(o, len[x]);
      for (auto b : w) put32(o, b);
    }
  }
  if (what & DUM_DUMP_RES) {
    std::vector<uint32_t> bof(g.C), fof(g.W), sof(g.W);
    CK(cudaMemcpy(bof.data(), e->d_block_of, 4ull * g.C, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(fof.data(), e->d_frame_of, 4ull * g.W, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(sof.data(), e->d_stamp_of, 4ull * g.W, cudaMemcpyDeviceToHost));
    const uint32_t nlog = st.lrm_tail - st.lrm_head;
    std::vector<uint32_t> lb(nlog), ls(nlog);
    if (nlog) {
      CK(cudaMemcpy(lb.data(), e->d_lrm_blk + st.lrm_head, 4ull * nlog, cudaMemcpyDeviceToHost));
      CK(cudaMemcpy(ls.data(), e->d_lrm_stamp + st.lrm_head, 4ull * nlog, cudaMemcpyDeviceToHost));
    }
    put32(o, g.C);
    for (auto b : bof) put32(o, b);
    std::vector<uint32_t> lrm;
    for (uint32_t i = 0; i < nlog; ++i) {
      const uint32_t b = lb[i] & 0x7FFFFFFFu;
      if (b < g.W && fof[b] != NONE && sof[b] == ls[i]) lrm.push_back(b);
    }
    put32(o, (uint32_t)lrm.size());
    for (auto b : lrm) put32(o, b);
  }
  if (what & DUM_DUMP_HIST) {
    for (int q = 0; q < 4; ++q) put32(o, st.hist[q]);
    put64(o, e->launches);
  }
  if (needed) *needed = o.size();
  if (o.size() > cap) return fail(e, DUM_ECAPACITY, "dump buffer too small");
  if (!o.empty()) std::memcpy(host_buf, o.data(), o.size());
  return DUM_OK;
}

}  // extern "C"
