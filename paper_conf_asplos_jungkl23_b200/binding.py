"""ctypes binding of include/deepum_b200.h (same names, argument marshalling
only).  Device buffers are torch CUDA tensors; uint32 / uint64 data travel in
int32 / int64 tensors with identical bits."""
from __future__ import annotations

import ctypes
import os
from typing import Optional, Tuple

import numpy as np
import torch

HERE = os.path.dirname(os.path.abspath(__file__))
_LIBPATH = os.environ.get("DUM_LIB") or os.path.join(HERE, "libdeepum_b200.so")

DUM_NONE = NONE = 0xFFFFFFFF
DUM_INPUTS_READY = 2
DUM_HOST_PTRS = 0x1
DUM_CFG_SEQ_WALKS = 0x1
DUM_CFG_FAST_WINDOWS = 0x2
SIM_PREFETCH, SIM_PREEVICT, SIM_INVALIDATE = 0x1, 0x2, 0x4
SIM_FIELDS = ("faults", "demand_wb", "demand_inv", "pre_wb", "pre_inv", "prefetched")
DUMP_EXEC, DUMP_CORR, DUMP_BLK, DUMP_WALK, DUMP_RES, DUMP_HIST = 1, 2, 4, 8, 16, 32
H2D, D2H, INVALIDATE, D2D = 0, 1, 2, 3
NCOUNTERS, NTIMERS = 40, 24
CTR = {n: i for i, n in enumerate(["RAW_RECORDS", "NORM_RECORDS", "LAUNCHES", "CORR_UPSERTS", "EXEC_BUILT", "OPS",
                                   "SETS", "WALK_ROWS", "WALK_OUT", "QUERIES", "CHAIN", "GATHERED", "EMITTED",
                                   "SEL_WINDOW", "SEL_SCANNED", "SEL_VICTIMS", "MIG_BLOCKS", "RUNS",
                                   "Q_NODUP", "Q_DUP", "Q_FALLBACK", "WALK_PREFIX", "WALK_DEDUPE", "WALK_SLOW",
                                   "Q_FAST", "ANCHOR_WALKS", "INGEST_DUP", "Q_SLOW", "FAST_EMITTED", "FAST_SCANNED",
                                   "FAST_VICTIMS", "SLOW_CONFLICT", "SLOW_UNRECORDED", "SLOW_SPAN",
                                   "SLOW_ANCHOR", "FAST_DIRTY"])}
TIMER = {n: i for i, n in enumerate(["INGEST", "EXEC_ASSIGN", "BUILD_PREP", "APPLY_WALK", "WALK_SLOW",
                                     "MAKE_QUERIES", "ANCHOR_WALK", "PREDICT", "SELECT", "MIG_PLAN", "COPY",
                                     "RESIDENCY", "CHAIN", "JUMP", "WALK", "EXACT", "WALK_INDEX", "WALK_RES", "SELECT_FAST", "COMMIT"])}
KERNEL_OF_TIMER = {"INGEST": "k_ingest", "EXEC_ASSIGN": "k_exec_assign", "BUILD_PREP": "k_build_prep",
                   "APPLY_WALK": "k_build_exec", "WALK": "k_walk", "WALK_SLOW": "k_walk_slow", "MAKE_QUERIES": "k_make_queries",
                   "ANCHOR_WALK": "k_anchor_walk", "PREDICT": "k_copy_fast", "SELECT": "k_select", "SELECT_FAST": "k_window_fast",
                   "MIG_PLAN": "k_mig_plan", "COPY": "k_copy_blocks", "RESIDENCY": "k_load_res",
                   "CHAIN": "k_chain", "JUMP": "k_jump0", "EXACT": "k_predict", "WALK_INDEX": "k_walk_index",
                   "WALK_RES": "k_walk_res", "COMMIT": "k_walk_commit"}
# timers of kernels launched on the engine's side streams (overlapping others)
SIDE_TIMERS = {"JUMP": "side stream, overlaps k_apply / k_walk (k_jump0 + k_jumpk levels)",
               "SELECT_FAST": "second side stream, beside the exact path (k_window_fast: pairs + selection of the fast windows)",
               "WALK_RES": "ingest-side fork in dum_step (beside k_ingest .. k_anchor_walk)",
               "WALK_INDEX": "third side stream (high priority) after the build (replayed step graphs: at the start of the next step, beside its ingest)"}
_ERR = {0: "DUM_OK", -1: "DUM_EINVAL", -2: "DUM_ECAPACITY", -3: "DUM_ENOMEM", -4: "DUM_ECUDA", -5: "DUM_ESTATE"}


class EngineError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__("%s: %s" % (_ERR.get(code, code), msg))
        self.code = code


class DumConfig(ctypes.Structure):
    _fields_ = [
        ("num_rows", ctypes.c_uint32), ("assoc", ctypes.c_uint32), ("num_succs", ctypes.c_uint32),
        ("degree_n", ctypes.c_uint32), ("max_blocks", ctypes.c_uint32), ("max_exec_ids", ctypes.c_uint32),
        ("hbm_frames", ctypes.c_uint32), ("row_index", ctypes.c_uint32), ("max_batch_launches", ctypes.c_uint32),
        ("max_batch_faults", ctypes.c_uint64), ("corr_capacity", ctypes.c_uint32), ("device", ctypes.c_int),
        ("host_arena", ctypes.c_void_p), ("host_arena_bytes", ctypes.c_uint64),
        ("frame_pool", ctypes.c_void_p), ("frame_pool_bytes", ctypes.c_uint64),
        ("flags", ctypes.c_uint32),
    ]


class DumStats(ctypes.Structure):
    _fields_ = [
        ("num_exec", ctypes.c_uint32), ("corr_records", ctypes.c_uint32), ("free_frames", ctypes.c_uint32),
        ("staged_launches", ctypes.c_uint32), ("launches", ctypes.c_uint64), ("staged_faults", ctypes.c_uint64),
        ("slow_walks", ctypes.c_uint32), ("n_resident", ctypes.c_uint32),
        ("guard_line", ctypes.c_uint32), ("guard_val", ctypes.c_uint32),
    ]


_LIB = None


def library_path() -> str:
    return _LIBPATH


def load_library() -> ctypes.CDLL:
    global _LIB
    if _LIB is not None:
        return _LIB
    if not os.path.exists(_LIBPATH):
        raise ImportError("libdeepum_b200.so is not built (run: python -m paper_conf_asplos_jungkl23_b200.build); "
                          "there is no CPU fallback")
    L = ctypes.CDLL(_LIBPATH)
    P, U32, U64, I = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    sig = {
        "dum_config_default": (None, [P]),
        "dum_create": (I, [P, P]),
        "dum_destroy": (I, [P]),
        "dum_reset": (I, [P, P]),
        "dum_record_faults": (I, [P, P, P, U32, P, U64, P, U32, P]),
        "dum_build_tables": (I, [P, P]),
        "dum_make_queries": (I, [P, P, U32, U32, U32, P, P]),
        "dum_predict_prefetch": (I, [P, P, U32, P, U64, P, P, P, P, P]),
        "dum_select_evictions": (I, [P, P, P, U32, P, P, P, U64, P, P, P]),
        "dum_predict_select": (I, [P, P, U32, P, U64, P, P, P, P, P, P, U64, P, P, P]),
        "dum_mark_inactive": (I, [P, P, U32, I, P]),
        "dum_load_residency": (I, [P, P, U32, P]),
        "dum_migrate_blocks": (I, [P, I, P, P, U32, U32, P]),
        "dum_block_checksums": (I, [P, I, P, U32, P, P]),
        "dum_dump_state": (I, [P, U32, P, U64, P]),
        "dum_sync": (I, [P, P, P]),
        "dum_get_stats": (I, [P, P]),
        "dum_last_error": (ctypes.c_char_p, [P]),
        "dum_kernel_launches": (U64, [P]),
        "dum_read_counters": (I, [P, P, I]),
        "dum_set_counting": (I, [P, I]),
        "dum_set_copy_sms": (I, [P, ctypes.c_uint32]),
        "dum_set_timing": (I, [P, I]),
        "dum_host_ptr_kind": (I, [P]),
        "dum_read_timing": (I, [P, P, P, I]),
        "dum_read_timeline": (I, [P, I, P, P, P]),
        "dum_simulate": (I, [P, P, U32, P, P, U32, U32, U32, P, P]),
        "dum_step": (I, [P, P, P, U32, P, U64, U32, U32, P, U64, P, P, P, P, P, P, U64, P, P, P]),
        "dum_set_step_graphs": (I, [P, I]),
    }
    for name, (res, args) in sig.items():
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _LIB = L
    return L


def _dev(t: Optional[torch.Tensor], itemsize: int = 0):
    if t is None:
        return None
    if not t.is_cuda or not t.is_contiguous():
        raise ValueError("expected a contiguous CUDA tensor")
    if itemsize and t.element_size() != itemsize:
        raise ValueError("expected %d-byte elements" % itemsize)
    return ctypes.c_void_p(t.data_ptr())


def as_u32_tensor(a, device) -> torch.Tensor:
    if isinstance(a, torch.Tensor):
        return a.to(device=device, dtype=torch.int32) if a.dtype != torch.int32 else a.to(device)
    return torch.from_numpy(np.ascontiguousarray(np.asarray(a, dtype=np.uint32)).view(np.int32)).to(device)


def as_u64_tensor(a, device) -> torch.Tensor:
    if isinstance(a, torch.Tensor):
        return a.to(device)
    return torch.from_numpy(np.ascontiguousarray(np.asarray(a, dtype=np.uint64)).view(np.int64)).to(device)


def u32(t: torch.Tensor) -> np.ndarray:
    return t.detach().cpu().numpy().view(np.uint32)


def u64(t: torch.Tensor) -> np.ndarray:
    return t.detach().cpu().numpy().view(np.uint64)


class Engine:
    """One engine per GPU / replica (engines share nothing)."""

    def __init__(self, num_rows=2048, assoc=2, num_succs=4, degree_n=32, max_blocks=1 << 16, max_exec_ids=8192,
                 hbm_frames=1024, row_index=0, max_batch_launches=0, max_batch_faults=0, corr_capacity=0,
                 device: int = 0, host_arena: Optional[torch.Tensor] = None,
                 frame_pool: Optional[torch.Tensor] = None, flags: int = 0):
        self.lib = load_library()
        self.device = torch.device("cuda", device)
        c = DumConfig()
        self.lib.dum_config_default(ctypes.byref(c))
        c.num_rows, c.assoc, c.num_succs, c.degree_n = num_rows, assoc, num_succs, degree_n
        c.max_blocks, c.max_exec_ids, c.hbm_frames, c.row_index = max_blocks, max_exec_ids, hbm_frames, row_index
        c.max_batch_launches, c.max_batch_faults, c.corr_capacity, c.device = (
            max_batch_launches, max_batch_faults, corr_capacity, device)
        c.flags = flags
        if host_arena is not None:
            c.host_arena, c.host_arena_bytes = host_arena.data_ptr(), host_arena.numel() * host_arena.element_size()
        if frame_pool is not None:
            c.frame_pool, c.frame_pool_bytes = frame_pool.data_ptr(), frame_pool.numel() * frame_pool.element_size()
        self._keep = (host_arena, frame_pool)
        self.R, self.A, self.S, self.N, self.W, self.C = num_rows, assoc, num_succs, degree_n, max_blocks, hbm_frames
        h = ctypes.c_void_p()
        rc = self.lib.dum_create(ctypes.byref(c), ctypes.byref(h))
        if rc != 0:
            raise EngineError(rc, "dum_create failed")
        self._h = h

    # ------------------------------------------------------------------
    def _stream(self):
        return ctypes.c_void_p(torch.cuda.current_stream(self.device).cuda_stream)

    def _ck(self, rc: int, what: str):
        if rc != 0:
            raise EngineError(rc, "%s: %s" % (what, self.lib.dum_last_error(self._h).decode()))

    def close(self):
        if getattr(self, "_h", None):
            self.lib.dum_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # ------------------------------------------------------------------
    def reset(self):
        self._ck(self.lib.dum_reset(self._h, self._stream()), "dum_reset")

    def record_faults(self, hashes, offs, faults, out_exec: Optional[torch.Tensor] = None,
                      ready: bool = False) -> Optional[torch.Tensor]:
        """Device tensors -> device path; numpy arrays -> DUM_HOST_PTRS.
        ready=True (device tensors): the inputs do not depend on work queued on
        the current stream (DUM_INPUTS_READY), so the ingest may overlap it."""
        if isinstance(hashes, np.ndarray):
            h = np.ascontiguousarray(hashes, dtype=np.uint64)
            o = np.ascontiguousarray(offs, dtype=np.uint64)
            f = np.ascontiguousarray(faults, dtype=np.uint32)
            n = len(h)
            self._ck(self.lib.dum_record_faults(self._h, h.ctypes.data, o.ctypes.data, n,
                                                f.ctypes.data if len(f) else None, len(f), _dev(out_exec, 4),
                                                DUM_HOST_PTRS, self._stream()), "dum_record_faults")
            return out_exec
        n = hashes.numel()
        self._ck(self.lib.dum_record_faults(self._h, _dev(hashes, 8), _dev(offs, 8), n, _dev(faults, 4),
                                            faults.numel(), _dev(out_exec, 4), DUM_INPUTS_READY if ready else 0,
                                            self._stream()),
                 "dum_record_faults")
        return out_exec

    def build_tables(self):
        self._ck(self.lib.dum_build_tables(self._h, self._stream()), "dum_build_tables")

    def make_queries(self, exec_seq: torch.Tensor, first: int, degree: Optional[int] = None,
                     out: Optional[torch.Tensor] = None) -> torch.Tensor:
        n_seq = exec_seq.numel()
        if out is None:
            out = torch.empty((max(n_seq - first, 0), 6), dtype=torch.int32, device=self.device)
        self._ck(self.lib.dum_make_queries(self._h, _dev(exec_seq, 4), n_seq, first,
                                           self.N if degree is None else degree, _dev(out, 4), self._stream()),
                 "dum_make_queries")
        return out

    def predict_prefetch(self, queries: torch.Tensor, cap: int, pairs: Optional[torch.Tensor] = None,
                         rng: Optional[torch.Tensor] = None, kern_off: Optional[torch.Tensor] = None,
                         chain: Optional[torch.Tensor] = None, needed: Optional[torch.Tensor] = None,
                         want_kern_off: bool = True, want_chain: bool = True):
        nq = queries.shape[0]
        if pairs is None:
            pairs = torch.empty((max(cap, 1), 2), dtype=torch.int32, device=self.device)
        if rng is None:
            rng = torch.empty((nq, 2), dtype=torch.int64, device=self.device)
        if kern_off is None and want_kern_off:
            kern_off = torch.empty((nq, self.N + 2), dtype=torch.int32, device=self.device)
        if chain is None and want_chain:
            chain = torch.empty((nq, self.N + 1), dtype=torch.int32, device=self.device)
        if needed is None:
            needed = torch.zeros(1, dtype=torch.int64, device=self.device)
        self._ck(self.lib.dum_predict_prefetch(self._h, _dev(queries, 4), nq, _dev(pairs, 4), cap, _dev(rng, 8),
                                               _dev(kern_off, 4), _dev(chain, 4), _dev(needed, 8), self._stream()),
                 "dum_predict_prefetch")
        return pairs, rng, kern_off, chain, needed

    def select_evictions(self, rng: torch.Tensor, pairs: torch.Tensor, queries: Optional[torch.Tensor], cap: int,
                         wb: Optional[torch.Tensor] = None, inv: Optional[torch.Tensor] = None,
                         out_rng: Optional[torch.Tensor] = None, needed: Optional[torch.Tensor] = None):
        nq = rng.shape[0]
        if wb is None:
            wb = torch.empty(max(cap, 1), dtype=torch.int32, device=self.device)
        if inv is None:
            inv = torch.empty(max(cap, 1), dtype=torch.int32, device=self.device)
        if out_rng is None:
            out_rng = torch.empty((nq, 4), dtype=torch.int64, device=self.device)
        if needed is None:
            needed = torch.zeros(1, dtype=torch.int64, device=self.device)
        self._ck(self.lib.dum_select_evictions(self._h, _dev(rng, 8), _dev(pairs, 4), nq, _dev(queries, 4),
                                               _dev(wb, 4), _dev(inv, 4), cap, _dev(out_rng, 8), _dev(needed, 8),
                                               self._stream()), "dum_select_evictions")
        return wb, inv, out_rng, needed

    def predict_select(self, queries: torch.Tensor, cap: int, sel_cap: Optional[int] = None, pairs=None, rng=None,
                       kern_off=None, chain=None, needed=None, wb=None, inv=None, sel_rng=None, sel_needed=None,
                       want_kern_off: bool = True, want_chain: bool = True):
        """Fused a7 + a8 (dum_predict_select)."""
        nq = queries.shape[0]
        sel_cap = cap if sel_cap is None else sel_cap
        d = self.device
        if pairs is None:
            pairs = torch.empty((max(cap, 1), 2), dtype=torch.int32, device=d)
        if rng is None:
            rng = torch.empty((nq, 2), dtype=torch.int64, device=d)
        if kern_off is None and want_kern_off:
            kern_off = torch.empty((nq, self.N + 2), dtype=torch.int32, device=d)
        if chain is None and want_chain:
            chain = torch.empty((nq, self.N + 1), dtype=torch.int32, device=d)
        if needed is None:
            needed = torch.zeros(1, dtype=torch.int64, device=d)
        if wb is None:
            wb = torch.empty(max(sel_cap, 1), dtype=torch.int32, device=d)
        if inv is None:
            inv = torch.empty(max(sel_cap, 1), dtype=torch.int32, device=d)
        if sel_rng is None:
            sel_rng = torch.empty((nq, 4), dtype=torch.int64, device=d)
        if sel_needed is None:
            sel_needed = torch.zeros(1, dtype=torch.int64, device=d)
        self._ck(self.lib.dum_predict_select(self._h, _dev(queries, 4), nq, _dev(pairs, 4), cap, _dev(rng, 8),
                                             _dev(kern_off, 4), _dev(chain, 4), _dev(needed, 8), _dev(wb, 4),
                                             _dev(inv, 4), sel_cap, _dev(sel_rng, 8), _dev(sel_needed, 8),
                                             self._stream()), "dum_predict_select")
        return pairs, rng, kern_off, chain, needed, wb, inv, sel_rng, sel_needed

    def simulate(self, launch_hash: torch.Tensor, acc_off: np.ndarray, acc_blk: torch.Tensor, degree: int,
                 flags: int, stats: Optional[torch.Tensor] = None) -> torch.Tensor:
        """dum_simulate: the closed loop over len(launch_hash) launches; launch k
        accesses acc_blk[acc_off[k % K] : acc_off[k % K + 1]] (K = len(acc_off) - 1).
        Returns the per-launch statistics, a [n_launch, 6] int32 device tensor
        (columns SIM_FIELDS)."""
        n = launch_hash.numel()
        off = np.ascontiguousarray(acc_off, dtype=np.uint64)
        if stats is None:
            stats = torch.zeros((n, len(SIM_FIELDS)), dtype=torch.int32, device=self.device)
        self._ck(self.lib.dum_simulate(self._h, _dev(launch_hash, 8), n, off.ctypes.data, _dev(acc_blk, 4),
                                       len(off) - 1, degree, flags, _dev(stats, 4), self._stream()), "dum_simulate")
        return stats

    def step(self, hashes, offs, faults, cap: int, sel_cap: int, out: dict, degree: Optional[int] = None,
             ready: bool = False):
        """dum_step: record -> one transition query per launch -> predict+select
        -> build, in one C call.  numpy inputs -> DUM_HOST_PTRS (pinned arrays
        upload asynchronously); device tensors otherwise.  `out` holds the
        output tensors (pairs, rng, kern_off, chain, needed, wb, inv, sel_rng,
        sel_needed), allocated on first use for the batch size."""
        n = len(hashes) if isinstance(hashes, np.ndarray) else hashes.numel()
        d = self.device
        if out.get("n") != n or out.get("cap") != cap or out.get("sel_cap") != sel_cap:
            out.update(n=n, cap=cap, sel_cap=sel_cap,
                       pairs=torch.empty((max(cap, 1), 2), dtype=torch.int32, device=d),
                       rng=torch.empty((n, 2), dtype=torch.int64, device=d),
                       kern_off=torch.empty((n, self.N + 2), dtype=torch.int32, device=d),
                       chain=torch.empty((n, self.N + 1), dtype=torch.int32, device=d),
                       needed=torch.zeros(1, dtype=torch.int64, device=d),
                       wb=torch.empty(max(sel_cap, 1), dtype=torch.int32, device=d),
                       inv=torch.empty(max(sel_cap, 1), dtype=torch.int32, device=d),
                       sel_rng=torch.empty((n, 4), dtype=torch.int64, device=d),
                       sel_needed=torch.zeros(1, dtype=torch.int64, device=d))
        if isinstance(hashes, np.ndarray):
            h, o, f = hashes, offs, faults
            args = (h.ctypes.data, o.ctypes.data, n, f.ctypes.data if len(f) else None, len(f), DUM_HOST_PTRS)
        else:
            args = (_dev(hashes, 8), _dev(offs, 8), n, _dev(faults, 4), faults.numel(),
                    DUM_INPUTS_READY if ready else 0)
        self._ck(self.lib.dum_step(self._h, *args, self.N if degree is None else degree, _dev(out["pairs"], 4), cap,
                                   _dev(out["rng"], 8), _dev(out["kern_off"], 4), _dev(out["chain"], 4),
                                   _dev(out["needed"], 8), _dev(out["wb"], 4), _dev(out["inv"], 4), sel_cap,
                                   _dev(out["sel_rng"], 8), _dev(out["sel_needed"], 8), self._stream()), "dum_step")
        return out

    def set_step_graphs(self, on: bool):
        self._ck(self.lib.dum_set_step_graphs(self._h, 1 if on else 0), "dum_set_step_graphs")

    def mark_inactive(self, blocks: torch.Tensor, inactive: bool = True):
        self._ck(self.lib.dum_mark_inactive(self._h, _dev(blocks, 4), blocks.numel(), 1 if inactive else 0,
                                            self._stream()), "dum_mark_inactive")

    def load_residency(self, lrm: torch.Tensor):
        self._ck(self.lib.dum_load_residency(self._h, _dev(lrm, 4), lrm.numel(), self._stream()),
                 "dum_load_residency")

    def migrate_blocks(self, direction: int, blocks: Optional[torch.Tensor] = None,
                       dst_frames: Optional[torch.Tensor] = None, method: int = 0):
        n = 0 if blocks is None else blocks.numel()
        self._ck(self.lib.dum_migrate_blocks(self._h, direction, _dev(blocks, 4), _dev(dst_frames, 4), n, method,
                                             self._stream()), "dum_migrate_blocks")

    def block_checksums(self, where: int, ids: torch.Tensor) -> torch.Tensor:
        out = torch.empty(ids.numel(), dtype=torch.int64, device=self.device)
        self._ck(self.lib.dum_block_checksums(self._h, where, _dev(ids, 4), ids.numel(), _dev(out, 8),
                                              self._stream()), "dum_block_checksums")
        return out

    def sync(self) -> int:
        need = ctypes.c_uint64(0)
        rc = self.lib.dum_sync(self._h, self._stream(), ctypes.byref(need))
        if rc != 0:
            e = EngineError(rc, "%s (needed=%d)" % (self.lib.dum_last_error(self._h).decode(), need.value))
            e.needed = need.value
            raise e
        return need.value

    def dump_state(self, what: int) -> bytes:
        need = ctypes.c_uint64(0)
        self.lib.dum_dump_state(self._h, what, None, 0, ctypes.byref(need))
        buf = (ctypes.c_uint8 * max(need.value, 1))()
        self._ck(self.lib.dum_dump_state(self._h, what, buf, len(buf), ctypes.byref(need)), "dum_dump_state")
        return bytes(buf)[: need.value]

    def stats(self) -> DumStats:
        s = DumStats()
        self._ck(self.lib.dum_get_stats(self._h, ctypes.byref(s)), "dum_get_stats")
        return s

    def read_counters(self, reset: bool = False) -> np.ndarray:
        out = np.zeros(NCOUNTERS, dtype=np.uint64)
        self._ck(self.lib.dum_read_counters(self._h, out.ctypes.data, 1 if reset else 0), "dum_read_counters")
        return out

    def set_counting(self, on: bool):
        self._ck(self.lib.dum_set_counting(self._h, 1 if on else 0), "dum_set_counting")

    def counters(self, reset: bool = False) -> dict:
        c = self.read_counters(reset)
        return {k: int(c[v]) for k, v in CTR.items()}

    def set_copy_sms(self, n_sms: int):
        """Cap the copy kernels of this engine at n_sms SMs' worth of CTAs (0 = all)."""
        self._ck(self.lib.dum_set_copy_sms(self._h, int(n_sms)), "dum_set_copy_sms")

    def set_timing(self, on: bool):
        self._ck(self.lib.dum_set_timing(self._h, 1 if on else 0), "dum_set_timing")

    def read_timing(self, reset: bool = False):
        ms = np.zeros(NTIMERS, dtype=np.float64)
        cnt = np.zeros(NTIMERS, dtype=np.uint64)
        self._ck(self.lib.dum_read_timing(self._h, ms.ctypes.data, cnt.ctypes.data, 1 if reset else 0),
                 "dum_read_timing")
        return ms, cnt

    def read_timeline(self, cap: int = 4096):
        """(timer ids, start ms, end ms) of the timed regions since the last read, issue order."""
        ids = np.zeros(cap, dtype=np.int32)
        t0 = np.zeros(cap, dtype=np.float32)
        t1 = np.zeros(cap, dtype=np.float32)
        n = int(self.lib.dum_read_timeline(self._h, cap, ids.ctypes.data, t0.ctypes.data, t1.ctypes.data))
        if n < 0:
            self._ck(n, "dum_read_timeline")
        return ids[:n], t0[:n], t1[:n]

    @property
    def kernel_launches(self) -> int:
        return int(self.lib.dum_kernel_launches(self._h))
