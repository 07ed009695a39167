"""CPU oracle of DeepUM's correlation-prefetch and migration engine.

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / ``--impl reference`` leg may import this package.  The product
path (paper_conf_asplos_jungkl23_b200) never imports it, and the two share no
code: the oracle is oracle/deepum_oracle.cpp (plain sequential C++17, written
from PAPER.md) plus this ctypes wrapper.

Parity status per function (details in DESIGN.md "Oracle pins"):
  record_faults   pinned: brute-force first-occurrence dedupe, exec IDs dense
                  and first-seen (tests/test_oracle_pins.py)
  build_tables    pinned: Fig. 7 exactly, Fig. 6
                  (L178-L185) entries 0 and 2 exactly / entry 1 superset,
                  Fig. 5 (L168-L170) reconstructed, R=1 textbook LRU, brute-force
                  MRU successor lists, Config-T closed form
  walk / predict  pinned: L222 worked example, periodic-trace closed form,
                  Config-T closed form
  select          pinned: brute-force sort/filter/take + invariant I7
  migrate         pinned: bookkeeping invariants (bijection, lowest-free-frame)
  Parity unpinned (no value in the paper fixes them; the readings are listed in
  DESIGN.md): D2 alternative, D5 storage, D7 index fn, D8 recency under
  conflicts, D13 successor choice, D18 amount, D21 frame choice.
"""
from __future__ import annotations

import ctypes
import os
import struct
import subprocess
from typing import Dict, List, Optional, Tuple

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
_SO = os.path.join(HERE, "liboracle.so")
_SRC = os.path.join(HERE, "deepum_oracle.cpp")
NONE = 0xFFFFFFFF

EXEC, CORR, BLK, WALK, RES, HIST = 1, 2, 4, 8, 16, 32
H2D, D2H, INVALIDATE, D2D = 0, 1, 2, 3


def build() -> str:
    """Compile the oracle (plain g++, no CUDA)."""
    tmp = _SO + ".tmp%d" % os.getpid()
    subprocess.check_call(["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-pthread", "-o", tmp, _SRC])
    os.replace(tmp, _SO)
    return _SO


_LIB = None


def _lib() -> ctypes.CDLL:
    global _LIB
    if _LIB is not None:
        return _LIB
    if not os.path.exists(_SO) or os.path.getmtime(_SO) < os.path.getmtime(_SRC):
        build()
    L = ctypes.CDLL(_SO)
    P, U32, U64, I = ctypes.c_void_p, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int
    L.orc_create.restype = P
    L.orc_create.argtypes = [U32] * 7
    L.orc_destroy.argtypes = [P]
    L.orc_record_faults.argtypes = [P, P, P, U32, P, P]
    L.orc_build_tables.argtypes = [P]
    L.orc_num_exec.argtypes = [P]
    L.orc_num_exec.restype = U32
    L.orc_predict.argtypes = [P, P, U32, P, P, U64, P, P, P]
    L.orc_select.argtypes = [P, P, P, U32, P, P, P, P, P, U64, P]
    L.orc_mark_inactive.argtypes = [P, P, U32, I]
    L.orc_load_residency.argtypes = [P, P, U32]
    L.orc_migrate.argtypes = [P, I, P, P, U32]
    L.orc_free_frames.argtypes = [P]
    L.orc_free_frames.restype = U32
    L.orc_dump.argtypes = [P, U32, P, U64, P]
    L.orc_set_threads.argtypes = [P, U32]
    _LIB = L
    return L


def _p(a):
    return None if a is None else ctypes.c_void_p(a.ctypes.data)


def _u32(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.uint32))


def _u64(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.uint64))


class OracleError(RuntimeError):
    pass


class Oracle:
    """Sequential CPU reference.  Geometry (R rows, A ways, S successors) as in
    PAPER.md Table 6 (L429-L443); default Config9 = 2048/2/4 (L303)."""

    def __init__(self, R: int = 2048, A: int = 2, S: int = 4, N: int = 32, W: int = 256, C: int = 128,
                 row_index: int = 0, threads: int = 1):
        self.R, self.A, self.S, self.N, self.W, self.C = R, A, S, N, W, C
        self._h = _lib().orc_create(R, A, S, N, W, C, row_index)
        if not self._h:
            raise OracleError("bad geometry")
        self._cap_hint = 1 << 16
        self.set_threads(threads)

    def set_threads(self, n: int) -> None:
        """predict / select split their (independent) queries over n threads;
        the outputs are identical for every n (concatenated in query order)."""
        self.threads = max(1, int(n))
        _lib().orc_set_threads(self._h, self.threads)

    def __del__(self):
        h = getattr(self, "_h", None)
        if h:
            _lib().orc_destroy(h)
            self._h = None

    # a1 + a2
    def record_faults(self, hashes, offs, faults) -> np.ndarray:
        h, o, f = _u64(hashes), _u64(offs), _u32(faults)
        n = len(h)
        out = np.zeros(max(n, 1), dtype=np.uint32)
        _lib().orc_record_faults(self._h, _p(h), _p(o), n, _p(f) if len(f) else None, _p(out))
        return out[:n]

    # a3 - a5
    def build_tables(self) -> None:
        _lib().orc_build_tables(self._h)

    @property
    def num_exec(self) -> int:
        return int(_lib().orc_num_exec(self._h))

    # a6 + a7
    def predict(self, queries) -> Tuple[np.ndarray, np.ndarray, np.ndarray, np.ndarray]:
        """queries: [n,6] u32 (exec, h1, h2, h3, anchor, n).  Returns (off[n+1],
        pairs[P,2], kern_off[n,N+2], chain[n,N+1])."""
        q = _u32(queries).reshape(-1, 6)
        nq = q.shape[0]
        off = np.zeros(nq + 1, dtype=np.uint64)
        ko = np.zeros((max(nq, 1), self.N + 2), dtype=np.uint32)
        ch = np.zeros((max(nq, 1), self.N + 1), dtype=np.uint32)
        need = np.zeros(1, dtype=np.uint64)
        cap = self._cap_hint
        while True:
            pairs = np.empty((cap, 2), dtype=np.uint32)
            rc = _lib().orc_predict(self._h, _p(q), nq, _p(off), _p(pairs), cap, _p(ko), _p(ch), _p(need))
            if rc == 0:
                return off, pairs[: int(need[0])], ko[:nq], ch[:nq]
            cap = int(need[0]) + 1
            self._cap_hint = max(self._cap_hint, cap)

    # a8
    def select(self, qoff, pairs, anchors=None):
        qoff = _u64(qoff)
        pr = _u32(pairs).reshape(-1)
        nq = len(qoff) - 1
        an = None if anchors is None else _u32(anchors)
        wb_off = np.zeros(nq + 1, dtype=np.uint64)
        inv_off = np.zeros(nq + 1, dtype=np.uint64)
        need = np.zeros(1, dtype=np.uint64)
        cap = self._cap_hint
        while True:
            wb = np.empty(cap, dtype=np.uint32)
            inv = np.empty(cap, dtype=np.uint32)
            rc = _lib().orc_select(self._h, _p(qoff), _p(pr) if len(pr) else _p(np.zeros(2, np.uint32)), nq,
                                   _p(an), _p(wb), _p(wb_off), _p(inv), _p(inv_off), cap, _p(need))
            if rc == 0:
                return wb_off, wb[: int(wb_off[-1])], inv_off, inv[: int(inv_off[-1])]
            cap = int(need[0]) + 1
            self._cap_hint = max(self._cap_hint, cap)

    def mark_inactive(self, blocks, inactive: bool = True) -> None:
        b = _u32(blocks)
        rc = _lib().orc_mark_inactive(self._h, _p(b), len(b), 1 if inactive else 0)
        if rc:
            raise OracleError("mark_inactive rc=%d" % rc)

    def load_residency(self, lrm_blocks) -> None:
        b = _u32(lrm_blocks)
        rc = _lib().orc_load_residency(self._h, _p(b), len(b))
        if rc:
            raise OracleError("load_residency rc=%d" % rc)

    def migrate(self, direction: int, blocks=None, dst_frames=None) -> int:
        b = None if blocks is None else _u32(blocks)
        d = None if dst_frames is None else _u32(dst_frames)
        n = 0 if b is None else len(b)
        return _lib().orc_migrate(self._h, direction, _p(b), _p(d), n)

    @property
    def free_frames(self) -> int:
        return int(_lib().orc_free_frames(self._h))

    def dump(self, what: int) -> bytes:
        need = np.zeros(1, dtype=np.uint64)
        _lib().orc_dump(self._h, what, None, 0, _p(need))
        buf = np.zeros(max(int(need[0]), 1), dtype=np.uint8)
        rc = _lib().orc_dump(self._h, what, _p(buf), len(buf), _p(need))
        assert rc == 0
        return buf[: int(need[0])].tobytes()


# ----------------------------------------------------------------------------
# canonical-dump parsing (format: SURVEY.md Sec. 8c / DESIGN.md "Canonical dump")
# ----------------------------------------------------------------------------
def parse_dump(buf: bytes, what: int, E: int, R: int, A: int, S: int) -> Dict[str, object]:
    """Decode a canonical dump into Python structures (used by tests for both
    the oracle's and the engine's dumps)."""
    a = np.frombuffer(buf, dtype=np.uint8)
    pos = 0
    out: Dict[str, object] = {}

    def u32() -> int:
        nonlocal pos
        v = int.from_bytes(buf[pos:pos + 4], "little")
        pos += 4
        return v

    if what & EXEC:
        n = u32()
        out["exec_hash"] = np.frombuffer(buf, dtype=np.uint64, count=n, offset=pos).copy()
        pos += 8 * n
        E = n
    if what & CORR:
        corr = []
        for _ in range(E):
            n = u32()
            recs = np.frombuffer(buf, dtype=np.uint32, count=4 * n, offset=pos).reshape(n, 4)
            pos += 16 * n
            corr.append([tuple(int(x) for x in r) for r in recs])
        out["corr"] = corr
    if what & BLK:
        per = R * A * (1 + S) + 2
        blk = np.frombuffer(buf, dtype=np.uint32, count=per * E, offset=pos).reshape(E, per)
        pos += 4 * per * E
        out["blk"] = blk[:, :-2].reshape(E, R, A, 1 + S)
        out["start"] = blk[:, -2].copy()
        out["end"] = blk[:, -1].copy()
    if what & WALK:
        walks = []
        for _ in range(E):
            n = u32()
            walks.append(np.frombuffer(buf, dtype=np.uint32, count=n, offset=pos).copy())
            pos += 4 * n
        out["walk"] = walks
    if what & RES:
        C = u32()
        out["block_of_frame"] = np.frombuffer(buf, dtype=np.uint32, count=C, offset=pos).copy()
        pos += 4 * C
        n = u32()
        out["lrm"] = np.frombuffer(buf, dtype=np.uint32, count=n, offset=pos).copy()
        pos += 4 * n
    if what & HIST:
        out["hist"] = tuple(u32() for _ in range(4))
        out["launches"] = int.from_bytes(buf[pos:pos + 8], "little")
        pos += 8
    assert pos == len(a), (pos, len(a))
    return out


def table_rows(blk_e: np.ndarray) -> Dict[int, List[int]]:
    """{tag: [successors MRU first]} for one exec ID's BLK section."""
    rows: Dict[int, List[int]] = {}
    R, A, _ = blk_e.shape
    for r in range(R):
        for w in range(A):
            tag = int(blk_e[r, w, 0])
            if tag != NONE:
                rows[tag] = [int(x) for x in blk_e[r, w, 1:] if x != NONE]
    return rows
