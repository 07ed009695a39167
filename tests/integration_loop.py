"""T-scale closed-loop driver (SURVEY.md Sec. 8a "T-scale integration loop").

Drives any engine object that offers the five calls (record_faults,
build_tables, predict, select, migrate) plus a residency view, per launch of
the generator's ACCESS stream:
  1. faults = the launch's accesses with no frame (closed loop, not the
     naive-UM trace)
  2. record_faults([k])
  3. demand H2D of the faults; if frames run out, LRM eviction excluding the
     current launch's blocks (D22; PAPER.md L158 fault queue first, L238)
  4. build_tables
  5. transition query for launch k+1 (true next exec ID and history)
                                                        PAPER.md L220-L224
  6. select_evictions for that window
  7. D2H / invalidate the victims
  8. H2D of the window's non-resident prefix that fits
The driver holds only bookkeeping of the engine's outputs (which hash got which
exec ID) and host-side list manipulation; every decision comes from the engine.
"""
from __future__ import annotations

from typing import Dict, List

import numpy as np

NONE = 0xFFFFFFFF
H2D, D2H, INVALIDATE = 0, 1, 2


class LoopEngine:
    """Adapter interface; see OracleLoop in this file and the GPU adapter in
    tests/test_gpu_parity.py."""

    def record(self, h: int, faults: List[int]) -> int: ...
    def build(self) -> None: ...
    def predict1(self, q) -> List[int]: ...           # window blocks in order
    def select1(self, blocks: List[int], anchor: int): ...
    def migrate(self, d: int, blocks: List[int]) -> None: ...
    def resident(self) -> List[int]: ...               # LRM order
    def free(self) -> int: ...
    def snapshot(self) -> bytes: ...


def run_loop(eng: LoopEngine, tr, N: int, inactive: set = frozenset(), check=None, preevict: bool = True,
             invalidate: bool = True, n_launch: int = None, per_launch: list = None) -> Dict[str, object]:
    """N < 0: no queries (naive UM, demand path only).  preevict=False
    (prefetch only): the whole non-resident window is prefetched, the driver
    evicting the least recently migrated blocks beyond the free frames.  invalidate=False: inactive
    victims are written back too.  Faults are the first occurrence of each
    non-resident access of the launch (D2; the T trace has no repeats).
    per_launch (a list) receives (faults, demand_wb, demand_inv, pre_wb,
    pre_inv, prefetched) per launch."""
    ids: Dict[int, int] = {}
    execs: List[int] = []
    faults_per_iter = [0] * tr.n_iter
    h2d = d2h = inv = 0
    K = tr.K
    total = tr.n_iter * K if n_launch is None else n_launch
    for it in range(tr.n_iter):
        for j in range(K):
            k = it * K + j
            if k >= total:
                break
            acc = [int(b) for b in tr.access_blk[int(tr.access_off[j]):int(tr.access_off[j + 1])]]
            res = eng.resident()
            rset = set(res)
            faults = [b for b in dict.fromkeys(acc) if b not in rset]
            st = [len(faults), 0, 0, 0, 0, 0]
            faults_per_iter[it] += len(faults)
            h = int(tr.launch_hash[k])
            e = eng.record(h, faults)
            ids.setdefault(h, e)
            execs.append(e)
            # demand path (D22)
            nf = eng.free()
            if len(faults) > nf:
                need = len(faults) - nf
                aset = set(acc)
                victims = [b for b in res if b not in aset][:need]
                wb = [b for b in victims if b not in inactive]
                iv = [b for b in victims if b in inactive]
                if not invalidate:
                    wb, iv = wb + iv, []  # (the engine writes the inactive list back after the active one)
                st[1], st[2] = len(wb), len(iv)
                if wb:
                    eng.migrate(D2H, wb); d2h += len(wb)
                if iv:
                    eng.migrate(INVALIDATE, iv); inv += len(iv)
            if faults:
                eng.migrate(H2D, faults); h2d += len(faults)
            eng.build()
            # transition query for the next launch
            k1 = k + 1
            if k1 < total and N >= 0:
                h1 = int(tr.launch_hash[k1])
                if h1 in ids:
                    hist = ([NONE, NONE, NONE] + execs)[-3:]
                    q = [ids[h1], hist[0], hist[1], hist[2], NONE, N]
                    window = eng.predict1(q)
                    if preevict:
                        wb, iv = eng.select1(window, NONE)
                        if not invalidate:
                            wb, iv = wb + iv, []
                        st[3], st[4] = len(wb), len(iv)
                        if wb:
                            eng.migrate(D2H, wb); d2h += len(wb)
                        if iv:
                            eng.migrate(INVALIDATE, iv); inv += len(iv)
                    res = eng.resident()
                    rset = set(res)
                    if preevict:
                        todo = [b for b in window if b not in rset][: eng.free()]
                    else:
                        # prefetch only: the whole non-resident window; the driver
                        # evicts least recently migrated blocks (any) beyond the
                        # free frames
                        todo = [b for b in window if b not in rset][: eng.free() + len(res)]
                        extra = len(todo) - eng.free()
                        if extra > 0:
                            victims = res[:extra]
                            wb = [b for b in victims if b not in inactive]
                            iv = [b for b in victims if b in inactive]
                            if not invalidate:
                                wb, iv = wb + iv, []
                            st[3], st[4] = len(wb), len(iv)
                            if wb:
                                eng.migrate(D2H, wb); d2h += len(wb)
                            if iv:
                                eng.migrate(INVALIDATE, iv); inv += len(iv)
                    st[5] = len(todo)
                    if todo:
                        eng.migrate(H2D, todo); h2d += len(todo)
            if per_launch is not None:
                per_launch.append(tuple(st))
            if check is not None:
                check(k, eng)
    return {"faults_per_iter": faults_per_iter, "h2d": h2d, "d2h": d2h, "inv": inv}


class OracleLoop(LoopEngine):
    def __init__(self, tr, N: int, R=2048, A=2, S=4, inactive=None):
        import oracle as orc
        self.orc = orc
        self.o = orc.Oracle(R=R, A=A, S=S, N=max(N, 0), W=tr.W, C=tr.C)
        if inactive is not None and len(inactive):
            self.o.mark_inactive(np.asarray(sorted(inactive), np.uint32), True)

    def record(self, h, faults):
        return int(self.o.record_faults(np.array([h], np.uint64), np.array([0, len(faults)], np.uint64),
                                        np.array(faults, np.uint32))[0])

    def build(self):
        self.o.build_tables()

    def predict1(self, q):
        off, pairs, _, _ = self.o.predict(np.array([q], np.uint32))
        return [int(b) for b in pairs[:, 0]]

    def select1(self, blocks, anchor):
        pairs = np.array([[b, 0] for b in blocks], np.uint32).reshape(-1, 2)
        wo, wb, io, iv = self.o.select(np.array([0, len(blocks)], np.uint64), pairs, np.array([anchor], np.uint32))
        return [int(x) for x in wb], [int(x) for x in iv]

    def migrate(self, d, blocks):
        rc = self.o.migrate(d, blocks)
        assert rc == 0, rc

    def resident(self):
        st = self.orc.parse_dump(self.o.dump(self.orc.RES), self.orc.RES, 0, 1, 1, 1)
        return [int(x) for x in st["lrm"]]

    def free(self):
        return self.o.free_frames

    def snapshot(self):
        return self.o.dump(self.orc.RES)
