"""Shared helpers for the GPU parity tests: drive the CUDA engine and the CPU
oracle with the same seeded inputs and compare their outputs."""
from __future__ import annotations

from typing import List, Tuple

import numpy as np
import torch

import oracle as orc
from paper_conf_asplos_jungkl23_b200 import binding as B
from paper_conf_asplos_jungkl23_b200 import Engine

NONE = 0xFFFFFFFF
ALL_TABLES = orc.EXEC | orc.CORR | orc.BLK | orc.WALK | orc.HIST


# engines created by the current test (conftest reads their path counters at teardown)
LIVE_ENGINES: list = []


def make_pair(R=2048, A=2, S=4, N=32, W=256, C=128, row_index=0, Emax=1024, fast=True, **kw):
    """An engine and the oracle on the same geometry.  fast: the engine answers
    conflict-free windows on the fast path (DUM_CFG_FAST_WINDOWS) -- the suite's
    default, so that both predict paths are covered; False: every window on the
    exact kernel (the library default, what bench.py times)."""
    if fast:
        kw["flags"] = kw.get("flags", 0) | B.DUM_CFG_FAST_WINDOWS
    eng = Engine(num_rows=R, assoc=A, num_succs=S, degree_n=N, max_blocks=W, max_exec_ids=Emax, hbm_frames=C,
                 row_index=row_index, **kw)
    LIVE_ENGINES.append(eng)
    o = orc.Oracle(R=R, A=A, S=S, N=N, W=W, C=C, row_index=row_index)
    return eng, o


def dev(a, dtype=np.uint32):
    if dtype == np.uint64:
        return B.as_u64_tensor(a, "cuda")
    return B.as_u32_tensor(a, "cuda")


def record_both(eng: Engine, o: orc.Oracle, h, off, f, host_ptrs=False) -> Tuple[np.ndarray, np.ndarray]:
    ex_o = o.record_faults(h, off, f)
    n = len(h)
    out = torch.empty(max(n, 1), dtype=torch.int32, device="cuda")
    if host_ptrs:
        eng.record_faults(np.asarray(h, np.uint64), np.asarray(off, np.uint64), np.asarray(f, np.uint32), out[:n])
    else:
        eng.record_faults(dev(h, np.uint64), dev(off, np.uint64), dev(f), out[:n])
    ex_g = B.u32(out[:n])
    return ex_o, ex_g


def build_both(eng: Engine, o: orc.Oracle):
    o.build_tables()
    eng.build_tables()
    eng.sync()


def assert_same_state(eng: Engine, o: orc.Oracle, what=ALL_TABLES, msg=""):
    a = eng.dump_state(what)
    b = o.dump(what)
    if a != b:
        E = o.num_exec
        da = orc.parse_dump(a, what, E, o.R, o.A, o.S) if what & orc.EXEC else None
        db = orc.parse_dump(b, what, E, o.R, o.A, o.S) if what & orc.EXEC else None
        detail = ""
        if da is not None and db is not None:
            for k in db:
                va, vb = da.get(k), db[k]
                if isinstance(vb, np.ndarray):
                    same = isinstance(va, np.ndarray) and va.shape == vb.shape and np.array_equal(va, vb)
                elif isinstance(vb, list) and vb and isinstance(vb[0], np.ndarray):
                    same = len(va) == len(vb) and all(np.array_equal(x, y) for x, y in zip(va, vb))
                    if not same:
                        for i, (x, y) in enumerate(zip(va, vb)):
                            if not np.array_equal(x, y):
                                detail += " %s[e=%d] gpu=%s orc=%s" % (k, i, list(x[:20]), list(y[:20]))
                                break
                else:
                    same = va == vb
                if not same:
                    detail += " differs:%s" % k
        raise AssertionError("state mismatch %s (%d vs %d bytes)%s" % (msg, len(a), len(b), detail))


def predict_both(eng: Engine, o: orc.Oracle, queries: np.ndarray):
    """Returns per-query lists from both sides: [(pairs, kern_off, chain)]"""
    q = np.ascontiguousarray(queries, dtype=np.uint32).reshape(-1, 6)
    off, pairs, ko, ch = o.predict(q)
    cap = int(off[-1]) + 16
    qd = dev(q.reshape(-1)).reshape(-1, 6)
    gp, grng, gko, gch, need = eng.predict_prefetch(qd, cap)
    try:
        eng.sync()
    except B.EngineError as e:      # pool reservation = pre-dedupe upper bound
        assert e.code == -2 and e.needed > cap, e
        gp, grng, gko, gch, need = eng.predict_prefetch(qd, int(e.needed))
        eng.sync()
    gp = B.u32(gp).reshape(-1, 2)
    grng = B.u64(grng).reshape(-1, 2)
    gko = B.u32(gko).reshape(len(q), -1)
    gch = B.u32(gch).reshape(len(q), -1)
    res_o, res_g = [], []
    for i in range(len(q)):
        res_o.append((pairs[int(off[i]):int(off[i + 1])], ko[i], ch[i]))
        res_g.append((gp[int(grng[i, 0]):int(grng[i, 1])], gko[i], gch[i]))
    return res_o, res_g, (gp, grng, qd)


def assert_same_predictions(res_o, res_g, msg=""):
    assert len(res_o) == len(res_g)
    for i, ((po, ko, co), (pg, kg, cg)) in enumerate(zip(res_o, res_g)):
        if not (np.array_equal(co, cg) and np.array_equal(ko, kg) and np.array_equal(po, pg)):
            raise AssertionError("query %d differs %s: chain gpu=%s orc=%s; n gpu=%d orc=%d; kern_off gpu=%s orc=%s"
                                 % (i, msg, list(cg[:6]), list(co[:6]), len(pg), len(po), list(kg[:6]), list(ko[:6])))


def select_both(eng: Engine, o: orc.Oracle, gp, grng, qd, queries: np.ndarray, res_o):
    q = np.asarray(queries, dtype=np.uint32).reshape(-1, 6)
    qoff = np.zeros(len(q) + 1, dtype=np.uint64)
    qoff[1:] = np.cumsum([len(p) for p, _, _ in res_o])
    allp = np.concatenate([p for p, _, _ in res_o]) if len(res_o) and qoff[-1] else np.zeros((0, 2), np.uint32)
    wo, wb, io, iv = o.select(qoff, allp, q[:, 4])
    # the GPU reserves `need` <= |window| entries per query in each pool
    cap = int(qoff[-1]) + 1
    # GPU side reads the predict output in place (ranges + pairs pool)
    gwb, ginv, grng2, need = eng.select_evictions(dev(grng.reshape(-1).view(np.uint64), np.uint64).reshape(-1, 2),
                                                  dev(gp.reshape(-1)), qd, cap)
    eng.sync()
    gwb, ginv, r = B.u32(gwb), B.u32(ginv), B.u64(grng2).reshape(-1, 4)
    for i in range(len(q)):
        ew, ei = wb[int(wo[i]):int(wo[i + 1])], iv[int(io[i]):int(io[i + 1])]
        aw, ai = gwb[int(r[i, 0]):int(r[i, 1])], ginv[int(r[i, 2]):int(r[i, 3])]
        if not (np.array_equal(ew, aw) and np.array_equal(ei, ai)):
            raise AssertionError("select query %d: wb gpu=%d orc=%d inv gpu=%d orc=%d" % (i, len(aw), len(ew), len(ai), len(ei)))
    return wb, iv


def fused_both(eng: Engine, o: orc.Oracle, queries: np.ndarray):
    """dum_predict_select (fused a7+a8) vs the oracle's predict then select."""
    q = np.ascontiguousarray(queries, dtype=np.uint32).reshape(-1, 6)
    off, pairs, ko, ch = o.predict(q)
    wo, wb, io, iv = o.select(off, pairs, q[:, 4])
    qd = dev(q.reshape(-1)).reshape(-1, 6)
    cap = int(off[-1]) + 16
    while True:
        out = eng.predict_select(qd, cap, sel_cap=cap)
        try:
            eng.sync()
            break
        except B.EngineError as e:
            assert e.code == -2 and e.needed > cap, e
            cap = int(e.needed)
    gp, grng, gko, gch, _, gwb, ginv, gsr, _ = out
    gp = B.u32(gp).reshape(-1, 2)
    grng = B.u64(grng).reshape(-1, 2)
    gko = B.u32(gko).reshape(len(q), -1)
    gch = B.u32(gch).reshape(len(q), -1)
    gwb, ginv, r = B.u32(gwb), B.u32(ginv), B.u64(gsr).reshape(-1, 4)
    for i in range(len(q)):
        po = pairs[int(off[i]):int(off[i + 1])]
        pg = gp[int(grng[i, 0]):int(grng[i, 1])]
        assert np.array_equal(po, pg) and np.array_equal(ko[i], gko[i]) and np.array_equal(ch[i], gch[i]), \
            "fused predict query %d: n gpu=%d orc=%d" % (i, len(pg), len(po))
        ew, ei = wb[int(wo[i]):int(wo[i + 1])], iv[int(io[i]):int(io[i + 1])]
        aw, ai = gwb[int(r[i, 0]):int(r[i, 1])], ginv[int(r[i, 2]):int(r[i, 3])]
        assert np.array_equal(ew, aw) and np.array_equal(ei, ai), \
            "fused select query %d: wb gpu=%d orc=%d inv gpu=%d orc=%d" % (i, len(aw), len(ew), len(ai), len(ei))


def transition_queries(exec_seq: List[int], first: int, n: int, N: int) -> np.ndarray:
    pad = [NONE, NONE, NONE] + list(exec_seq)
    qs = []
    for k in range(first, first + n):
        qs.append([exec_seq[k], pad[k], pad[k + 1], pad[k + 2], NONE, N])
    return np.array(qs, dtype=np.uint32).reshape(-1, 6)
