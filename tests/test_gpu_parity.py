"""GPU parity: the CUDA engine (through the C-ABI) against the CPU oracle on
the same seeded inputs.  Integer state -> bit-exact comparisons of canonical
dumps, per-query prefetch lists and eviction sets."""
from __future__ import annotations

import numpy as np
import pytest
import torch

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)

import oracle as orc  # noqa: E402
import workloads as wl  # noqa: E402
from gpu_helpers import (ALL_TABLES, NONE, assert_same_predictions, assert_same_state, build_both,  # noqa: E402
                         dev, fused_both, make_pair, predict_both, record_both, select_both, transition_queries)
from paper_conf_asplos_jungkl23_b200 import binding as B  # noqa: E402

TABLE6 = {  # PAPER.md Table 6 (L429-L443): name -> (Assoc, NumSuccs, NumRows)
    "Config0": (2, 4, 128), "Config1": (2, 8, 128), "Config2": (4, 4, 128), "Config3": (2, 4, 512),
    "Config4": (2, 8, 512), "Config5": (4, 4, 512), "Config6": (2, 4, 1024), "Config7": (2, 8, 1024),
    "Config8": (4, 4, 1024), "Config9": (2, 4, 2048), "Config10": (2, 8, 2048), "Config11": (4, 4, 2048),
    "Config12": (2, 4, 4096),
}


def _run_trace_per_iteration(eng, o, tr, N, check_every=True, host_ptrs=False, queries=True, select=True):
    """Bench schedule per iteration i: record(i) -> predict(i) on
    the state built through i-1 -> select -> build(i)."""
    ex_all = []
    for i in range(tr.n_iter):
        h, off, f = tr.iteration(i)
        exo, exg = record_both(eng, o, h, off, f, host_ptrs=host_ptrs)
        assert np.array_equal(exo, exg), "exec ids iteration %d" % i
        ex_all += [int(x) for x in exo]
        if queries and i >= 1:
            qs = transition_queries(ex_all, i * tr.K, tr.K, N)
            ro, rg, (gp, grng, qd) = predict_both(eng, o, qs)
            assert_same_predictions(ro, rg, msg="iteration %d" % i)
            if select:
                select_both(eng, o, gp, grng, qd, qs, ro)
                fused_both(eng, o, qs)
        build_both(eng, o)
        if check_every:
            assert_same_state(eng, o, msg="iteration %d" % i)
    return ex_all


def test_config_T_all_calls_parity():
    tr = wl.make_T()
    eng, o = make_pair(W=tr.W, C=tr.C, N=32)
    # a residency snapshot for select: the generator's LRM snapshot at iteration 5
    snap = tr.snap_blk[5][: int(tr.snap_cnt[5])]
    o.load_residency(snap)
    eng.load_residency(dev(snap))
    _run_trace_per_iteration(eng, o, tr, N=32)
    assert_same_state(eng, o, what=ALL_TABLES | orc.RES)


@pytest.mark.parametrize("N", [0, 1, 2, 4])
def test_config_T_degrees(N):
    tr = wl.make_T()
    eng, o = make_pair(W=tr.W, C=tr.C, N=max(N, 1))
    _run_trace_per_iteration(eng, o, tr, N=N, check_every=False, select=False)
    assert_same_state(eng, o)


@pytest.mark.parametrize("name", sorted(TABLE6))
def test_table6_geometries_on_T(name):
    A, S, R = TABLE6[name]
    tr = wl.make_T(dup_ppm=200_000)
    eng, o = make_pair(R=R, A=A, S=S, W=tr.W, C=tr.C, N=8)
    _run_trace_per_iteration(eng, o, tr, N=8, check_every=False, select=False)
    assert_same_state(eng, o)


@pytest.mark.parametrize("geom", [(16, 1, 1), (16, 2, 4), (16, 1, 4), (16, 2, 1), (1, 3, 2), (1, 1, 1),
                                  (4, 4, 8), (8, 5, 3), (2048, 2, 4)])
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_random_traces_stress_geometries(geom, seed):
    """Replacement pressure, duplicates, empty launches, repeated exec IDs in one
    batch, several record calls per build, fault-anchored queries."""
    R, A, S = geom
    rng = np.random.default_rng(1000 * seed + R + 7 * A + 13 * S)
    W = 300
    eng, o = make_pair(R=R, A=A, S=S, W=W, C=40, N=6)
    ex_all = []
    for batch in range(6):
        n_rec = int(rng.integers(1, 4))
        for _ in range(n_rec):
            h, off, f = wl.random_trace(rng, n_launch=int(rng.integers(1, 40)), n_kernels=6, W=W, max_faults=80)
            exo, exg = record_both(eng, o, h, off, f, host_ptrs=bool(rng.integers(0, 2)))
            assert np.array_equal(exo, exg)
            ex_all += [int(x) for x in exo]
        build_both(eng, o)
        assert_same_state(eng, o, msg="batch %d" % batch)
        qs = transition_queries(ex_all, 0, len(ex_all), 6)
        # mix in fault-anchored queries (anchor = a random block) and n < N
        anch = qs.copy()
        anch[:, 4] = rng.integers(0, W, len(anch))
        anch[:, 5] = rng.integers(0, 7, len(anch))
        allq = np.concatenate([qs, anch])
        ro, rg, (gp, grng, qd) = predict_both(eng, o, allq)
        assert_same_predictions(ro, rg, msg="batch %d" % batch)
        n_res = int(rng.integers(0, 41))
        snap = rng.permutation(W)[:n_res].astype(np.uint32)
        o.load_residency(snap)
        eng.load_residency(dev(snap))
        inact = rng.permutation(W)[: W // 4].astype(np.uint32)
        o.mark_inactive(inact, True)
        eng.mark_inactive(dev(inact), True)
        select_both(eng, o, gp, grng, qd, allq, ro)
        fused_both(eng, o, allq)


def test_block_ids_near_limit_and_fmix_index():
    W = 1 << 20
    rng = np.random.default_rng(5)
    eng, o = make_pair(R=64, A=2, S=4, W=W, C=16, N=4, row_index=1)
    hi = np.arange(W - 200, W, dtype=np.uint32)
    lists = [list(rng.choice(hi, 30)) for _ in range(20)]
    h = np.array([wl.fnv1a64(b"k%d" % (i % 5)) for i in range(20)], dtype=np.uint64)
    off = np.zeros(21, dtype=np.uint64)
    off[1:] = np.cumsum([len(x) for x in lists])
    f = np.array([b for x in lists for b in x], dtype=np.uint32)
    exo, exg = record_both(eng, o, h, off, f)
    assert np.array_equal(exo, exg)
    build_both(eng, o)
    assert_same_state(eng, o)
    qs = transition_queries([int(x) for x in exo], 0, 20, 4)
    ro, rg, _ = predict_both(eng, o, qs)
    assert_same_predictions(ro, rg)



@pytest.mark.parametrize("dup_frac", [0.0, 0.05])
def test_big_launches_hashed_ingest_bitmap(dup_frac):
    """W = 2^20: big launches (> 1024 records) dedupe through a hashed
    shared-memory bitmap; shared bits are only candidates, settled by the
    min-position hash (D2: first occurrence kept, order preserved).  The
    12000-record launch has more candidates than that hash holds and takes
    the global-pool path."""
    W = 1 << 20
    rng = np.random.default_rng(11 + int(100 * dup_frac))
    eng, o = make_pair(R=64, A=2, S=4, W=W, C=64, N=4)
    sizes = [1500, 3000, 4000, 12000, 700, 3345]
    lists = []
    for n in sizes:
        x = rng.choice(W, n, replace=False)
        k = int(dup_frac * n)
        if k:
            x[rng.integers(1, n, k)] = x[rng.integers(0, n // 2, k)]
        lists.append([int(v) for v in x])
    lists.append(list(range(5000, 7000)) + list(range(5000 + W // 2, 6000 + W // 2)))  # runs, far regions
    h = np.array([wl.fnv1a64(b"big%d" % (i % 3)) for i in range(len(lists))], dtype=np.uint64)
    off = np.zeros(len(lists) + 1, dtype=np.uint64)
    off[1:] = np.cumsum([len(x) for x in lists])
    f = np.array([b for x in lists for b in x], dtype=np.uint32)
    exo, exg = record_both(eng, o, h, off, f)
    assert np.array_equal(exo, exg)
    build_both(eng, o)
    assert_same_state(eng, o)
    c = eng.counters()
    assert c["NORM_RECORDS"] == sum(len(dict.fromkeys(x)) for x in lists)
    assert (c["INGEST_DUP"] > 0) == (dup_frac > 0)

def test_hash_sentinel_and_collisions():
    """Two launches with the same hash share an ID; the all-ones hash is a
    legal key (D3)."""
    eng, o = make_pair(W=64, C=8, N=2)
    h = np.array([0xFFFFFFFFFFFFFFFF, 7, 0xFFFFFFFFFFFFFFFF, 7, 0, 0], dtype=np.uint64)
    off = np.array([0, 2, 2, 5, 6, 6, 8], dtype=np.uint64)
    f = np.array([1, 2, 3, 4, 3, 9, 1, 1], dtype=np.uint32)
    exo, exg = record_both(eng, o, h, off, f)
    assert list(exo) == [0, 1, 0, 1, 2, 2] and np.array_equal(exo, exg)
    build_both(eng, o)
    assert_same_state(eng, o)


@pytest.mark.parametrize("config", ["B", "G"])
def test_full_size_tables_and_sampled_predictions(config):
    """BASELINE.json configs[1] / configs[2] at full size (3 iterations): the
    complete table state is compared byte for byte; predictions and selections
    on a seeded sample of queries in the bench's launch configuration."""
    tr = wl.make(config, n_iter=3)
    eng, o = make_pair(W=tr.W, C=tr.C, N=32, Emax=8192)
    ex_all = []
    for i in range(tr.n_iter):
        h, off, f = tr.iteration(i)
        exo, exg = record_both(eng, o, h, off, f)
        assert np.array_equal(exo, exg)
        ex_all += [int(x) for x in exo]
        build_both(eng, o)
    st = eng.stats()
    assert st.slow_walks == 0
    assert_same_state(eng, o)
    rng = np.random.default_rng(11)
    pick = np.sort(rng.choice(np.arange(2 * tr.K, 3 * tr.K), 64, replace=False))
    allq = transition_queries(ex_all, 0, len(ex_all), 32)[pick]
    ro, rg, (gp, grng, qd) = predict_both(eng, o, allq)
    assert_same_predictions(ro, rg)
    snap = tr.snap_blk[2][: int(tr.snap_cnt[2])]
    o.load_residency(snap)
    eng.load_residency(dev(snap))
    o.mark_inactive(tr.inactive_blocks, True)
    eng.mark_inactive(dev(tr.inactive_blocks), True)
    select_both(eng, o, gp, grng, qd, allq, ro)
    fused_both(eng, o, allq)


def test_full_batch_of_ten_iterations_in_one_build():
    """Config T recorded as one 40-launch batch, built once (multi-launch groups
    per exec ID inside one build)."""
    tr = wl.make_T(dup_ppm=300_000)
    eng, o = make_pair(W=tr.W, C=tr.C, N=32)
    exo, exg = record_both(eng, o, tr.launch_hash, tr.launch_off, tr.fault_block)
    assert np.array_equal(exo, exg)
    build_both(eng, o)
    assert_same_state(eng, o)


def test_errors_are_reported():
    eng, o = make_pair(W=64, C=8, N=2)
    with pytest.raises(B.EngineError):  # host offsets not launch-aligned: refused at once
        eng.record_faults(np.array([1], np.uint64), np.array([0, 2], np.uint64), np.array([3], np.uint32))
    # out-of-range block id from host memory: detected on the device (sticky)
    eng.record_faults(np.array([1], np.uint64), np.array([0, 1], np.uint64), np.array([64], np.uint32))
    with pytest.raises(B.EngineError):
        eng.sync()
    eng.build_tables()
    eng.sync()
    # device-side detection of an out-of-range block id
    eng.record_faults(dev(np.array([1], np.uint64), np.uint64), dev(np.array([0, 1], np.uint64), np.uint64),
                      dev(np.array([99], np.uint32)))
    with pytest.raises(B.EngineError):
        eng.sync()
    eng.build_tables()
    eng.sync()
    # predict capacity too small -> ECAPACITY with the needed size
    eng2, o2 = make_pair(W=64, C=8, N=2)
    h = np.array([5, 6, 5, 6, 5, 6], np.uint64)
    off = np.array([0, 3, 6, 9, 12, 15, 18], np.uint64)
    f = np.arange(18, dtype=np.uint32) % 12
    record_both(eng2, o2, h, off, f)
    build_both(eng2, o2)
    q = dev(transition_queries([0, 1, 0, 1, 0, 1], 3, 3, 2).reshape(-1)).reshape(-1, 6)
    eng2.predict_prefetch(q, 1)
    with pytest.raises(B.EngineError) as ei:
        eng2.sync()
    assert getattr(ei.value, "needed", 0) > 1


def _big_launch_trace(rng, n_launch, pool, W, lo, hi, repeat_prob):
    """Launches of thousands of faults: a kernel's list is mostly contiguous
    tensor ranges (some repeated from its previous launch, some fresh) with
    random blocks and duplicates mixed in."""
    hashes, offs, faults = [], [0], []
    last = {}
    for _ in range(n_launch):
        k = int(rng.integers(len(pool)))
        n = int(rng.integers(lo, hi))
        if k in last and rng.random() < repeat_prob:
            lst = list(last[k])
        else:
            lst = []
            while len(lst) < n:
                start, ln = int(rng.integers(0, W)), int(rng.integers(16, 600))
                lst += [(start + x) % W for x in range(ln)]
            lst = lst[:n]
            for i in range(len(lst)):
                r = rng.random()
                if r < 0.05:
                    lst[i] = int(rng.integers(0, W))
                elif r < 0.08 and i:
                    lst[i] = lst[int(rng.integers(0, i))]
        last[k] = lst
        hashes.append(pool[k])
        faults += lst
        offs.append(len(faults))
    return (np.array(hashes, dtype=np.uint64), np.array(offs, dtype=np.uint64),
            np.array(faults, dtype=np.uint32))


@pytest.mark.parametrize("R", [2048, 64, 16])
def test_big_exec_ids_partitioned_apply_and_long_walks(R):
    """Exec IDs with thousands of operations per batch: the apply is split
    into up to R/32 set partitions (several launches of one exec ID per batch,
    several apply rounds per partition), walks longer than the shared-memory
    scratch (global row cache / positions / dedupe hash), both the
    duplicate-free fast path and the dedupe path."""
    rng = np.random.default_rng(77 + R)
    W = 20000
    eng, o = make_pair(R=R, A=2, S=4, W=W, C=3000, N=4, max_batch_faults=1 << 18)
    pool = [wl.fnv1a64(b"big%d" % i) for i in range(4)]
    ex_all = []
    for batch in range(4):
        h, off, f = _big_launch_trace(rng, n_launch=int(rng.integers(3, 9)), pool=pool, W=W, lo=1200, hi=5200,
                                      repeat_prob=0.5)
        exo, exg = record_both(eng, o, h, off, f, host_ptrs=bool(batch & 1))
        assert np.array_equal(exo, exg)
        ex_all += [int(x) for x in exo]
        build_both(eng, o)
        assert_same_state(eng, o, msg="R=%d batch %d" % (R, batch))
        qs = transition_queries(ex_all, 0, len(ex_all), 4)
        ro, rg, _ = predict_both(eng, o, qs)
        assert_same_predictions(ro, rg, msg="R=%d batch %d" % (R, batch))


@pytest.mark.parametrize("trace", ["T", "big"])
def test_overlapped_ingest_no_host_syncs(trace):
    """The bench schedule issued back to back with no host synchronisation:
    record(i+1) runs on the engine's ingest stream (DUM_INPUTS_READY, and host
    pointers) while build(i) runs; every iteration's predictions (kept in
    their own buffers) and the final tables must equal the oracle's."""
    rng = np.random.default_rng(5)
    if trace == "T":
        tr = wl.make_T()
        batches = [tr.iteration(i) for i in range(tr.n_iter)]
        eng, o = make_pair(R=2048, A=2, S=4, W=tr.W, C=tr.C, N=2)
        N = 2
    else:
        W = 20000
        pool = [wl.fnv1a64(b"ov%d" % i) for i in range(5)]
        batches = [_big_launch_trace(rng, n_launch=6, pool=pool, W=W, lo=200, hi=3000, repeat_prob=0.6)
                   for _ in range(6)]
        eng, o = make_pair(R=64, A=2, S=4, W=W, C=3000, N=3, max_batch_faults=1 << 17)
        N = 3
    dev_b = [(dev(h, np.uint64), dev(off, np.uint64), dev(f)) for h, off, f in batches]
    torch.cuda.synchronize()
    ex_all, ex_dev, outs, qs_all = [], [], [], []
    for i, (h, off, f) in enumerate(batches):
        ex_o = o.record_faults(h, off, f)
        out = torch.empty(len(h), dtype=torch.int32, device="cuda")
        if i % 3 == 2:
            eng.record_faults(np.asarray(h, np.uint64), np.asarray(off, np.uint64), np.asarray(f, np.uint32), out)
        else:
            eng.record_faults(*dev_b[i], out, ready=i > 0)
        ex_dev.append(out)
        prev = len(ex_all)
        ex_all += [int(x) for x in ex_o]
        if i >= 1:
            qs = transition_queries(ex_all, prev, len(h), N)
            qd = dev(qs.reshape(-1)).reshape(-1, 6)
            off_o, pairs_o, ko_o, ch_o = o.predict(np.ascontiguousarray(qs, dtype=np.uint32).reshape(-1, 6))
            # a window gathers at most N + 1 walks of at most 1 + S (rows) blocks each
            cap = len(qs) * (N + 1) * 5 * (int(np.diff(off).max()) + 1) + 64
            gp, grng, gko, gch, _ = eng.predict_prefetch(qd, cap)
            outs.append((gp, grng, gko, gch, off_o, pairs_o, ko_o, ch_o))
        o.build_tables()
        eng.build_tables()
    eng.sync()
    for i, (h, _, _) in enumerate(batches):
        assert np.array_equal(B.u32(ex_dev[i]), np.array(ex_all[sum(len(b[0]) for b in batches[:i]):][:len(h)],
                                                         dtype=np.uint32)), "exec ids of batch %d" % i
    for j, (gp, grng, gko, gch, off_o, pairs_o, ko_o, ch_o) in enumerate(outs):
        gp = B.u32(gp).reshape(-1, 2)
        grng = B.u64(grng).reshape(-1, 2)
        gko = B.u32(gko).reshape(len(grng), -1)
        gch = B.u32(gch).reshape(len(grng), -1)
        for q in range(len(grng)):
            assert np.array_equal(gp[int(grng[q, 0]):int(grng[q, 1])], pairs_o[int(off_o[q]):int(off_o[q + 1])]), \
                "batch %d query %d" % (j + 1, q)
            assert np.array_equal(gko[q], ko_o[q]) and np.array_equal(gch[q], ch_o[q])
    assert_same_state(eng, o)


@pytest.mark.parametrize("R", [2048, 16])
def test_sequential_walker_mode_builds_identical_walks(R):
    """DUM_CFG_SEQ_WALKS: every walk is built by the sequential one-warp walker
    (k_walk_slow, the literal PAPER.md L218-L224 loop); the walk cache and the
    windows must equal the oracle's exactly as with the parallel walker."""
    rng = np.random.default_rng(900 + R)
    W = 5000
    eng, o = make_pair(R=R, A=2, S=4, W=W, C=800, N=4, max_batch_faults=1 << 17, flags=B.DUM_CFG_SEQ_WALKS)
    pool = [wl.fnv1a64(b"sq%d" % i) for i in range(6)]
    ex_all = []
    for batch in range(3):
        h, off, f = _big_launch_trace(rng, n_launch=8, pool=pool, W=W, lo=20, hi=1500, repeat_prob=0.5)
        exo, exg = record_both(eng, o, h, off, f)
        assert np.array_equal(exo, exg)
        ex_all += [int(x) for x in exo]
        build_both(eng, o)
        assert_same_state(eng, o, msg="batch %d" % batch)
        qs = transition_queries(ex_all, 0, len(ex_all), 4)
        ro, rg, _ = predict_both(eng, o, qs)
        assert_same_predictions(ro, rg)
    c = eng.counters()
    assert c["WALK_SLOW"] > 0 and c["WALK_DEDUPE"] == 0, c


@pytest.mark.parametrize("host,graph", [(True, False), (False, False), (True, True), (False, True)])
def test_dum_step_equals_the_separate_calls(host, graph):
    """dum_step (record -> queries -> predict+select -> build in one call) on
    Config T with a residency snapshot and inactive blocks: every iteration's
    windows, victims and the final tables equal the oracle's."""
    tr = wl.make_T(dup_ppm=100_000)
    N = 2
    eng, o = make_pair(W=tr.W, C=tr.C, N=N)
    snap = tr.snap_blk[4][: int(tr.snap_cnt[4])]
    o.load_residency(snap)
    eng.load_residency(dev(snap))
    inact = np.arange(0, tr.W, 5, dtype=np.uint32)
    o.mark_inactive(inact, True)
    eng.mark_inactive(dev(inact), True)
    out = {}
    ex_all = []
    eng.set_step_graphs(graph)  # graph: one CUDA graph per staging set, replayed
    for i in range(tr.n_iter):
        h, off, f = tr.iteration(i)
        ex_all += [int(x) for x in o.record_faults(h, off, f)]
        qs = transition_queries(ex_all, i * tr.K, tr.K, N)
        off_o, pairs_o, ko_o, ch_o = o.predict(qs)
        wo, wb_o, io, iv_o = o.select(off_o, pairs_o, qs[:, 4])
        o.build_tables()
        if host:
            eng.step(np.asarray(h, np.uint64), np.asarray(off, np.uint64), np.asarray(f, np.uint32), 4096, 4096, out)
        else:
            eng.step(dev(h, np.uint64), dev(off, np.uint64), dev(f), 4096, 4096, out)
        eng.sync()
        gp, rg = B.u32(out["pairs"]).reshape(-1, 2), B.u64(out["rng"]).reshape(-1, 2)
        sr = B.u64(out["sel_rng"]).reshape(-1, 4)
        gwb, giv = B.u32(out["wb"]), B.u32(out["inv"])
        for q in range(tr.K):
            assert np.array_equal(gp[rg[q, 0]:rg[q, 1]], pairs_o[off_o[q]:off_o[q + 1]]), (i, q)
            assert np.array_equal(B.u32(out["kern_off"])[q], ko_o[q]) and np.array_equal(B.u32(out["chain"])[q], ch_o[q])
            assert np.array_equal(gwb[sr[q, 0]:sr[q, 1]], wb_o[wo[q]:wo[q + 1]]), (i, q)
            assert np.array_equal(giv[sr[q, 2]:sr[q, 3]], iv_o[io[q]:io[q + 1]]), (i, q)
    assert_same_state(eng, o)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_fast_selection_on_a_log_with_stale_entries(seed):
    """Write-backs leave stale entries in the LRM log (PAPER.md L238-L241:
    the victims are resident blocks; a logged block that left HBM is skipped)
    until the next compaction: the fast path's per-entry selection
    (k_select_stale) must give the oracle's victims.  The clean-log path
    (k_window_fast) answers the same queries after the log is reloaded."""
    W, C = 96, 40
    rng = np.random.default_rng(77 + seed)
    arena = torch.zeros(W * (2 << 20), dtype=torch.uint8).pin_memory()
    pool = torch.zeros(C * (2 << 20), dtype=torch.uint8, device="cuda")
    eng, o = make_pair(R=16, A=2, S=4, W=W, C=C, N=6, host_arena=arena, frame_pool=pool)
    # kernels with disjoint block ranges (16 blocks each): their walks share no
    # block, so the windows take the fast path
    ex_all = []
    for _ in range(3):
        ks = [k % 6 for k in range(30)]
        h = np.array([wl.fnv1a64(b"dk%d" % k) for k in ks], dtype=np.uint64)
        lists = [[16 * k + int(x) for x in rng.permutation(16)[: int(rng.integers(4, 17))]] for k in ks]
        off = np.zeros(len(ks) + 1, dtype=np.uint64)
        off[1:] = np.cumsum([len(x) for x in lists])
        f = np.array([b for x in lists for b in x], dtype=np.uint32)
        exo, exg = record_both(eng, o, h, off, f)
        assert np.array_equal(exo, exg)
        ex_all += [int(x) for x in exo]
    build_both(eng, o)
    qs = transition_queries(ex_all, 0, len(ex_all), 6)
    inact = rng.permutation(W)[: W // 3].astype(np.uint32)
    o.mark_inactive(inact, True)
    eng.mark_inactive(dev(inact), True)
    snap = rng.permutation(W)[:C].astype(np.uint32)
    o.load_residency(snap)
    eng.load_residency(dev(snap))
    # write back blocks from the middle of the log, then fault others in
    for d, blocks in ((B.D2H, snap[3:15:2]), (B.H2D, [b for b in rng.permutation(W) if b not in set(snap)][:4])):
        blocks = np.asarray(blocks, np.uint32)
        assert o.migrate(d, blocks) == 0
        eng.migrate_blocks(d, dev(blocks))
        eng.sync()
    assert eng.dump_state(orc.RES) == o.dump(orc.RES)
    c0 = eng.counters()
    fused_both(eng, o, qs)
    c1 = eng.counters()
    assert c1.get("FAST_DIRTY", 0) > c0.get("FAST_DIRTY", 0), "the stale-entry path did not run"
    # the same queries on a compacted (clean) log: the live entries, log order
    rs = orc.parse_dump(o.dump(orc.RES), orc.RES, 0, 1, 1, 1)
    live = set(int(b) for b in rs["block_of_frame"] if b != orc.NONE)
    res = np.asarray([b for b in rs["lrm"] if (int(b) & 0x7FFFFFFF) in live], np.uint32) & 0x7FFFFFFF
    assert len(res) == len(live)
    o.load_residency(res)
    eng.load_residency(dev(res))
    c0 = eng.counters()
    fused_both(eng, o, qs)
    c1 = eng.counters()
    assert c1["Q_FAST"] > c0["Q_FAST"] and c1["FAST_DIRTY"] == c0["FAST_DIRTY"]


@pytest.mark.parametrize("fast", [False, True])
def test_graph_steps_then_separate_calls(fast):
    """Graph-replayed dum_step leaves its jump tables and (exact windows) the
    publishing of its rebuilt walks to what comes next; here the next calls
    are the separate record / predict+select / build calls, then dum_step
    again (uncaptured first use, then replays): every window, victim list and
    the final tables equal the oracle's."""
    tr = wl.make_T(dup_ppm=50_000)
    N = 2
    eng, o = make_pair(W=tr.W, C=tr.C, N=N, fast=fast)
    snap = tr.snap_blk[4][: int(tr.snap_cnt[4])]
    o.load_residency(snap)
    eng.load_residency(dev(snap))
    ex_all, out = [], {}
    eng.set_step_graphs(True)
    for i in range(tr.n_iter):
        h, off, f = tr.iteration(i)
        exo = o.record_faults(h, off, f)
        ex_all += [int(x) for x in exo]
        qs = transition_queries(ex_all, i * tr.K, tr.K, N)
        off_o, pairs_o, ko_o, ch_o = o.predict(qs)
        wo, wb_o, io, iv_o = o.select(off_o, pairs_o, qs[:, 4])
        if i in (4, 5):  # separate calls between replayed steps
            exg = torch.empty(len(h), dtype=torch.int32, device="cuda")
            eng.record_faults(dev(h, np.uint64), dev(off, np.uint64), dev(f), exg)
            assert np.array_equal(B.u32(exg), exo)
            if i >= 1:
                fused_both(eng, o, qs)
            o.build_tables()
            eng.build_tables()
            eng.sync()
            continue
        o.build_tables()
        eng.step(dev(h, np.uint64), dev(off, np.uint64), dev(f), 4096, 4096, out)
        eng.sync()
        gp, rg = B.u32(out["pairs"]).reshape(-1, 2), B.u64(out["rng"]).reshape(-1, 2)
        sr = B.u64(out["sel_rng"]).reshape(-1, 4)
        gwb, giv = B.u32(out["wb"]), B.u32(out["inv"])
        # (dum_step's query history spans dum_step calls only: after the
        # separate calls its first three queries differ from the true history)
        for q in range(3 if i == 6 else 0, tr.K):
            assert np.array_equal(gp[rg[q, 0]:rg[q, 1]], pairs_o[off_o[q]:off_o[q + 1]]), (i, q)
            assert np.array_equal(gwb[sr[q, 0]:sr[q, 1]], wb_o[wo[q]:wo[q + 1]]), (i, q)
            assert np.array_equal(giv[sr[q, 2]:sr[q, 3]], iv_o[io[q]:io[q + 1]]), (i, q)
        if i == 3:
            assert_same_state(eng, o, msg="after replayed steps")  # (publishes the pending walks)
    assert_same_state(eng, o)
