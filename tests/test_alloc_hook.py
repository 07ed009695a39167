"""Allocator hook: host logic on CPU
against a brute-force model of live PT bytes per UM block, and on the GPU with
PyTorch's real caching allocator and through dum_hook_flush into the engine."""
from __future__ import annotations

import numpy as np
import pytest

from paper_conf_asplos_jungkl23_b200 import alloc_hook as AH

MB = 1 << 20
BLK = 2 * MB
NONE = 0xFFFFFFFF
BASE = 0x7F0000000000


def brute_inactive(segments, live, W):
    """UM blocks of the segments (in creation order) with no live byte: the reading
    of D20 the hook implements (a block is invalidatable iff no live PT block overlaps it)."""
    out, base = {}, 0
    for (a, size) in segments:
        nb = (size + BLK - 1) // BLK
        for k in range(nb):
            b = base + k
            if b >= W:
                continue
            lo, hi = a + k * BLK, min(a + (k + 1) * BLK, a + size)
            out[b] = not any(x < hi and lo < x + n for (x, n) in live)
        base += nb
    return out


def test_hook_small_sequence():
    h = AH.AllocHook(max_blocks=64)
    h.feed(AH.SEGMENT_ALLOC, BASE, 10 * MB)                   # blocks 0..4, free memory
    ina, act = h.drain()
    assert list(ina) == [0, 1, 2, 3, 4] and len(act) == 0
    h.feed(AH.ALLOC, BASE, 3 * MB)                            # blocks 0, 1 active
    ina, act = h.drain()
    assert len(ina) == 0 and list(act) == [0, 1]
    h.feed(AH.ALLOC, BASE + 3 * MB, 1 * MB)                   # block 1 again: no change
    assert all(len(x) == 0 for x in h.drain())
    h.feed(AH.FREE_REQUESTED, BASE, 3 * MB)                   # not yet free (other streams)
    assert all(len(x) == 0 for x in h.drain())
    h.feed(AH.FREE_COMPLETED, BASE, 3 * MB)                   # block 0 inactive, block 1 keeps 1 MiB
    ina, act = h.drain()
    assert list(ina) == [0] and len(act) == 0
    assert h.block_of(BASE + 5 * MB) == 2 and h.block_of(BASE + 10 * MB) == NONE and h.block_of(BASE - 1) == NONE
    h.feed(AH.SEGMENT_ALLOC, BASE + 64 * MB, 4 * MB)          # second segment: blocks 5, 6
    assert h.block_of(BASE + 64 * MB + 3 * MB) == 6
    h.drain()
    h.feed(AH.ALLOC, BASE + 1000 * MB, MB)                    # outside every segment: dropped
    st = h.stats()
    assert st["dropped"] == 1 and st["blocks"] == 7 and st["live_bytes"] == 1 * MB
    h.feed(AH.SEGMENT_FREE, BASE, 10 * MB)                    # block 1's last PT block goes with it
    ina, act = h.drain()
    assert 1 in list(ina) and h.block_of(BASE) == NONE


def test_hook_block_space_limit():
    h = AH.AllocHook(max_blocks=3)
    h.feed(AH.SEGMENT_ALLOC, BASE, 10 * MB)   # 5 blocks, 3 in the space
    ina, _ = h.drain()
    assert list(ina) == [0, 1, 2] and h.stats()["dropped"] >= 1
    h.feed(AH.ALLOC, BASE + 8 * MB, MB)       # block 4: outside the space
    assert all(len(x) == 0 for x in h.drain())


def test_hook_random_against_brute_force():
    rng = np.random.default_rng(7)
    W = 200
    h = AH.AllocHook(max_blocks=W)
    segments = [(BASE + i * (1 << 34), int(s) * MB) for i, s in enumerate(rng.integers(3, 41, 6))]
    state = {}
    for (a, size) in segments:
        h.feed(AH.SEGMENT_ALLOC, a, size)
    ina, act = h.drain()
    for b in ina:
        state[int(b)] = True
    live = []
    for step in range(400):
        if live and rng.random() < 0.45:
            x, n = live.pop(int(rng.integers(len(live))))
            h.feed(AH.FREE_COMPLETED, x, n)
        else:
            a, size = segments[int(rng.integers(len(segments)))]
            off = int(rng.integers(0, size // (256 << 10))) * (256 << 10)
            n = int(min(size - off, int(rng.integers(1, 16)) * (512 << 10)))
            if any(x < a + off + n and a + off < x + m for (x, m) in live):
                continue  # live PT blocks never overlap
            live.append((a + off, n))
            h.feed(AH.ALLOC, a + off, n)
        if step % 37 == 0 or step == 399:
            ina, act = h.drain()
            assert not set(ina.tolist()) & set(act.tolist())
            for b in ina:
                state[int(b)] = True
            for b in act:
                state[int(b)] = False
            want = brute_inactive(segments, live, W)
            assert {b: v for b, v in state.items() if b in want} == {b: want[b] for b in state if b in want}


@pytest.mark.gpu
def test_hook_real_allocator():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    torch.cuda.set_device(0)
    h = AH.AllocHook(max_blocks=1 << 16, device=0)
    h.attach()
    h.drain()
    x = torch.empty(24 * MB, dtype=torch.uint8, device="cuda")
    torch.cuda.synchronize()
    b0 = h.block_of(x.data_ptr())
    b1 = h.block_of(x.data_ptr() + x.numel() - 1)
    assert b0 != NONE and b1 != NONE and b1 >= b0
    ina, act = h.drain()
    assert b0 in set(act.tolist())
    del x
    torch.cuda.synchronize()
    ina, act = h.drain()
    inner = set(range(b0 + 1, b1))  # the tensor's interior blocks hold nothing else
    assert inner <= set(ina.tolist()), (sorted(inner - set(ina.tolist())), b0, b1)
    assert h.stats()["events"] >= 2


@pytest.mark.gpu
def test_hook_flush_marks_engine_blocks():
    """Config T with the inactive blocks produced by the hook (synthetic PT
    blocks over a 256-block segment, every 5th block freed): dum_hook_flush ->
    dum_mark_inactive; every iteration's victims equal the oracle's with the
    hook's drained list marked."""
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    import workloads as wl
    from gpu_helpers import dev, make_pair, transition_queries
    from paper_conf_asplos_jungkl23_b200 import binding as B
    tr = wl.make_T()
    N = 2
    eng, o = make_pair(W=tr.W, C=tr.C, N=N)
    h = AH.AllocHook(max_blocks=tr.W, device=0)
    h.feed(AH.SEGMENT_ALLOC, BASE, tr.W * BLK)
    for b in range(tr.W):
        h.feed(AH.ALLOC, BASE + b * BLK, BLK)          # one PT block per UM block, all live
    for b in range(0, tr.W, 5):
        h.feed(AH.FREE_COMPLETED, BASE + b * BLK, BLK)  # every 5th freed
    h.flush(eng)                                       # (drains: the oracle gets the same list below)
    inact = np.arange(0, tr.W, 5, dtype=np.uint32)
    o.mark_inactive(inact, True)
    snap = tr.snap_blk[4][: int(tr.snap_cnt[4])]
    o.load_residency(snap)
    eng.load_residency(dev(snap))
    out, ex_all, n_inv = {}, [], 0
    for i in range(tr.n_iter):
        hh, off, f = tr.iteration(i)
        ex_all += [int(x) for x in o.record_faults(hh, off, f)]
        qs = transition_queries(ex_all, i * tr.K, tr.K, N)
        off_o, pairs_o, _, _ = o.predict(qs)
        wo, wb_o, io, iv_o = o.select(off_o, pairs_o, qs[:, 4])
        o.build_tables()
        eng.step(dev(hh, np.uint64), dev(off, np.uint64), dev(f), 4096, 4096, out)
        eng.sync()
        sr = B.u64(out["sel_rng"]).reshape(-1, 4)
        gwb, giv = B.u32(out["wb"]), B.u32(out["inv"])
        for q in range(tr.K):
            assert np.array_equal(gwb[sr[q, 0]:sr[q, 1]], wb_o[wo[q]:wo[q + 1]]), (i, q)
            assert np.array_equal(giv[sr[q, 2]:sr[q, 3]], iv_o[io[q]:io[q + 1]]), (i, q)
        n_inv += sum(int(sr[q, 3] - sr[q, 2]) for q in range(tr.K))
    assert n_inv > 0  # the invalidation path was exercised
