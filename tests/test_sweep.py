"""Host logic of the §8(f) row-2 sensitivity sweep (tools/sweep_f2.py)."""
import os
import sys

import numpy as np
import pytest

sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tools"))
import sweep_f2  # noqa: E402
import workloads as wl  # noqa: E402


def _windows(norm, N, drop=0):
    pairs, rng, pos = [], [], 0
    for k in range(len(norm)):
        u = np.unique(np.concatenate(norm[k:k + N + 1]))[drop:]
        pairs.append(u)
        rng.append((pos, pos + u.size))
        pos += u.size
    return np.concatenate(pairs).astype(np.uint32), np.array(rng, dtype=np.int64)


def test_normalised_keeps_first_occurrence_in_order():
    tr = wl.make_T(n_iter=2, dup_ppm=200000)
    norm = sweep_f2.normalised(tr, 1)
    h, off, f = tr.iteration(1)
    for k, seg in enumerate(norm):
        raw = f[int(off[k]):int(off[k + 1])]
        want = list(dict.fromkeys(raw.tolist()))  # D2: first occurrence, in order
        assert seg.tolist() == want


def test_score_perfect_and_partial_windows():
    tr = wl.make_T(n_iter=2)
    norm = sweep_f2.normalised(tr, 1)
    p, r, _ = sweep_f2.score(norm, *_windows(norm, 1), 1, tr.K)
    assert (p, r) == (1.0, 1.0)
    # a window missing its first 8 blocks: precision stays 1, recall drops by 8 per query
    pairs, rng = _windows(norm, 1, drop=8)
    p, r, _ = sweep_f2.score(norm, pairs, rng, 1, tr.K)
    true = sum(np.unique(np.concatenate(norm[k:k + 2])).size for k in range(tr.K))
    assert p == 1.0 and r == pytest.approx((true - 8 * tr.K) / true)
    # empty windows score 0 / 0 without dividing by zero
    p, r, w = sweep_f2.score(norm, np.zeros(0, np.uint32), np.zeros((tr.K, 2), np.int64), 1, tr.K)
    assert (p, r, w) == (0.0, 0.0, 0.0)


@pytest.mark.gpu
@pytest.mark.parametrize("name,N", [("Config0", 1), ("Config9", 4), ("Config11", 2)])
def test_sweep_windows_match_oracle_on_T(name, N):
    """The sweep's engine path (record/build of iterations 0..i-1, then the
    transition windows of iteration i through the C-ABI) emits the oracle's
    windows, so its precision/recall are the oracle's."""
    import torch
    import oracle as orc
    from gpu_helpers import transition_queries
    A, S, R = sweep_f2.TABLE6[name]
    tr = wl.make_T(n_iter=3, dup_ppm=200_000)
    pairs_g, rng_g, _, n_exec, _ = sweep_f2.run(tr, (A, S, R), N, 2, torch.device("cuda", 0))
    o = orc.Oracle(R=R, A=A, S=S, N=N, W=tr.W, C=tr.C)
    ex = []
    for i in range(3):
        ex += [int(x) for x in o.record_faults(*tr.iteration(i))]
        if i < 2:
            o.build_tables()
    off, pairs_o, _, _ = o.predict(transition_queries(ex, 2 * tr.K, tr.K, N))
    assert n_exec == o.num_exec
    for k in range(tr.K):
        assert pairs_g[int(rng_g[k, 0]):int(rng_g[k, 1])].tolist() == \
            pairs_o[int(off[k]):int(off[k + 1]), 0].tolist(), (name, N, k)
    norm = sweep_f2.normalised(tr, 2)
    rng_o = np.stack([off[:-1], off[1:]], axis=1).astype(np.int64)
    assert sweep_f2.score(norm, pairs_g, rng_g, N, tr.K) == sweep_f2.score(norm, pairs_o[:, 0], rng_o, N, tr.K)
