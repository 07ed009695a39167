"""SURVEY.md 8(f) row 1 on the GPU: dum_simulate, the closed loop of the
paper's runtime (demand faults first, table update,
chained prediction, pre-eviction L236-L243, invalidation L285, prefetch),
replayed launch by launch entirely in the library's kernels, against the
host-driven reference loop (tests/integration_loop.run_loop) over the CPU
oracle: per-launch fault / eviction / prefetch counts and the final residency
and table state must be identical.
  * T with real bytes (host arena + frame pool): the survey's closed-form
    totals (faults per iteration, H2D, D2H) and frame checksums.
  * B, metadata-only (720 GB of host memory would be needed for bytes): the
    first 1.5 iterations, every ablation of PAPER.md Fig. 10 (L457)."""
from __future__ import annotations

import numpy as np
import pytest
import torch

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)

import integration_loop as il  # noqa: E402
import oracle as orc  # noqa: E402
import workloads as wl  # noqa: E402
from gpu_helpers import ALL_TABLES, LIVE_ENGINES, dev  # noqa: E402
from paper_conf_asplos_jungkl23_b200 import Engine, binding as B  # noqa: E402

ALL = B.SIM_PREFETCH | B.SIM_PREEVICT | B.SIM_INVALIDATE


def _sim(eng, tr, N, flags, n_launch=None):
    n = tr.n_iter * tr.K if n_launch is None else n_launch
    h = dev(np.asarray(tr.launch_hash[:n], np.uint64), np.uint64)
    st = eng.simulate(h, np.asarray(tr.access_off, np.uint64), dev(tr.access_blk), max(N, 0),
                      flags if N >= 0 else 0)
    eng.sync()
    return B.u32(st).reshape(n, -1)


@pytest.mark.parametrize("N", [-1, 0, 1, 2, 32])
def test_T_closed_loop_matches_reference_and_closed_form(N):
    tr = wl.make_T()
    eng = Engine(num_rows=2048, assoc=2, num_succs=4, degree_n=max(N, 1), max_blocks=tr.W, max_exec_ids=64,
                 hbm_frames=tr.C)
    LIVE_ENGINES.append(eng)
    st = _sim(eng, tr, N, ALL)
    ref = il.OracleLoop(tr, N)
    rows = []
    out = il.run_loop(ref, tr, N, per_launch=rows)
    assert np.array_equal(st, np.array(rows, np.uint32)), "per-launch counts differ from the reference loop"
    K = tr.K
    per_iter = st[:, 0].reshape(tr.n_iter, K).sum(axis=1)
    assert list(per_iter) == list(out["faults_per_iter"])
    assert int(st[:, 0].sum() + st[:, 5].sum()) == out["h2d"]
    assert int(st[:, 1].sum() + st[:, 3].sum()) == out["d2h"]
    if N in (0, 1, 2, 32):  # the survey's independent derivation (SURVEY 8c "T integration loop")
        import test_oracle_pins as pins
        gold = {r[0]: r for r in pins._loop_rows()}[N]
        assert list(per_iter) == list(gold[1]) and out["h2d"] == gold[2] and out["d2h"] == gold[3]
    assert eng.dump_state(orc.RES) == ref.o.dump(orc.RES)
    assert eng.dump_state(ALL_TABLES) == ref.o.dump(ALL_TABLES)


@pytest.mark.parametrize("flags", [B.SIM_PREFETCH, B.SIM_PREFETCH | B.SIM_PREEVICT])
def test_T_closed_loop_ablations_match_reference(flags):
    """Fig. 10's intermediate configurations: prefetch only (the driver evicts
    least recently migrated blocks for the prefetch), + pre-eviction."""
    tr = wl.make_T()
    N = 2
    eng = Engine(num_rows=2048, assoc=2, num_succs=4, degree_n=N, max_blocks=tr.W, max_exec_ids=64, hbm_frames=tr.C)
    LIVE_ENGINES.append(eng)
    st = _sim(eng, tr, N, flags)
    ref = il.OracleLoop(tr, N)
    rows = []
    il.run_loop(ref, tr, N, per_launch=rows, preevict=bool(flags & B.SIM_PREEVICT))
    assert np.array_equal(st, np.array(rows, np.uint32))
    assert eng.dump_state(orc.RES) == ref.o.dump(orc.RES)


@pytest.mark.parametrize("flags", [0, B.SIM_PREFETCH, ALL])
def test_B_closed_loop_sample_matches_reference(flags):
    """BERT-large-shaped trace (configs[1]), 1.5 iterations, metadata-only."""
    tr = wl.make("B", n_iter=2)
    N = 32 if flags else -1
    n_launch = tr.K + tr.K // 2
    eng = Engine(num_rows=2048, assoc=2, num_succs=4, degree_n=32, max_blocks=tr.W, max_exec_ids=8192,
                 hbm_frames=tr.C, corr_capacity=1 << 16)
    LIVE_ENGINES.append(eng)
    inactive = set(int(b) for b in tr.inactive_blocks)
    eng.mark_inactive(dev(tr.inactive_blocks), True)
    st = _sim(eng, tr, N, flags, n_launch=n_launch)
    ref = il.OracleLoop(tr, N, inactive=inactive)
    rows = []
    il.run_loop(ref, tr, N, inactive=inactive, per_launch=rows, n_launch=n_launch,
                preevict=bool(flags & B.SIM_PREEVICT), invalidate=bool(flags & B.SIM_INVALIDATE))
    ref_rows = np.array(rows, np.uint32)
    bad = np.nonzero((st != ref_rows).any(axis=1))[0]
    assert len(bad) == 0, "launch %d: gpu %s ref %s" % (bad[0], st[bad[0]], ref_rows[bad[0]])
    assert eng.dump_state(orc.RES) == ref.o.dump(orc.RES)
