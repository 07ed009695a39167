"""a9 on the GPU: batched 2 MiB block migration between pinned host memory and
HBM (PAPER.md L124 steps (4)-(7), L158, L285), checked against the oracle's
bookkeeping (frames, LRM order) and against closed-form content checksums
(SURVEY.md Sec. 8c a9 pin: host block b holds u64 words
splitmix64(seed ^ (b << 20 | w)); checksum = sum_w word_w * (2w + 1) mod 2^64)."""
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
from gpu_helpers import dev  # noqa: E402
from paper_conf_asplos_jungkl23_b200 import Engine, binding as B  # noqa: E402

BLOCK = 2 << 20
WORDS = BLOCK // 8
SEED = 4


def splitmix64_np(x: np.ndarray) -> np.ndarray:
    z = x + np.uint64(0x9E3779B97F4A7C15)
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def block_words(b: int) -> np.ndarray:
    w = np.arange(WORDS, dtype=np.uint64)
    return splitmix64_np(np.uint64(SEED) ^ ((np.uint64(b) << np.uint64(20)) | w))


_WEIGHT = (2 * np.arange(WORDS, dtype=np.uint64) + np.uint64(1))


def expected_sum(b: int) -> int:
    with np.errstate(over="ignore"):
        return int(np.sum(block_words(b) * _WEIGHT, dtype=np.uint64))


def make_arena(W: int):
    host = torch.empty(W * BLOCK, dtype=torch.uint8).pin_memory()
    hv = host.numpy().view(np.uint64).reshape(W, WORDS)
    with np.errstate(over="ignore"):
        for b in range(W):
            hv[b] = block_words(b)
    return host


@pytest.fixture(scope="module")
def arena_T():
    return make_arena(256)


def res_state(x):
    return orc.parse_dump(x, orc.RES, 0, 1, 1, 1)


@pytest.mark.parametrize("method", [1, 2])
def test_migration_ops_match_oracle_and_checksums(arena_T, method):
    W, C = 256, 64
    pool = torch.zeros(C * BLOCK, dtype=torch.uint8, device="cuda")
    eng = Engine(max_blocks=W, hbm_frames=C, max_exec_ids=16, host_arena=arena_T, frame_pool=pool)
    o = orc.Oracle(R=16, A=1, S=1, N=1, W=W, C=C)
    rng = np.random.default_rng(7 + method)
    exp = {b: expected_sum(b) for b in range(W)}

    def check():
        eng.sync()
        a, b = eng.dump_state(orc.RES), o.dump(orc.RES)
        assert a == b
        bof = res_state(a)["block_of_frame"]
        frames = [f for f in range(C) if bof[f] != orc.NONE]
        if frames:
            cs = B.u64(eng.block_checksums(0, dev(np.array(frames, np.uint32))))
            assert [int(x) for x in cs] == [exp[int(bof[f])] for f in frames]

    def both(d, blocks=None, dst=None):
        rc = o.migrate(d, blocks, dst)
        assert rc == 0, rc
        eng.migrate_blocks(d, None if blocks is None else dev(np.array(blocks, np.uint32)),
                           None if dst is None else dev(np.array(dst, np.uint32)), method=method)
        check()

    perm = [int(x) for x in rng.permutation(W)]
    both(B.H2D, perm[:40])                         # scattered blocks -> frames 0..39
    both(B.D2H, perm[5:15])                        # write-back: holes at frames 5..14
    both(B.INVALIDATE, perm[30:33])
    both(B.H2D, perm[100:120])                     # refills the lowest free frames first (D21)
    both(B.D2D, None, None)                        # compaction: free frames become a tail
    res = res_state(o.dump(orc.RES))
    bof = res["block_of_frame"]
    n_res = int(np.sum(bof != orc.NONE))
    assert np.all(bof[:n_res] != orc.NONE) and np.all(bof[n_res:] == orc.NONE)
    lrm = [int(x) for x in res["lrm"]]
    free = [f for f in range(C) if bof[f] == orc.NONE]
    both(B.D2D, lrm[:3], free[-3:])                # explicit moves into free frames
    # D2H copies back exactly the bytes of the block (host side checksum)
    both(B.D2H, lrm[3:8])
    cs = B.u64(eng.block_checksums(1, dev(np.array(lrm[3:8], np.uint32))))
    assert [int(x) for x in cs] == [exp[b] for b in lrm[3:8]]
    # invalid requests move nothing and raise
    eng.migrate_blocks(B.H2D, dev(np.array([lrm[10], lrm[10]], np.uint32)), method=method)
    with pytest.raises(B.EngineError):
        eng.sync()
    eng.migrate_blocks(B.D2H, dev(np.array([perm[200]], np.uint32)), method=method)
    with pytest.raises(B.EngineError):
        eng.sync()
    check()


class GpuLoop(il.LoopEngine):
    """Adapter: the T closed loop through the C-ABI with real bytes."""

    def __init__(self, tr, N, host, method=1):
        self.pool = torch.zeros(tr.C * BLOCK, dtype=torch.uint8, device="cuda")
        self.eng = Engine(num_rows=2048, assoc=2, num_succs=4, degree_n=max(N, 1), max_blocks=tr.W,
                          hbm_frames=tr.C, max_exec_ids=64, host_arena=host, frame_pool=self.pool)
        self.method = method

    def record(self, h, faults):
        out = torch.empty(1, dtype=torch.int32, device="cuda")
        self.eng.record_faults(np.array([h], np.uint64), np.array([0, len(faults)], np.uint64),
                               np.array(faults, np.uint32), out)
        return int(B.u32(out)[0])

    def build(self):
        self.eng.build_tables()

    def predict1(self, q):
        qd = dev(np.array(q, np.uint32)).reshape(1, 6)
        pairs, rng, _, _, _ = self.eng.predict_prefetch(qd, 4096)
        self.eng.sync()
        r = B.u64(rng)
        self._last = (pairs, rng, qd)
        p = B.u32(pairs).reshape(-1, 2)
        return [int(b) for b in p[int(r[0, 0]):int(r[0, 1]), 0]]

    def select1(self, blocks, anchor):
        pairs, rng, qd = self._last
        wb, inv, r, _ = self.eng.select_evictions(rng, pairs.reshape(-1), qd, 4096)
        self.eng.sync()
        r = B.u64(r)[0]
        return ([int(x) for x in B.u32(wb)[int(r[0]):int(r[1])]],
                [int(x) for x in B.u32(inv)[int(r[2]):int(r[3])]])

    def migrate(self, d, blocks):
        self.eng.migrate_blocks(d, dev(np.array(blocks, np.uint32)), method=self.method)
        self.eng.sync()

    def resident(self):
        return [int(x) for x in res_state(self.eng.dump_state(orc.RES))["lrm"]]

    def free(self):
        return int(self.eng.stats().free_frames)

    def snapshot(self):
        return self.eng.dump_state(orc.RES)


def _golden_loop_rows():
    import test_oracle_pins as pins
    return {r[0]: r for r in pins._loop_rows()}


@pytest.mark.parametrize("N", [0, 1, 2, 32])
def test_T_integration_loop_gpu_matches_oracle(arena_T, N):
    """All five calls in the closed loop with real bytes:
    residency and LRM order equal the oracle's after every launch; the fault /
    H2D / D2H totals equal the survey's independent derivation; every resident
    frame holds the right bytes at the end."""
    tr = wl.make_T()
    g = GpuLoop(tr, N, arena_T, method=1 if N % 2 == 0 else 2)
    o = il.OracleLoop(tr, N)
    snaps = []

    def check(k, eng):
        snaps.append(eng.snapshot())

    rg = il.run_loop(g, tr, N, check=check)
    osnaps = []
    ro = il.run_loop(o, tr, N, check=lambda k, e: osnaps.append(e.snapshot()))
    assert rg == ro
    assert snaps == osnaps
    n, faults, h2d, d2h = _golden_loop_rows()[N]
    assert rg["faults_per_iter"] == faults and rg["h2d"] == h2d and rg["d2h"] == d2h
    bof = res_state(snaps[-1])["block_of_frame"]
    frames = [f for f in range(tr.C) if bof[f] != orc.NONE]
    cs = B.u64(g.eng.block_checksums(0, dev(np.array(frames, np.uint32))))
    assert [int(x) for x in cs] == [expected_sum(int(bof[f])) for f in frames]


def test_migration_sweep_sizes():
    """M config shape: batches of 1..256 blocks, contiguous
    and permuted, both directions, bytes verified."""
    W = C = 256
    host = torch.empty(W * BLOCK, dtype=torch.uint8).pin_memory()
    hv = host.view(torch.int64)
    hv.copy_(torch.arange(hv.numel(), dtype=torch.int64))
    pool = torch.zeros(C * BLOCK, dtype=torch.uint8, device="cuda")
    eng = Engine(max_blocks=W, hbm_frames=C, max_exec_ids=16, host_arena=host, frame_pool=pool)
    rng = np.random.default_rng(3)
    for n in (1, 2, 4, 16, 64, 256):
        for order in ("contig", "perm"):
            blocks = np.arange(n, dtype=np.uint32) if order == "contig" else rng.permutation(W)[:n].astype(np.uint32)
            eng.load_residency(dev(np.zeros(0, np.uint32)))
            eng.migrate_blocks(B.H2D, dev(blocks))
            eng.sync()
            pv = pool.view(torch.int64).view(C, -1)
            for i in (0, n - 1):
                assert torch.equal(pv[i].cpu(), hv.view(W, -1)[int(blocks[i])])
            # D2H into a zeroed host copy region: clear, copy back, compare
            saved = hv.view(W, -1)[torch.from_numpy(blocks.astype(np.int64))].clone()
            hv.view(W, -1)[torch.from_numpy(blocks.astype(np.int64))] = 0
            eng.migrate_blocks(B.D2H, dev(blocks))
            eng.sync()
            assert torch.equal(hv.view(W, -1)[torch.from_numpy(blocks.astype(np.int64))], saved)
