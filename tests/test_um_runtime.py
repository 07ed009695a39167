"""Real-UM runtime: the library
exports its C-ABI (CPU); on the GPU, launch interposition gives equal hashes to
equal (kernel, arguments), prefetched UM blocks are read faster than faulting
ones, and one engine-predicted window, prefetched before an iteration of a
repeating kernel sequence over a managed arena, makes that iteration faster."""
from __future__ import annotations

import os
import re
import subprocess

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "include", "deepum_um.h")


def test_um_library_exports_every_declared_symbol():
    from paper_conf_asplos_jungkl23_b200 import build as bld
    so = bld.build_um()
    txt = re.sub(r"/\*.*?\*/", "", open(HDR).read(), flags=re.S)
    names = sorted(set(re.findall(r"\b(dum_um_[a-z_0-9]+)\s*\(", txt)))
    assert "dum_um_take" in names and "dum_um_prefetch" in names
    syms = subprocess.run(["nm", "-D", "--defined-only", so], capture_output=True, text=True).stdout
    missing = [n for n in names if not re.search(r"\bT %s\b" % n, syms)]
    assert not missing, missing


def _gpu():
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a GPU")
    torch.cuda.set_device(0)
    return torch


def _timed(torch, fn):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    fn()
    b.record()
    b.synchronize()
    return a.elapsed_time(b)


@pytest.mark.gpu
def test_um_interposition_hashes_and_prefetch():
    torch = _gpu()
    from paper_conf_asplos_jungkl23_b200.um_runtime import UmRuntime
    um = UmRuntime(96)
    A = torch.arange(0, 8, dtype=torch.int32, device="cuda")
    Bk = torch.arange(8, 16, dtype=torch.int32, device="cuda")
    C = torch.arange(32, 48, dtype=torch.int32, device="cuda")
    D = torch.arange(48, 64, dtype=torch.int32, device="cuda")
    W = torch.arange(80, 96, dtype=torch.int32, device="cuda")
    um.prefetch(np.arange(96), to_device=False)  # every block in host memory
    torch.cuda.synchronize()
    um.touch(W)  # module load / first launch outside the measurement
    torch.cuda.synchronize()
    um.intercept(True, faults=True)
    on, why = um.fault_source()
    um.touch(A)
    um.touch(Bk)
    um.touch(A)
    torch.cuda.synchronize()
    h, off, f = um.take()
    um.intercept(False)
    assert len(h) == 3 and h[0] == h[2] and h[0] != h[1], (h, why)
    if on:  # CUPTI fault records: launch 0 faulted on A's blocks
        assert set(f[off[0]:off[1]].tolist()) <= set(range(0, 8)) and off[1] > off[0]
    else:
        assert "unavailable" in why and len(f) == 0
    # prefetched blocks are read faster than demand-faulted ones
    um.prefetch(np.arange(32, 48), to_device=True)
    torch.cuda.synchronize()
    t_pre = _timed(torch, lambda: um.touch(C))
    t_flt = _timed(torch, lambda: um.touch(D))
    print("UM fault source: %s; touch 16 blocks prefetched %.3f ms vs demand-faulted %.3f ms" % (why, t_pre, t_flt))
    assert t_pre * 2 < t_flt, (t_pre, t_flt)


@pytest.mark.gpu
def test_um_engine_predicted_prefetch_speeds_up_an_iteration():
    """Four kernels touching disjoint block sets, repeated: iteration 1 runs on
    demand faults and is recorded (interposed hashes; faults = each launch's
    accesses when CUPTI UM records are unavailable); after build_tables, the
    engine's window for the first kernel (N = 3) is prefetched and iteration 2
    runs faster.  Every block is pushed back to host memory before each
    iteration."""
    torch = _gpu()
    from paper_conf_asplos_jungkl23_b200 import Engine, binding as B
    from paper_conf_asplos_jungkl23_b200.um_runtime import UmRuntime
    nb = 128
    um = UmRuntime(nb)
    sets = [np.arange(32 * k, 32 * k + 24, dtype=np.uint32) for k in range(4)]
    devs = [torch.from_numpy(s.view(np.int32)).cuda() for s in sets]
    warm = torch.arange(120, 128, dtype=torch.int32, device="cuda")
    um.prefetch(np.arange(nb), to_device=False)
    torch.cuda.synchronize()
    um.touch(warm)
    torch.cuda.synchronize()
    eng = Engine(num_rows=256, assoc=2, num_succs=4, degree_n=3, max_blocks=nb, max_exec_ids=64, hbm_frames=nb)

    def iteration(record: bool):
        um.prefetch(np.arange(nb), to_device=False)
        torch.cuda.synchronize()
        if record:
            um.intercept(True, faults=True)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for k in range(4):
            um.touch(devs[k])
            if record and not um.fault_source()[0]:
                um.add_faults(sets[k])  # the launch's accesses stand in for its fault records
        b.record()
        b.synchronize()
        return a.elapsed_time(b)

    t1 = iteration(record=True)
    h, off, f = um.take()
    um.intercept(False)
    assert len(h) == 4
    ex = torch.empty(4, dtype=torch.int32, device="cuda")
    eng.record_faults(B.as_u64_tensor(h, "cuda"), B.as_u64_tensor(off, "cuda"), B.as_u32_tensor(f, "cuda"), ex)
    eng.build_tables()
    eng.sync()
    e0 = int(B.u32(ex)[0])
    q = torch.tensor([[e0, -1, -1, -1, -1, 3]], dtype=torch.int32, device="cuda")
    pairs, rng, ko, ch, need = eng.predict_prefetch(q, 4096)
    eng.sync()
    r = B.u64(rng).reshape(-1, 2)[0]
    window = B.u32(pairs).reshape(-1, 2)[int(r[0]):int(r[1]), 0]
    assert set(window.tolist()) == set(np.concatenate(sets).tolist())
    t_naive = iteration(record=False)  # demand faults again, for a like-for-like baseline
    um.prefetch(np.arange(nb), to_device=False)
    um.prefetch(np.sort(window), to_device=True)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for k in range(4):
        um.touch(devs[k])
    b.record()
    b.synchronize()
    t2 = a.elapsed_time(b)
    print("UM iteration (4 kernels, 96 blocks): recorded %.3f ms, demand faults %.3f ms, engine-prefetched %.3f ms"
          % (t1, t_naive, t2))
    assert t2 * 2 < t_naive, (t1, t_naive, t2)
