"""Host-side cost of one e2e step (CPU time per C-ABI call, no synchronisation)
on the G workload:  python tools/host_overhead.py"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import workloads as wl
from paper_conf_asplos_jungkl23_b200 import Engine, binding as B

tr = wl.make("G", n_iter=8, seed=3)
K = tr.K
dev = torch.device("cuda", 0)
eng = Engine(num_rows=2048, assoc=2, num_succs=4, degree_n=32, max_blocks=tr.W, max_exec_ids=8192, hbm_frames=tr.C,
             device=0, corr_capacity=1 << 16, max_batch_faults=1 << 20, max_batch_launches=K * 2)
keep = []
hh, ho, hf = [], [], []
for i in range(8):
    h, off, f = tr.iteration(i)
    th = torch.from_numpy(h.view(np.int64)).pin_memory()
    to = torch.from_numpy(off.view(np.int64)).pin_memory()
    tf = torch.from_numpy(f.view(np.int32)).pin_memory()
    keep.append((th, to, tf))
    hh.append(th.numpy().view(np.uint64)); ho.append(to.numpy().view(np.uint64)); hf.append(tf.numpy().view(np.uint32))
exec_all = torch.full((8 * K + 3,), -1, dtype=torch.int32, device=dev)
qbuf = torch.empty((K, 6), dtype=torch.int32, device=dev)
cap = 40 << 20
pairs = torch.empty((cap, 2), dtype=torch.int32, device=dev)
wb = torch.empty(cap, dtype=torch.int32, device=dev)
inv = torch.empty(cap, dtype=torch.int32, device=dev)
rng = torch.empty((K, 2), dtype=torch.int64, device=dev)
ko = torch.empty((K, 34), dtype=torch.int32, device=dev)
ch = torch.empty((K, 33), dtype=torch.int32, device=dev)
srng = torch.empty((K, 4), dtype=torch.int64, device=dev)
np_ = torch.zeros(1, dtype=torch.int64, device=dev)
ns = torch.zeros(1, dtype=torch.int64, device=dev)
snaps = [torch.from_numpy(tr.snap_blk[i][: int(tr.snap_cnt[i])].view(np.int32)).to(dev) for i in range(8)]
eng.mark_inactive(torch.from_numpy(tr.inactive_blocks.view(np.int32)).to(dev), True)
rows = []
for i in range(8):
    eng.load_residency(snaps[i])
    torch.cuda.synchronize()
    t = [time.perf_counter()]
    eng.record_faults(hh[i], ho[i], hf[i], exec_all[3 + i * K: 3 + (i + 1) * K]); t.append(time.perf_counter())
    if i >= 1:
        eng.make_queries(exec_all[i * K: 3 + (i + 1) * K], 3, 32, out=qbuf); t.append(time.perf_counter())
        eng.predict_select(qbuf, cap, cap, pairs=pairs, rng=rng, kern_off=ko, chain=ch, needed=np_, wb=wb, inv=inv,
                           sel_rng=srng, sel_needed=ns); t.append(time.perf_counter())
    eng.build_tables(); t.append(time.perf_counter())
    torch.cuda.synchronize(); t.append(time.perf_counter())
    if i >= 1:
        rows.append(np.diff(np.array(t)) * 1e6)
r = np.median(np.array(rows[1:]), axis=0)
print("host us per call (median): record %.1f | make_queries %.1f | predict_select %.1f | build %.1f | "
      "wait for GPU %.1f | total %.1f" % (r[0], r[1], r[2], r[3], r[4], r.sum()))

# where does record_faults(host) go?  device-pointer record, plain torch H2D copies
dh = [torch.from_numpy(hh[1].view(np.int64)).to(dev), torch.from_numpy(ho[1].view(np.int64)).to(dev),
      torch.from_numpy(hf[1].view(np.int32)).to(dev)]
for name, fn in (
        ("record(device ptrs)", lambda: eng.record_faults(dh[0], dh[1], dh[2])),
        ("record(host ptrs)", lambda: eng.record_faults(hh[1], ho[1], hf[1])),
        ("torch H2D copies of the same pinned arrays", lambda: [d.copy_(h, non_blocking=True) for d, h in zip(dh, keep[1])]),
        ("is_pinned", lambda: [k.is_pinned() for k in keep[1]])):
    ts = []
    for r in range(5):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        out = fn()
        ts.append((time.perf_counter() - t0) * 1e6)
        eng.build_tables() if name.startswith("record") else None
    torch.cuda.synchronize()
    print("%-45s host us: %s %s" % (name, " ".join("%.1f" % x for x in ts), out if name == "is_pinned" else ""))
