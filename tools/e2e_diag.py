"""Host-side timeline of the e2e loop (bench.run_e2e's steps issued back to
back): host microseconds per call, median over steps.  python tools/e2e_diag.py"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import workloads as wl
from paper_conf_asplos_jungkl23_b200 import Engine

NI = 12
tr = wl.make("G", n_iter=NI, seed=3)
K = tr.K
dev = torch.device("cuda", 0)
eng = Engine(num_rows=2048, assoc=2, num_succs=4, degree_n=32, max_blocks=tr.W, max_exec_ids=8192, hbm_frames=tr.C,
             device=0, corr_capacity=1 << 16, max_batch_faults=1 << 20, max_batch_launches=K * 2)
hh, ho, hf, hs, keep = [], [], [], [], []
for i in range(NI):
    h, off, f = tr.iteration(i)
    th = torch.from_numpy(h.view(np.int64)).pin_memory()
    to = torch.from_numpy(off.view(np.int64)).pin_memory()
    tf = torch.from_numpy(f.view(np.int32)).pin_memory()
    ts = torch.from_numpy(np.ascontiguousarray(tr.snap_blk[i][: int(tr.snap_cnt[i])]).view(np.int32)).pin_memory()
    keep.append((th, to, tf))
    hh.append(th.numpy().view(np.uint64)); ho.append(to.numpy().view(np.uint64)); hf.append(tf.numpy().view(np.uint32))
    hs.append(ts)
exec_all = torch.full((NI * K + 3,), -1, dtype=torch.int32, device=dev)
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
snap_dev = torch.empty(tr.C, dtype=torch.int32, device=dev)
out_r = [torch.empty((K, 2), dtype=torch.int64).pin_memory() for _ in range(NI)]
out_s = [torch.empty((K, 4), dtype=torch.int64).pin_memory() for _ in range(NI)]
print("ptr kind (this library's runtime) of a pinned torch tensor:", eng.lib.dum_host_ptr_kind(keep[0][2].data_ptr()),
      "numpy view:", eng.lib.dum_host_ptr_kind(hf[0].ctypes.data))
eng.mark_inactive(torch.from_numpy(tr.inactive_blocks.view(np.int32)).to(dev), True)
names = ["snap_copy", "load_res", "record", "make_q", "predict_sel", "build", "d2h"]
rows, gpu = [], []
evs = []
stream = torch.cuda.current_stream(dev)
for i in range(NI):
    if i == 4:
        torch.cuda.synchronize()
        a = torch.cuda.Event(enable_timing=True); a.record(stream); t_start = time.perf_counter()
    t = [time.perf_counter()]
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(8)]
    ev[0].record(stream)
    n = hs[i].numel()
    snap_dev[:n].copy_(hs[i], non_blocking=True); t.append(time.perf_counter()); ev[1].record(stream)
    eng.load_residency(snap_dev[:n]); t.append(time.perf_counter()); ev[2].record(stream)
    eng.record_faults(hh[i], ho[i], hf[i], exec_all[3 + i * K: 3 + (i + 1) * K]); t.append(time.perf_counter()); ev[3].record(stream)
    if i >= 1:
        eng.make_queries(exec_all[i * K: 3 + (i + 1) * K], 3, 32, out=qbuf); t.append(time.perf_counter()); ev[4].record(stream)
        eng.predict_select(qbuf, cap, cap, pairs=pairs, rng=rng, kern_off=ko, chain=ch, needed=np_, wb=wb, inv=inv,
                           sel_rng=srng, sel_needed=ns); t.append(time.perf_counter()); ev[5].record(stream)
    else:
        t += [t[-1], t[-1]]; ev[4].record(stream); ev[5].record(stream)
    eng.build_tables(); t.append(time.perf_counter()); ev[6].record(stream)
    out_r[i].copy_(rng, non_blocking=True); out_s[i].copy_(srng, non_blocking=True); t.append(time.perf_counter()); ev[7].record(stream)
    if i >= 4:
        evs.append(ev)
    if i >= 4:
        rows.append(np.diff(np.array(t)) * 1e6)
b = torch.cuda.Event(enable_timing=True); b.record(stream); t_end = time.perf_counter(); b.synchronize()
r = np.median(np.array(rows), axis=0)
g = np.median(np.array([[e[k].elapsed_time(e[k + 1]) * 1000 for k in range(7)] for e in evs]), axis=0)
print("GPU us per call (median, events between calls): " + " | ".join("%s %.1f" % (nm, x) for nm, x in zip(names, g)) + " | sum %.1f" % g.sum())
print("host us per call (median): " + " | ".join("%s %.1f" % (nm, x) for nm, x in zip(names, r)) + " | sum %.1f" % r.sum())
print("steps %d: host issue %.1f us/step, GPU %.1f us/step" % (NI - 4, (t_end - t_start) * 1e6 / (NI - 4),
                                                               a.elapsed_time(b) * 1000 / (NI - 4)))

# H2D of the same record inputs with torch copies vs the DUM_HOST_PTRS memcpys
dbuf = [torch.empty(keep[0][k].numel() * 2, dtype=keep[0][k].dtype, device=dev) for k in range(3)]
res = {"torch copies": [], "host-ptr record": [], "device-ptr record": []}
for i in range(4, NI):
    torch.cuda.synchronize()
    e0, e1, e2, e3 = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
    e0.record(stream)
    for k in range(3):
        dbuf[k][: keep[i][k].numel()].copy_(keep[i][k], non_blocking=True)
    e1.record(stream)
    eng.record_faults(dbuf[0][: keep[i][0].numel()], dbuf[1][: keep[i][1].numel()], dbuf[2][: keep[i][2].numel()])
    e2.record(stream)
    eng.build_tables()
    torch.cuda.synchronize()
    e3.record(stream)
    eng.record_faults(hh[i], ho[i], hf[i])
    e4 = torch.cuda.Event(enable_timing=True); e4.record(stream)
    eng.build_tables()
    torch.cuda.synchronize()
    res["torch copies"].append(e0.elapsed_time(e1) * 1000)
    res["device-ptr record"].append(e1.elapsed_time(e2) * 1000)
    res["host-ptr record"].append(e3.elapsed_time(e4) * 1000)
print("GPU us (median): " + " | ".join("%s %.1f" % (k, np.median(v)) for k, v in res.items()))
