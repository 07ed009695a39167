"""Experiment (EXP_TRACE builds only): per-item timeline of k_window_fast on G.
   python tools/exp_trace.py out.json"""
import ctypes
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as wl  # noqa: E402
from paper_conf_asplos_jungkl23_b200 import Engine, binding as B  # noqa: E402

dev = torch.device("cuda", 0)
tr = wl.make("G", n_iter=5, seed=3)
K, N = tr.K, 32
eng = Engine(num_rows=2048, assoc=2, num_succs=4, degree_n=N, max_blocks=tr.W, max_exec_ids=8192,
             hbm_frames=tr.C, device=0, corr_capacity=1 << 16,
             max_batch_faults=1 << 20, max_batch_launches=4096)
eng.mark_inactive(B.as_u32_tensor(tr.inactive_blocks, dev), True)
outs = {}
cap = 24 << 20
L = B.load_library()
L.dum_exp_trace.restype = ctypes.c_int
L.dum_exp_trace.argtypes = [ctypes.c_void_p, ctypes.c_ulonglong, ctypes.c_int]
buf = np.zeros(4 * 4096 + 8 * 65536, dtype=np.uint64)
for i in range(5):
    h, off, f = tr.iteration(i)
    eng.load_residency(B.as_u32_tensor(tr.snap_blk[i][: int(tr.snap_cnt[i])], dev))
    if i == 4:
        torch.cuda.synchronize()
        L.dum_exp_trace(None, 0, 1)
        torch.cuda.synchronize()
    eng.step(B.as_u64_tensor(h, dev), B.as_u64_tensor(off, dev), B.as_u32_tensor(f, dev), cap, cap, outs)
    eng.sync()
L.dum_exp_trace(buf.ctypes.data, buf.nbytes, 0)
cta = buf[:4 * 4096].reshape(4096, 4)
n_cta = int((cta[:, 0] > 0).sum())
t0 = int(cta[:n_cta, 0].min())
rel = lambda x: (x.astype(np.int64) - t0) / 1000.0  # noqa: E731
p1 = buf[4 * 4096:].reshape(-1, 8)
p1 = p1[p1[:, 0] > 0]
pc = lambda x: np.percentile(x, [10, 50, 90, 100]).round(2).tolist() if len(x) else []  # noqa: E731
res = {"ctas": n_cta,
       "cta_start_us": [float(rel(cta[:n_cta, 0]).min()), float(rel(cta[:n_cta, 0]).max())],
       "sel_end_us": pc(rel(cta[:n_cta, 1])), "copy_end_us": pc(rel(cta[:n_cta, 2])), "end_us": pc(rel(cta[:n_cta, 3])),
       "items": len(p1), "item_start_us": pc(rel(p1[:, 0])), "item_dur_us": pc((p1[:, 1] - p1[:, 0]) / 1000.0)}
st = p1[p1[:, 2] > 0]
if len(st):
    res["to_roff_us"] = pc((st[:, 2] - st[:, 0]) / 1000.0)
    res["to_marks_us"] = pc((st[:, 3] - st[:, 2]) / 1000.0)
    res["tma_issue_us"] = pc((st[:, 5] - st[:, 2]) / 1000.0)
    res["to_scan_us"] = pc((st[:, 4] - st[:, 3]) / 1000.0)
    res["emit_us"] = pc((st[:, 1] - st[:, 4]) / 1000.0)
    res["staged_items"] = len(st)
    R = (st[:, 6] >> 32).astype(np.int64)
    nw = (st[:, 6] & 0xFFFFFFFF).astype(np.int64)
    nk = (st[:, 7] >> 32).astype(np.int64)
    need = (st[:, 7] & 0xFFFFFFFF).astype(np.int64)
    res["R"] = pc(R)
    res["nw"] = pc(nw)
    res["nk"] = pc(nk)
    res["need"] = pc(need)
    top = np.argsort(-(st[:, 3] - st[:, 2]).astype(np.int64))[:8]
    res["slowest_marks"] = [[float((st[k, 3] - st[k, 2]) / 1000.0), int(R[k]), int(nw[k]), int(nk[k]), int(need[k])]
                            for k in top]
json.dump(res, open(sys.argv[1], "w"), indent=1)
print(json.dumps(res, indent=1))
