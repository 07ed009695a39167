"""Where the end-to-end step loses time (run under gpurun): bench.py's e2e loop
on G with its host-side pieces switched off one at a time.
    python tools/e2e_ablation.py [--steps 10]"""
import argparse
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import workloads as wl  # noqa: E402
from paper_conf_asplos_jungkl23_b200 import Engine, binding as B  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--steps", type=int, default=10)
ap.add_argument("--warmup", type=int, default=3)
args = ap.parse_args()
dev = torch.device("cuda", 0)
n_iter = 1 + args.warmup + args.steps
tr = wl.make("G", n_iter=n_iter, seed=3)
K = tr.K
eng = Engine(num_rows=2048, assoc=2, num_succs=4, degree_n=32, max_blocks=tr.W, max_exec_ids=8192, hbm_frames=tr.C,
             corr_capacity=1 << 16, max_batch_faults=max(1 << 20, int(max(tr.faults_in_iteration(i)
                                                                            for i in range(n_iter)) * 1.2)),
             max_batch_launches=max(K * 2, 4096))
stream = torch.cuda.current_stream(dev)
hh, ho, hf, hs, dh, do, df, ds = [], [], [], [], [], [], [], []
for i in range(n_iter):
    h, off, f = tr.iteration(i)
    th = torch.from_numpy(h.view(np.int64)).pin_memory()
    to = torch.from_numpy(off.view(np.int64)).pin_memory()
    tf = torch.from_numpy(f.view(np.int32)).pin_memory()
    hh.append((th, th.numpy().view(np.uint64)))
    ho.append((to, to.numpy().view(np.uint64)))
    hf.append((tf, tf.numpy().view(np.uint32)))
    sn = np.ascontiguousarray(tr.snap_blk[i][: int(tr.snap_cnt[i])])
    hs.append(torch.from_numpy(sn.view(np.int32)).pin_memory())
    dh.append(th.to(dev))
    do.append(to.to(dev))
    df.append(tf.to(dev))
    ds.append(hs[-1].to(dev))
cap = 24 << 20
res = {}
for mode in ["full", "counting_off", "one_copy_stream", "dev_inputs", "no_snap_upload", "no_d2h", "plain"]:
    host_in = mode not in ("dev_inputs", "plain")
    snap_up = mode not in ("no_snap_upload", "plain")
    d2h = mode not in ("no_d2h", "plain")
    eng.reset()
    eng.mark_inactive(B.as_u32_tensor(tr.inactive_blocks, dev), True)
    eng.set_step_graphs(True)
    eng.set_counting(mode != "counting_off")
    outs = {}
    snap_dev = [torch.empty(tr.C, dtype=torch.int32, device=dev) for _ in range(2)]
    out_r = [torch.empty((K, 2), dtype=torch.int64).pin_memory() for _ in range(args.steps)]
    out_s = [torch.empty((K, 4), dtype=torch.int64).pin_memory() for _ in range(args.steps)]
    cs = torch.cuda.Stream(device=dev)
    dstr = torch.cuda.Stream(device=dev) if mode != "one_copy_stream" else cs
    snap_used = [None, None]
    d2h_done = [None]

    def host_step(i, s=None):
        n = hs[i].numel()
        k = i & 1
        if snap_up:
            up = torch.cuda.Event()
            with torch.cuda.stream(cs):
                if snap_used[k] is not None:
                    cs.wait_event(snap_used[k])
                snap_dev[k][:n].copy_(hs[i], non_blocking=True)
                up.record(cs)
            stream.wait_event(up)
            eng.load_residency(snap_dev[k][:n])
            snap_used[k] = torch.cuda.Event()
            snap_used[k].record(stream)
        else:
            eng.load_residency(ds[i])
        if d2h and d2h_done[0] is not None:
            stream.wait_event(d2h_done[0])
        if host_in:
            eng.step(hh[i][1], ho[i][1], hf[i][1], cap, cap, outs)
        else:
            eng.step(dh[i], do[i], df[i], cap, cap, outs, ready=i > 1 + args.warmup)
        if d2h and s is not None:
            ev = torch.cuda.Event()
            ev.record(stream)
            with torch.cuda.stream(dstr):
                dstr.wait_event(ev)
                out_r[s].copy_(outs["rng"], non_blocking=True)
                out_s[s].copy_(outs["sel_rng"], non_blocking=True)
                d2h_done[0] = torch.cuda.Event()
                d2h_done[0].record(dstr)

    for i in range(0, 1 + args.warmup):
        host_step(i)
    eng.sync()
    torch.cuda.synchronize()
    a = torch.cuda.Event(enable_timing=True)
    b = torch.cuda.Event(enable_timing=True)
    a.record(stream)
    for s in range(args.steps):
        host_step(1 + args.warmup + s, s)
    if d2h_done[0] is not None:
        stream.wait_event(d2h_done[0])
    b.record(stream)
    b.synchronize()
    res[mode] = round(a.elapsed_time(b) / args.steps, 4)
    print(mode, res[mode], "ms/step", flush=True)
print(json.dumps(res))
