"""sensitivity sweeps over the Table 6 geometries
(Config0-12, Fig. 12) and the prefetch degree N (Fig. 11,
P:L463-465), run through the CUDA engine (C-ABI) on a B- or G-shaped trace.

Open-loop metrics (the closed loop is §8(f) row 1):
  * precision / recall of each launch's transition window (launch k from its
    Start plus the next <= N predicted kernels, a7) against the normalised
    faults of launches k..k+N of the SAME iteration, with the tables built from
    the iterations before it (the order bench.py times: predict(i) reads
    build(i-1));
  * table bytes, the Table 4 analogue: exec IDs with a block
    table x R x A x (1+S) x 4 B, plus the correlation table records x 24 B;
  * mean window length (pairs per query) and predict time per launch.

  python tools/sweep_f2.py [--workload B] [--iters 3] [--out gpurun_out/f2.json]
"""
import argparse
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

TABLE6 = {  # name: (assoc, num_succs, num_rows)
    "Config0": (2, 4, 128), "Config1": (2, 8, 128), "Config2": (4, 4, 128), "Config3": (2, 4, 512),
    "Config4": (2, 8, 512), "Config5": (4, 4, 512), "Config6": (2, 4, 1024), "Config7": (2, 8, 1024),
    "Config8": (4, 4, 1024), "Config9": (2, 4, 2048), "Config10": (2, 8, 2048), "Config11": (4, 4, 2048),
    "Config12": (2, 4, 4096),
}


def normalised(tr, it):
    """Per launch of iteration `it`: first occurrences of its fault blocks (D2)."""
    h, off, f = tr.iteration(it)
    out = []
    for k in range(len(off) - 1):
        seg = f[int(off[k]) - int(off[0]): int(off[k + 1]) - int(off[0])]
        _, first = np.unique(seg, return_index=True)
        out.append(seg[np.sort(first)])
    return out


def run(tr, geo, N, it_eval, dev):
    import torch
    from paper_conf_asplos_jungkl23_b200 import Engine, binding as B
    A, S, R = geo
    K = tr.K
    eng = Engine(num_rows=R, assoc=A, num_succs=S, degree_n=N, max_blocks=tr.W, max_exec_ids=8192,
                 hbm_frames=tr.C, device=dev.index or 0, corr_capacity=1 << 16,
                 max_batch_faults=max(1 << 22,  # also sizes predict's hash pool (4x) for long N=64 windows
                                       int(max(tr.faults_in_iteration(i) for i in range(tr.n_iter)) * 1.2)),
                 max_batch_launches=max(2 * K, 4096))
    exec_all = torch.full((tr.n_iter * K + 3,), -1, dtype=torch.int32, device=dev)
    for i in range(it_eval):
        h, off, f = tr.iteration(i)
        eng.record_faults(B.as_u64_tensor(h, dev), B.as_u64_tensor(off, dev), B.as_u32_tensor(f, dev),
                          exec_all[3 + i * K: 3 + (i + 1) * K])
        eng.build_tables()
    h, off, f = tr.iteration(it_eval)
    eng.record_faults(B.as_u64_tensor(h, dev), B.as_u64_tensor(off, dev), B.as_u32_tensor(f, dev),
                      exec_all[3 + it_eval * K: 3 + (it_eval + 1) * K])
    q = eng.make_queries(exec_all[it_eval * K: 3 + (it_eval + 1) * K], 3, N)
    cap = 1 << 25  # pairs; an overflow is a sticky DUM_ECAPACITY, so size for the largest window sum
    pairs, rng, _, _, needed = eng.predict_prefetch(q, cap, want_kern_off=False, want_chain=False)
    eng.sync()
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    t0.record(torch.cuda.current_stream(dev))
    eng.predict_prefetch(q, cap, pairs=pairs, rng=rng, want_kern_off=False, want_chain=False)
    t1.record(torch.cuda.current_stream(dev))
    eng.sync()
    torch.cuda.synchronize(dev)
    ms = t0.elapsed_time(t1)
    st = eng.stats()
    pairs_h = pairs[:, 0].cpu().numpy().astype(np.uint32)
    rng_h = rng.cpu().numpy()
    eng.close()
    return pairs_h, rng_h, ms, int(st.num_exec), int(st.corr_records)


def score(norm, pairs_h, rng_h, N, K):
    tp = n_win = n_true = 0
    for k in range(K):
        win = np.unique(pairs_h[int(rng_h[k, 0]): int(rng_h[k, 1])])
        true = np.unique(np.concatenate(norm[k: min(K, k + N + 1)])) if norm[k:k + N + 1] else np.zeros(0, np.uint32)
        tp += np.intersect1d(win, true, assume_unique=True).size
        n_win += win.size
        n_true += true.size
    return tp / max(n_win, 1), tp / max(n_true, 1), n_win / K


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="B")
    ap.add_argument("--iters", type=int, default=3)
    ap.add_argument("--degrees", default="8,16,32,64")
    ap.add_argument("--configs", default=",".join(TABLE6))
    ap.add_argument("--out", default="gpurun_out/f2_sweep.json")
    a = ap.parse_args()
    import torch
    import workloads as wl
    dev = torch.device("cuda", 0)
    tr = wl.make(a.workload, n_iter=a.iters, seed={"G": 3, "B": 2, "T": 1}[a.workload])
    it_eval = a.iters - 1
    norm = normalised(tr, it_eval)
    rows = []
    for name in a.configs.split(","):
        A, S, R = TABLE6[name]
        for N in [int(x) for x in a.degrees.split(",")]:
            t = time.time()
            pairs_h, rng_h, ms, n_exec, n_corr = run(tr, (A, S, R), N, it_eval, dev)
            p, r, wlen = score(norm, pairs_h, rng_h, N, tr.K)
            row = {"config": name, "assoc": A, "num_succs": S, "num_rows": R, "N": N,
                   "precision": round(p, 4), "recall": round(r, 4), "pairs_per_query": round(wlen, 1),
                   "table_bytes": n_exec * R * A * (1 + S) * 4 + n_corr * 24, "exec_ids": n_exec,
                   "corr_records": n_corr, "predict_us_per_launch": round(1000 * ms / tr.K, 4)}
            rows.append(row)
            print(json.dumps(row), "(%.1fs)" % (time.time() - t), flush=True)
    os.makedirs(os.path.dirname(a.out) or ".", exist_ok=True)
    with open(a.out, "w") as fh:
        json.dump({"workload": a.workload, "iters": a.iters, "eval_iteration": it_eval, "rows": rows}, fh, indent=1)


if __name__ == "__main__":
    main()
