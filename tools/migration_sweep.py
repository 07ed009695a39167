#!/usr/bin/env python
"""Config M (BASELINE.json configs[3]): the migration sweep.

    python tools/migration_sweep.py [--max-blocks 4096] [--reps 20] [--warmup 5] [--out FILE]

2 MiB-block batches of n = 1, 2, 4, ..., 4096 blocks through dum_migrate_blocks
(PAPER.md L124 steps (4)-(7), L158) between a pinned host arena and an HBM
frame pool, for
  order:     contiguous blocks -> contiguous frames, and a random permutation
             of blocks (frames still assigned lowest-free-first, D21);
  direction: H2D, D2H, H2D || D2H concurrently (two engines on two streams,
             disjoint halves of the arena / pool, half of the SMs each for
             the copy kernels; method 2 synchronizes per call, so its pair
             runs one after the other), D2D compaction (HBM);
  method:    1 = SM copy kernel, 3 = TMA bulk copies, 2 = copy engines (one
             cudaMemcpyAsync per contiguous run).
Per point: W warm-up + R timed repetitions (CUDA events on the engine's
stream; the residency is reset outside the timed region), median and best.
Fractions are of the host-link peak measured here (cudaMemcpyAsync of 1 GiB
pinned, best of 10, per direction and concurrently) and, for D2D, of the HBM
peak in MEASURED_PEAKS.json (2 x 2 MiB moved per block).  After timing, the
bytes of sampled blocks are checked (untimed)."""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_asplos_jungkl23_b200 import Engine, binding as B  # noqa: E402

BLOCK = 2 << 20
METHODS = {1: "sm_copy", 3: "tma_bulk", 2: "copy_engine"}


def hostlink_peak(host, pool, stream, nbytes=1 << 30, reps=10):
    def best(fn):
        t = 1e9
        for _ in range(reps):
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            fn()
            b.record(stream)
            b.synchronize()
            t = min(t, a.elapsed_time(b) / 1e3)
        return t
    h2d = nbytes / best(lambda: pool[:nbytes].copy_(host[:nbytes], non_blocking=True)) / 1e9
    d2h = nbytes / best(lambda: host[:nbytes].copy_(pool[:nbytes], non_blocking=True)) / 1e9
    s2 = torch.cuda.Stream()

    def both():
        ev = torch.cuda.Event()
        ev.record(stream)
        s2.wait_event(ev)
        pool[:nbytes].copy_(host[:nbytes], non_blocking=True)
        with torch.cuda.stream(s2):
            host[nbytes:2 * nbytes].copy_(pool[nbytes:2 * nbytes], non_blocking=True)
        ev2 = torch.cuda.Event()
        ev2.record(s2)
        stream.wait_event(ev2)
    bidir = 2 * nbytes / best(both) / 1e9
    return {"h2d_gbs": h2d, "d2h_gbs": d2h, "bidir_gbs": bidir,
            "how": "cudaMemcpyAsync of 1 GiB pinned, best of %d, per direction; bidir = both at once" % reps}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--max-blocks", type=int, default=4096)
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--methods", default="1,3,2")
    ap.add_argument("--out", default="")
    args = ap.parse_args()
    dev = torch.device("cuda", 0)
    torch.cuda.set_device(dev)
    nmax = args.max_blocks
    t0 = time.time()
    host = torch.empty(nmax * BLOCK, dtype=torch.uint8).pin_memory()
    pool = torch.empty(nmax * BLOCK, dtype=torch.uint8, device=dev)
    hv = host.view(torch.int64)
    hv.copy_(torch.arange(hv.numel(), dtype=torch.int64))  # word w of the arena holds w
    stream = torch.cuda.current_stream(dev)
    peaks = hostlink_peak(host, pool, stream)
    hbm = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
        os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
    half = nmax // 2
    eng = Engine(max_blocks=nmax, hbm_frames=nmax, max_exec_ids=16, host_arena=host, frame_pool=pool)
    # the concurrent pair: engine A owns arena/pool [0, half), engine B [half, nmax)
    engA = Engine(max_blocks=half, hbm_frames=half, max_exec_ids=16, host_arena=host[: half * BLOCK],
                  frame_pool=pool[: half * BLOCK])
    engB = Engine(max_blocks=half, hbm_frames=half, max_exec_ids=16, host_arena=host[half * BLOCK:],
                  frame_pool=pool[half * BLOCK:])
    # the concurrent pair splits the SMs: each engine's copy kernels take half
    # (dum_set_copy_sms), so the write-back and the fetch run side by side
    nsm = torch.cuda.get_device_properties(dev).multi_processor_count
    engA.set_copy_sms(nsm // 2)
    engB.set_copy_sms(nsm - nsm // 2)
    sB = torch.cuda.Stream(device=dev)
    rng = np.random.default_rng(4)
    methods = [int(m) for m in args.methods.split(",")]
    sizes = [1 << k for k in range(0, 13) if (1 << k) <= nmax]
    out = {"host_link_peak": peaks, "hbm_peak_gbs": hbm, "reps": args.reps, "warmup": args.warmup,
           "block_bytes": BLOCK, "points": []}

    def timed(fn, setup):
        ts = []
        for r in range(args.warmup + args.reps):
            setup()
            torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            fn()
            b.record(stream)
            b.synchronize()
            if r >= args.warmup:
                ts.append(a.elapsed_time(b) / 1e3)
        return statistics.median(ts), min(ts)

    for order in ("contiguous", "permuted"):
        for n in sizes:
            blocks = np.arange(n, dtype=np.uint32) if order == "contiguous" else \
                rng.permutation(nmax)[:n].astype(np.uint32)
            bd = torch.from_numpy(blocks.view(np.int32)).to(dev)
            empty = torch.empty(0, dtype=torch.int32, device=dev)
            for m in methods:
                for d, dname in ((B.H2D, "h2d"), (B.D2H, "d2h")):
                    setup = (lambda: eng.load_residency(empty)) if d == B.H2D else (lambda: eng.load_residency(bd))
                    med, best = timed(lambda: eng.migrate_blocks(d, bd, method=m), setup)
                    eng.sync()
                    gbs_med, gbs_best = n * BLOCK / med / 1e9, n * BLOCK / best / 1e9
                    pk = peaks[dname + "_gbs"]
                    out["points"].append({"order": order, "n": n, "method": METHODS[m], "dir": dname,
                                          "median_s": med, "best_s": best, "gbs_median": gbs_med,
                                          "gbs_best": gbs_best, "frac_median": gbs_med / pk,
                                          "frac_best": gbs_best / pk})
                # H2D || D2H: engine A moves n/2 blocks in, engine B n/2 blocks out, concurrently
                if n >= 2:
                    k = n // 2
                    ba = torch.from_numpy((blocks[:k] % half).astype(np.uint32).view(np.int32)).to(dev)
                    ba = torch.unique(ba)
                    bb = torch.from_numpy(np.arange(k, dtype=np.uint32).view(np.int32)).to(dev)

                    def setup2():
                        engA.load_residency(empty)
                        engB.load_residency(bb)

                    def both():
                        ev = torch.cuda.Event()
                        ev.record(stream)
                        sB.wait_event(ev)
                        engA.migrate_blocks(B.H2D, ba, method=m)
                        with torch.cuda.stream(sB):
                            engB.migrate_blocks(B.D2H, bb, method=m)
                        ev2 = torch.cuda.Event()
                        ev2.record(sB)
                        stream.wait_event(ev2)
                    med, best = timed(both, setup2)
                    engA.sync()
                    engB.sync()
                    nb = ba.numel() + bb.numel()
                    out["points"].append({"order": order, "n": int(nb), "method": METHODS[m], "dir": "bidir",
                                          "median_s": med, "best_s": best, "gbs_median": nb * BLOCK / med / 1e9,
                                          "gbs_best": nb * BLOCK / best / 1e9,
                                          "frac_median": nb * BLOCK / med / 1e9 / peaks["bidir_gbs"],
                                          "frac_best": nb * BLOCK / best / 1e9 / peaks["bidir_gbs"]})
                # D2D compaction: n resident blocks spread over the top frames move into the lowest ones
                if n <= half:
                    keep = torch.from_numpy(np.arange(nmax, dtype=np.uint32).view(np.int32)).to(dev)
                    drop = torch.from_numpy(np.arange(n, dtype=np.uint32).view(np.int32)).to(dev)

                    def setup3():
                        eng.load_residency(keep)             # frame f holds block f
                        eng.migrate_blocks(B.INVALIDATE, drop)  # frames [0, n) free: n movers above

                    med, best = timed(lambda: eng.migrate_blocks(B.D2D, None, method=m), setup3)
                    eng.sync()
                    gbs_med, gbs_best = 2 * n * BLOCK / med / 1e9, 2 * n * BLOCK / best / 1e9
                    out["points"].append({"order": order, "n": n, "method": METHODS[m], "dir": "d2d_compaction",
                                          "median_s": med, "best_s": best, "gbs_median": gbs_med,
                                          "gbs_best": gbs_best, "frac_median": gbs_med / hbm,
                                          "frac_best": gbs_best / hbm})
        print("order %s done (%.0f s)" % (order, time.time() - t0), file=sys.stderr)
    # bytes check (untimed): H2D of a permuted batch with each method, compare frames with the arena
    checks = {}
    blocks = rng.permutation(nmax)[:64].astype(np.uint32)
    bd = torch.from_numpy(blocks.view(np.int32)).to(dev)
    for m in methods:
        eng.load_residency(torch.empty(0, dtype=torch.int32, device=dev))
        pool.zero_()
        eng.migrate_blocks(B.H2D, bd, method=m)
        eng.sync()
        ok = True
        for f, b in enumerate(blocks[:16]):
            ok &= bool(torch.equal(pool[f * BLOCK:(f + 1) * BLOCK].cpu(), host[int(b) * BLOCK:(int(b) + 1) * BLOCK]))
        checks[METHODS[m]] = ok
    out["bytes_verified"] = checks
    # summary: best method per direction at n = max, smallest n reaching 0.8 of the link
    summ = {}
    for dname in ("h2d", "d2h", "bidir", "d2d_compaction"):
        pts = [p for p in out["points"] if p["dir"] == dname and p["order"] == "contiguous"]
        if not pts:
            continue
        for m in set(p["method"] for p in pts):
            mp = sorted((p for p in pts if p["method"] == m), key=lambda p: p["n"])
            reach = [p["n"] for p in mp if p["frac_median"] >= 0.8]
            summ.setdefault(dname, {})[m] = {"n_max": mp[-1]["n"], "frac_median_at_max": mp[-1]["frac_median"],
                                             "gbs_median_at_max": mp[-1]["gbs_median"],
                                             "smallest_n_at_0.8": reach[0] if reach else None}
    out["summary"] = summ
    out["wall_s"] = time.time() - t0
    s = json.dumps(out)
    if args.out:
        open(args.out, "w").write(s + "\n")
    print(json.dumps(summ, indent=1))


if __name__ == "__main__":
    main()
