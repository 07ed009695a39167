"""Repeat a (record, build) of iteration 0 of a workload and compare the
engine's table state with the oracle's each time (intermittent-bug hunter)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np, torch
import workloads as wl, oracle as orc
from paper_conf_asplos_jungkl23_b200 import Engine, binding as B

cfg = sys.argv[1] if len(sys.argv) > 1 else "G"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 10
tr = wl.make(cfg, n_iter=1)
o = orc.Oracle(R=2048, A=2, S=4, N=32, W=tr.W, C=tr.C)
h, off, f = tr.iteration(0)
o.record_faults(h, off, f); o.build_tables()
what = orc.EXEC | orc.CORR | orc.BLK | orc.WALK | orc.HIST
ref = orc.parse_dump(o.dump(what), what, o.num_exec, 2048, 2, 4)
eng = Engine(max_blocks=tr.W, hbm_frames=tr.C, max_exec_ids=8192)
bad = 0
for r in range(reps):
    eng.reset()
    eng.record_faults(B.as_u64_tensor(h, "cuda"), B.as_u64_tensor(off, "cuda"), B.as_u32_tensor(f, "cuda"))
    eng.build_tables()
    try:
        eng.sync()
    except Exception as e:
        print("rep", r, "sync error", e)
    st = eng.stats()
    if st.guard_line:
        print("rep", r, "GUARD line", st.guard_line, "val", st.guard_val, "slow", st.slow_walks)
    got = orc.parse_dump(eng.dump_state(what), what, o.num_exec, 2048, 2, 4)
    for k in ("exec_hash", "start", "end"):
        if not np.array_equal(got[k], ref[k]):
            print("rep", r, "differs", k); bad += 1
    if got["corr"] != ref["corr"]:
        print("rep", r, "corr differs"); bad += 1
    for e in range(o.num_exec):
        if not np.array_equal(got["blk"][e], ref["blk"][e]):
            rows = np.nonzero((got["blk"][e] != ref["blk"][e]).any(axis=(1, 2)))[0]
            print("rep", r, "blk e=%d differing sets" % e, rows[:10], "gpu", got["blk"][e][rows[0]].tolist(),
                  "orc", ref["blk"][e][rows[0]].tolist()); bad += 1
            break
    for e in range(o.num_exec):
        if not np.array_equal(got["walk"][e], ref["walk"][e]):
            print("rep", r, "walk e=%d len gpu %d orc %d" % (e, len(got["walk"][e]), len(ref["walk"][e]))); bad += 1
            print("  gpu walk", got["walk"][e].tolist())
            print("  orc walk", ref["walk"][e].tolist())
            ks = [k for k in range(len(h)) if got["exec_hash"][e] == h[k]]
            for k in ks:
                L = f[int(off[k]):int(off[k + 1])].tolist()
                print("  launch", k, "faults", len(L), L[:40])
            rows = orc.table_rows(ref["blk"][e])
            print("  rows", {b: rows[b] for b in list(rows)[:40]})
            print("  start/end", got["start"][e], got["end"][e])
            break
    print("rep", r, "ok" if not bad else "BAD", flush=True)
    if bad:
        break
