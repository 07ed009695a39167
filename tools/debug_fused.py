"""GPU debug: G state after 3 iterations; fused predict+select vs oracle per
query, with the unfused GPU select for comparison."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import workloads as wl
from gpu_helpers import *

tr = wl.make("G", n_iter=3)
eng, o = make_pair(W=tr.W, C=tr.C, N=32, Emax=8192)
ex_all = []
for i in range(tr.n_iter):
    h, off, f = tr.iteration(i)
    exo, exg = record_both(eng, o, h, off, f)
    ex_all += [int(x) for x in exo]
    build_both(eng, o)
rng = np.random.default_rng(11)
pick = np.sort(rng.choice(np.arange(2 * tr.K, 3 * tr.K), 64, replace=False))
allq = transition_queries(ex_all, 0, len(ex_all), 32)[pick]
snap = tr.snap_blk[2][: int(tr.snap_cnt[2])]
o.load_residency(snap); eng.load_residency(dev(snap))
o.mark_inactive(tr.inactive_blocks, True); eng.mark_inactive(dev(tr.inactive_blocks), True)
MODE = os.environ.get("MODE", "plain")
if MODE == "test":
    ro, rg, (gp0, grng0, qd0) = predict_both(eng, o, allq)
    select_both(eng, o, gp0, grng0, qd0, allq, ro)
q = np.ascontiguousarray(allq, dtype=np.uint32).reshape(-1, 6)
off, pairs, ko, ch = o.predict(q)
wo, wb, io, iv = o.select(off, pairs, q[:, 4])
qd = dev(q.reshape(-1)).reshape(-1, 6)
cap = int(off[-1]) + 16
if MODE == "test":
    while True:
        out = eng.predict_select(qd, cap, sel_cap=cap)
        try:
            eng.sync()
            break
        except B.EngineError as e:
            print("retry", e, e.needed, cap)
            cap = int(e.needed)
else:
    out = eng.predict_select(qd, 2 * cap, sel_cap=2 * cap)
    eng.sync()
ctr = eng.read_counters(reset=True)
gp, grng, gko, gch, _, gwb, ginv, gsr, _ = out
gp = B.u32(gp).reshape(-1, 2); grng = B.u64(grng).reshape(-1, 2)
gwb, ginv, r = B.u32(gwb), B.u32(ginv), B.u64(gsr).reshape(-1, 4)
d = orc.parse_dump(o.dump(orc.WALK), orc.WALK, o.num_exec, 2048, 2, 4)
wl_ = np.array([len(w) for w in d["walk"]])
bad = 0
for i in range(len(q)):
    kern = [e for e in ch[i] if e != NONE]
    seen, U = set(), 0
    for e in kern:
        if e not in seen:
            seen.add(e); U += wl_[e]
    n = int(off[i + 1] - off[i])
    ew, ei = wb[int(wo[i]):int(wo[i + 1])], iv[int(io[i]):int(io[i + 1])]
    aw, ai = gwb[int(r[i, 0]):int(r[i, 1])], ginv[int(r[i, 2]):int(r[i, 3])]
    okp = np.array_equal(pairs[int(off[i]):int(off[i + 1])], gp[int(grng[i, 0]):int(grng[i, 1])])
    oks = np.array_equal(ew, aw) and np.array_equal(ei, ai)
    if not (okp and oks):
        bad += 1
        # first differing position
        fd = None
        if len(ei) and len(ai):
            m = min(len(ei), len(ai)); dd = np.nonzero(ei[:m] != ai[:m])[0]
            fd = int(dd[0]) if len(dd) else m
        print("q%d dup=%s U=%d n=%d pairs_ok=%s wb %d/%d inv %d/%d first_inv_diff=%s" % (
            i, U != n, U, n, okp, len(aw), len(ew), len(ai), len(ei), fd))
print("bad", bad, "of", len(q))
