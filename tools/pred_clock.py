"""Summarise DUM_PRED_CLOCK dumps of k_predict (per-CTA globaltimer stamps):
   python tools/pred_clock.py <prefix>"""
import sys, glob
import numpy as np
_fs = sorted(glob.glob(sys.argv[1] + ".[0-9]*"), key=lambda x: int(x.rsplit(".", 1)[1]))
_fs = [f for f in _fs if np.fromfile(f, dtype=np.uint64).reshape(-1, 12)[:, 0].max(initial=0) > 0]
for fn in _fs[-2:-1] or _fs[-1:]:
    a = np.fromfile(fn, dtype=np.uint64).reshape(-1, 12)
    dup = (a[:, 6] >> np.uint64(63)).astype(bool)
    a6 = (a[:, 6] & np.uint64((1 << 63) - 1)).astype(np.int64)
    t = a[:, :6].astype(np.int64)
    t0 = t[:, 0].min()
    print(fn, "ctas", len(a), "dup", dup.sum(), "span us %.1f" % ((a6.max() - t0) / 1e3))
    dur = (a6 - t[:, 0]) / 1e3
    print("  cta lifetime us: mean %.1f p50 %.1f p90 %.1f max %.1f" % (dur.mean(), np.median(dur), np.percentile(dur, 90), dur.max()))
    def seg(i, j, name, m=None):
        m = np.ones(len(a), bool) if m is None else m
        ok = m & (t[:, i] > 0) & ((t[:, j] if j < 6 else a6) > 0)
        x = ((t[:, j] if j < 6 else a6) - t[:, i])[ok] / 1e3
        if len(x):
            print("  %-22s mean %6.2f p50 %6.2f p90 %6.2f max %6.2f (n=%d)" % (name, x.mean(), np.median(x), np.percentile(x, 90), x.max(), len(x)))
    seg(0, 1, "pre (zero+loads)")
    seg(1, 2, "pass1")
    seg(2, 3, "reserve")
    seg(3, 4, "select")
    seg(1, 5, "copy")
    seg(4, 6, "group end -> cta end")
    seg(1, 6, "dup: rest", dup)
    if dup.any():
        d = a[dup].astype(np.int64)
        allm = (d[:, 8] >> 62) & 1
        d8 = d[:, 8] & ((1 << 62) - 1)
        fb = d[:, 9] > 0
        endp = np.where(fb, d[:, 9], d[:, 8])
        print("  dup ctas: fallback %d; dup path end from copy end %.1f; select %.1f; copy end from pre %.1f (means, us)" % (
            fb.sum(), ((endp - d[:, 5]) / 1e3).mean(), ((d[:, 11] - endp) / 1e3).mean(), ((d[:, 5] - d[:, 1]) / 1e3).mean()))
    # concurrency: starts over time
    st = (t[:, 0] - t0) / 1e3
    print("  start times: first 10%% by %.1f us, 50%% by %.1f, 90%% by %.1f, last %.1f" % tuple(np.percentile(st, [10, 50, 90, 100])))
