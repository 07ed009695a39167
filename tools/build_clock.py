"""Summarise DUM_BUILD_CLOCK dumps (per apply item / walk item globaltimer
stamps of k_apply and k_walk):  python tools/build_clock.py <prefix>"""
import sys, glob
import numpy as np
fs = sorted(glob.glob(sys.argv[1] + ".[0-9]*"), key=lambda x: int(x.rsplit(".", 1)[1]))
for fn in fs[-2:-1] or fs[-1:]:
    raw = np.fromfile(fn, dtype=np.uint64)
    ni, nl = int(raw[0] & 0xFFFFFFFF), int(raw[0] >> 32)
    a = raw[1:].reshape(-1, 4).astype(np.int64)
    ap, wk = a[:ni], a[ni:ni + nl]
    for name, x, szf in (("k_apply", ap, lambda r: r[:, 3] & 0xFFFFFFFF), ("k_walk", wk, lambda r: r[:, 3])):
        if not len(x):
            continue
        t0 = x[:, 0].min()
        dur = (x[:, 1] - x[:, 0]) / 1e3
        cta = x[:, 2] >> 32
        print("%s %s: items %d, span %.1f us (first start +%.1f, last end +%.1f)" % (
            fn, name, len(x), (x[:, 1].max() - t0) / 1e3, 0, (x[:, 1].max() - t0) / 1e3))
        print("  item dur us: mean %.2f p50 %.2f p90 %.2f max %.2f" % (dur.mean(), np.median(dur), np.percentile(dur, 90), dur.max()))
        st = (x[:, 0] - t0) / 1e3
        print("  starts: 10%% by %.1f, 50%% by %.1f, 90%% by %.1f, last %.1f us" % tuple(np.percentile(st, [10, 50, 90, 100])))
        busy = np.bincount(cta, weights=dur)
        print("  per-CTA busy us: mean %.1f max %.1f; CTAs %d" % (busy[busy > 0].mean(), busy.max(), (busy > 0).sum()))
        sz = szf(x)
        for lo, hi in ((0, 64), (64, 256), (256, 1024), (1024, 1 << 30)):
            m = (sz >= lo) & (sz < hi)
            if m.any():
                print("  size [%d,%d): %d items, mean dur %.2f us" % (lo, hi, m.sum(), dur[m].mean()))
