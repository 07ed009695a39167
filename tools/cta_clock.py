import sys, glob, numpy as np
names = ["group", "insert", "owners", "passA", "passB", "qhash", "passC"]
for fn in sorted(glob.glob(sys.argv[1] + ".*"))[-1:]:
    a = np.fromfile(fn, dtype=np.uint64).reshape(-1, 10).astype(np.int64)
    m = a[:, 0] > 0
    a = a[m]
    st, en = a[:, 0], a[:, 1]
    ops = a[:, 2] & 0xFFFFFFFF; n = a[:, 2] >> 32
    t0 = st.min(); dur = (en - st) / 1000.0
    print(fn, "leaders", m.sum(), "span us %.1f" % ((en.max() - t0) / 1000.0))
    for lo, hi in ((0, 64), (64, 256), (256, 1024), (1024, 2048), (2048, 10**9)):
        mm = (ops >= lo) & (ops < hi)
        if not mm.any():
            continue
        stamps = [a[mm, 0]] + [a[mm, k] for k in (3, 4, 5, 6, 7, 8)] + [a[mm, 1]]
        parts = []
        for k in range(len(stamps) - 1):
            x, y = stamps[k], stamps[k + 1]
            ok = (x > 0) & (y > 0)
            parts.append("%s %.1f" % (names[k], ((y - x)[ok].mean() / 1e3) if ok.any() else -1))
        print("  ops [%d,%d): %d ctas, mean dur %.1f us | %s" % (lo, hi, mm.sum(), dur[mm].mean(), ", ".join(parts)))
