"""Summarise an ncu launch-list CSV (gpu__time_duration + DRAM bytes per launch):
the kernels of the last bench step, in launch order, and per-kernel totals."""
import collections
import csv
import sys


def load(path):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[hi]
    ki, mi, vi, idi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
    d = collections.defaultdict(dict)
    for r in rows[hi + 1:]:
        if len(r) < len(h):
            continue
        name = r[ki].split("(")[0].replace("void ", "").replace("dum::", "")
        d[(int(r[idi]), name)][r[mi]] = float(r[vi].replace(",", ""))
    return sorted(d.items())


if __name__ == "__main__":
    items = load(sys.argv[1])
    last = int(sys.argv[2]) if len(sys.argv) > 2 else 30
    tot = 0
    for (i, k), m in items[-last:]:
        t = m.get("gpu__time_duration.sum", 0) / 1000
        tot += t
        print("%4d %-36s %8.2f us  rd %7.2f MB  wr %7.2f MB" % (i, k[:36], t, m.get("dram__bytes_read.sum", 0) / 1e6,
                                                             m.get("dram__bytes_write.sum", 0) / 1e6))
    print("sum %.1f us" % tot)
