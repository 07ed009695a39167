#!/usr/bin/env python3
"""Turn gpurun_out/<tag>_launches.csv and <tag>_<kernel>.ncu-rep into the
tracked summaries under profiles/ (and profiles/ncu_traffic.json, read by
bench.py for the roofline `traffic` field).
   python tools/summarize_profiles.py <tag> [kernels...]"""
import csv, io, json, os, subprocess, sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1]
kernels = sys.argv[2:] or ["k_predict", "k_apply", "k_walk", "k_chain", "k_ingest"]
out_dir = os.path.join(ROOT, "profiles")
os.makedirs(out_dir, exist_ok=True)
lines = ["# ncu summary `%s`" % tag, ""]

# ---- launch list ----
lp = os.path.join(ROOT, "gpurun_out", "%s_launches.csv" % tag)
if os.path.exists(lp):
    rows = list(csv.reader(open(lp)))
    start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[start]
    ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    t = defaultdict(float); n = defaultdict(int); rd = defaultdict(float); wr = defaultdict(float)
    for r in rows[start + 1:]:
        if len(r) <= vi:
            continue
        name = r[ki].split("(")[0].replace("void ", "").replace("dum::", "").replace("<unnamed>::", "")
        v = float(r[vi].replace(",", ""))
        if r[mi] == "gpu__time_duration.sum":
            t[name] += v; n[name] += 1
        elif r[mi] == "dram__bytes_read.sum":
            rd[name] += v
        elif r[mi] == "dram__bytes_write.sum":
            wr[name] += v
    tot = sum(t.values())
    lines += ["## Launch list (`ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum "
              "--clock-control none` over `bench.py --steps 2 --warmup 3`; cold-cache, serialised: compare shares)", "",
              "| kernel | launches | total us | share | DRAM MB/launch |", "|---|---|---|---|---|"]
    for k, v in sorted(t.items(), key=lambda x: -x[1]):
        lines.append("| %s | %d | %.1f | %.3f | %.1f |" % (k, n[k], v / 1000, v / tot, (rd[k] + wr[k]) / n[k] / 1e6))
    lines.append("")

# ---- per-kernel full captures ----
traffic_path = os.path.join(out_dir, "ncu_traffic.json")
traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
for k in kernels:
    rep = os.path.join(ROOT, "gpurun_out", "%s_%s.ncu-rep" % (tag, k))
    if not os.path.exists(rep):
        continue
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rr = list(csv.reader(io.StringIO(raw)))
    if len(rr) < 3:
        continue
    hdr, units, v = rr[0], rr[1], rr[2]
    def g(m):
        return (v[hdr.index(m)], units[hdr.index(m)]) if m in hdr else ("-", "")
    dur = g("gpu__time_duration.sum"); rdb = g("dram__bytes_read.sum"); wrb = g("dram__bytes_write.sum")
    lines += ["## `%s` (`ncu --set full --clock-control none --import-source on`, one launch)" % k, ""]
    for m in ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
              "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
              "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
              "launch__registers_per_thread", "launch__shared_mem_per_block_dynamic",
              "launch__shared_mem_per_block_static", "launch__occupancy_limit_shared_mem",
              "launch__occupancy_limit_registers", "launch__grid_size", "launch__block_size"]:
        val, u = g(m)
        lines.append("- %s: %s %s" % (m, val, u))
    def tobytes(x):
        val, u = x
        try:
            f = float(val.replace(",", ""))
        except ValueError:
            return None
        return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
    b1, b2 = tobytes(rdb), tobytes(wrb)
    if b1 is not None and b2 is not None:
        traffic[k] = {"dram_bytes_per_launch": int(b1 + b2), "source": "%s_%s.ncu-rep" % (tag, k)}
    top = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "ncu_lines.py"), rep, "12"],
                         capture_output=True, text=True).stdout
    lines += ["", "Top source lines by warp-stall samples:", "", "```", top.rstrip(), "```", ""]
json.dump(traffic, open(traffic_path, "w"), indent=1)
open(os.path.join(out_dir, "%s_ncu.md" % tag), "w").write("\n".join(lines) + "\n")
print("\n".join(lines[:40]))
