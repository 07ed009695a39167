#!/usr/bin/env python
"""Markdown tables from the round's committed measurement files (profiles/):
the migration sweep (config M), the closed-loop study,
the PCIe capture of the copy kernels and the kernel-boundary probe.

    python tools/summarize_r02.py [--migration F] [--f1 F] [--pcie F] [--pdl F] > profiles/r02_studies.md
"""
from __future__ import annotations

import argparse
import csv
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
P = os.path.join(ROOT, "profiles")


def migration(path):
    d = json.load(open(path))
    pk = d["host_link_peak"]
    out = ["## Config M: 2 MiB block migration (`tools/migration_sweep.py`)", "",
           "Host-link peak measured live: H2D %.1f GB/s, D2H %.1f GB/s, both directions at once %.1f GB/s "
           "(%s); HBM peak %.0f GB/s (MEASURED_PEAKS.json). Bytes of sampled blocks verified: %s."
           % (pk["h2d_gbs"], pk["d2h_gbs"], pk["bidir_gbs"], pk["how"], d["hbm_peak_gbs"], d["bytes_verified"]), "",
           "| direction | method | GB/s at n = max (median) | fraction of peak | smallest n at 0.8 |", "|---|---|---|---|---|"]
    for dn, v in d["summary"].items():
        for m, x in sorted(v.items()):
            out.append("| %s | %s | %.1f (n = %d) | %.3f | %s |" % (dn, m, x["gbs_median_at_max"], x["n_max"],
                                                                   x["frac_median_at_max"], x["smallest_n_at_0.8"]))
    out += ["", "Contiguous H2D, GB/s (median) by batch size:", "",
            "| n | " + " | ".join(["sm_copy", "tma_bulk", "copy_engine"]) + " |", "|---|---|---|---|"]
    pts = [p for p in d["points"] if p["order"] == "contiguous" and p["dir"] == "h2d"]
    for n in sorted(set(p["n"] for p in pts)):
        row = {p["method"]: p["gbs_median"] for p in pts if p["n"] == n}
        out.append("| %d | %s |" % (n, " | ".join("%.1f" % row.get(m, float("nan"))
                                                   for m in ("sm_copy", "tma_bulk", "copy_engine"))))
    perm = [p for p in d["points"] if p["order"] == "permuted" and p["dir"] == "h2d" and p["n"] == max(
        q["n"] for q in d["points"] if q["order"] == "permuted")]
    if perm:
        out += ["", "Permuted block order (n = %d, H2D): %s." % (perm[0]["n"], ", ".join(
            "%s %.1f GB/s" % (p["method"], p["gbs_median"]) for p in perm))]
    out += ["", "Concurrent H2D || D2H (two engines, half the SMs each for the copy kernels): TMA bulk reaches the "
            "bidirectional link; the copy-engine method synchronizes per call (its frame plan is read back), "
            "so its pair runs one after the other.", ""]
    return out


def f1(path):
    d = json.load(open(path))
    out = ["## Closed loop (SURVEY 8(f) row 1; `tools/sim_f1.py`, `dum_simulate`, metadata-only)", "",
           "Steady state = mean of iterations 1-9 of 10; per iteration. Fig. 10 ablation (PAPER.md L457): "
           "prefetch only = the whole window prefetched, the driver evicting least recently migrated blocks "
           "(window or not) beyond the free frames; + pre-eviction = D18 victims outside the window first; "
           "+ invalidation = inactive victims dropped without a write-back (L285).", ""]
    for c, r in d["configs"].items():
        out += ["### %s (W = %d blocks, C = %d frames, K = %d launches / iteration)" % (c, r["W"], r["C"], r["K"]),
                "", "| configuration | demand faults | demand write-back | demand invalidated | evicted for the "
                "window (write-back) | (invalidated) | prefetched |", "|---|---|---|---|---|---|---|"]
        for a, v in r["ablation"].items():
            s = v["steady_mean"]
            out.append("| %s | %.0f | %.0f | %.0f | %.0f | %.0f | %.0f |" % (
                a, s["faults"], s["demand_wb"], s["demand_inv"], s["pre_wb"], s["pre_inv"], s["prefetched"]))
        t = r["table5_shape"]
        nv = r["naive_um_vs_trace"]
        out += ["", "Table 5 shape: demand faults per iteration %.0f (naive UM) -> %.0f (engine, N = 32), ratio %.4f. "
                "Naive UM here vs the generator's naive-UM trace (`workloads/um_sim.c`): %+.2f%% (steady), "
                "from the demand rule (%s)." % (t["naive_um_faults_per_iter"], t["engine_faults_per_iter"], t["ratio"],
                                               100 * nv["rel_diff_steady"], nv["why"]), ""]
        if "degree_sweep" in r:
            out += ["Fig. 11 shape, degree N (demand faults per iteration, all three techniques):", "",
                    "| N | " + " | ".join(r["degree_sweep"].keys()) + " |",
                    "|---|" + "---|" * len(r["degree_sweep"]),
                    "| faults | " + " | ".join("%.0f" % v["faults"] for v in r["degree_sweep"].values()) + " |",
                    "| prefetched | " + " | ".join("%.0f" % v["prefetched"] for v in r["degree_sweep"].values()) + " |",
                    ""]
        if "geometry_sweep" in r:
            out += ["Fig. 12 / Table 6 shape, table geometry (N = 32):", "", "| config | faults | prefetched |",
                    "|---|---|---|"]
            for k, v in r["geometry_sweep"].items():
                out.append("| %s | %.0f | %.0f |" % (k, v["faults"], v["prefetched"]))
            out.append("")
    return out


def pcie(path):
    rows = list(csv.reader(open(path)))
    hdr = None
    recs = {}
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            x = dict(zip(hdr, r))
            recs.setdefault(x["ID"], {"kernel": x["Kernel Name"].split("(")[0]})[x["Metric Name"]] = float(
                x["Metric Value"].replace(",", ""))
    out = ["## PCIe traffic of the copy kernels (ncu, `%s`)" % os.path.basename(path), "",
           "One capture per launch (the sweep's first launches: 1-2 blocks of 2 MiB = 2,097,152 B each).", "",
           "| launch | kernel | us | PCIe read B | PCIe write B | DRAM read B | DRAM write B |",
           "|---|---|---|---|---|---|---|"]
    for i, x in sorted(recs.items(), key=lambda t: int(t[0])):
        out.append("| %s | %s | %.1f | %.0f | %.0f | %.0f | %.0f |" % (
            i, x["kernel"], x.get("gpu__time_duration.sum", 0) / 1000, x.get("pcie__read_bytes.sum", 0),
            x.get("pcie__write_bytes.sum", 0), x.get("dram__bytes_read.sum", 0), x.get("dram__bytes_write.sum", 0)))
    out += ["", "H2D moves ~1.09x the block over PCIe (request / completion headers), D2H ~1.13x: no re-reads.", ""]
    return out


def pdl(path):
    d = json.load(open(path))
    out = ["## Kernel boundaries inside a CUDA graph (`tools/pdl_probe.cu`)", "",
           "A chain of 20 dependent kernels captured once and replayed; with programmatic dependent launch "
           "(trigger at kernel start, wait before the first dependent load) vs plain stream order.", "",
           "| grid | work / thread | one kernel us | chain of 20 us | with PDL us |", "|---|---|---|---|---|"]
    for p in d["points"]:
        out.append("| %d | %d | %.2f | %.2f | %.2f |" % (p["grid"], p["iters"], p["one_kernel_us"], p["chain20_us"],
                                                        p["chain20_pdl_us"]))
    out += ["", "PDL made every chain slower here, so the engine keeps plain stream order inside its step graphs.", ""]
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--migration", default=os.path.join(P, "r02_migration_sweep.json"))
    ap.add_argument("--f1", default=os.path.join(P, "r02_f1_closed_loop.json"))
    ap.add_argument("--pcie", default=os.path.join(P, "r02_migration_pcie_ncu.csv"))
    ap.add_argument("--pdl", default=os.path.join(P, "r02_pdl_probe.json"))
    a = ap.parse_args()
    out = ["# Round-2 studies (B200): migration, closed loop, PCIe, kernel boundaries", ""]
    for fn, p in ((migration, a.migration), (f1, a.f1), (pcie, a.pcie), (pdl, a.pdl)):
        if os.path.exists(p):
            out += fn(p)
    print("\n".join(out))


if __name__ == "__main__":
    main()
