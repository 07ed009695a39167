#!/usr/bin/env python3
"""Round-end summary: profiles/<round>_summary.md (+ bench_<tag>.json,
bench_fast_<tag>.json, bench_ref_<tag>.json) from the gpurun_out/<tag>_* files
of tools/final_round.sh, and the ncu summaries via tools/summarize_profiles.py.

    python tools/summarize_final.py <tag> [round]"""
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
G = os.path.join(ROOT, "gpurun_out")
P = os.path.join(ROOT, "profiles")
tag = sys.argv[1]
rnd = sys.argv[2] if len(sys.argv) > 2 else "r02"


def line(path):
    if not os.path.exists(path):
        return None
    js = [l for l in open(path) if l.startswith("{")]
    return json.loads(js[-1]) if js else None


def tail(path, n=3):
    if not os.path.exists(path):
        return "(missing)"
    return "".join(open(path).readlines()[-n:]).strip()


out = ["# Round-2 results on B200 (`%s`)" % tag, ""]
out += ["## GPU tests and smoke", "", "```", tail(os.path.join(G, tag + "_tests.log"), 2),
        tail(os.path.join(G, tag + "_smoke.log"), 2), "```", ""]

b = line(os.path.join(G, tag + "_bench.log"))
if b:
    json.dump(b, open(os.path.join(P, "bench_%s.json" % tag), "w"), indent=1)
    r, sr = b.get("roofline", {}), b.get("step_roofline", {})
    out += ["## Headline (`python bench.py --verify`, G, N = 1)", "",
            "| quantity | value |", "|---|---|",
            "| fault records/s (device, K steps back to back) | %.3g (%.4f ms/step) |" % (b["value"], b["ms_per_step"]),
            "| e2e through the C-ABI with pinned host inputs | %.3g records/s (%.4f ms/step) |"
            % (b["e2e"]["value"], b["e2e"]["ms_per_step"]) if b.get("e2e") else "| e2e | - |",
            "| dominant kernel | %s: %.1f GB/s of SURVEY 8(d) bytes = %.3f of %.1f GB/s (%s) |"
            % (r.get("kernel"), r.get("achieved") or 0, r.get("frac") or 0, r.get("peak") or 0, r.get("peak_source")),
            "| whole step | %.1f GB/s = %.3f of peak |" % (sr.get("achieved_gbs", 0), sr.get("frac", 0)),
            "| verify (last timed step vs oracle) | %s |" % (b.get("verify", {}).get("ok")),
            "| clocks | %s |" % json.dumps(b.get("clocks")),
            "| oracle, 1 core | %.3g records/s |" % b["cpu_baseline"]["value"] if b.get("cpu_baseline") else "",
            "| oracle, all cores | %.3g records/s |" % b["cpu_baseline_mt"]["value"] if b.get("cpu_baseline_mt") else "",
            ""]
    out += ["Per-kernel (breakdown pass, CUDA events on the launching stream):", "",
            "| kernel | avg us | SURVEY 8(d) GB/s | stream |", "|---|---|---|---|"]
    for k, v in b.get("kernels", {}).items():
        out.append("| %s | %.2f | %s | %s |" % (k, v["avg_us"], v.get("achieved_gbs", ""), v.get("stream", "main")))
    out += ["", "Counters per step: `%s`" % json.dumps(b.get("counters_per_step")), ""]
    mig = b.get("migration")
    if mig:
        out += ["Migration (config M in brief): host link %s; best %s" % (json.dumps(mig.get("host_link_peak")),
                                                                     json.dumps(mig.get("best"))), ""]
bf = line(os.path.join(G, tag + "_bench_fast.log"))
if bf:
    json.dump(bf, open(os.path.join(P, "bench_fast_%s.json" % tag), "w"), indent=1)
    out += ["## The fast-window mode (`bench.py --fast-windows`)", "",
            "%.3g records/s (%.4f ms/step); dominant kernel %s %.1f us" % (
                bf["value"], bf["ms_per_step"], bf["roofline"].get("kernel"), bf["roofline"].get("avg_us") or 0), ""]
bg = line(os.path.join(G, tag + "_bench_graph.log"))
if bg:
    json.dump(bg, open(os.path.join(P, "bench_graph_%s.json" % tag), "w"), indent=1)
    out += ["## Steps replayed as CUDA graphs (`bench.py --graph`)", "",
            "%.3g records/s (%.4f ms/step); e2e %.3g records/s (%.4f ms/step)" % (
                bg["value"], bg["ms_per_step"], bg["e2e"]["value"], bg["e2e"]["ms_per_step"]), ""]
br = line(os.path.join(G, tag + "_ref.log"))
if br:
    json.dump(br, open(os.path.join(P, "bench_ref_%s.json" % tag), "w"), indent=1)
    out += ["## Reference arm (`bench.py --impl reference`: the oracle)", "",
            "%.3g records/s; %s" % (br.get("value", 0), json.dumps(br.get("cpu_baseline"))), ""]
um = os.path.join(G, tag + "_um.log")
if os.path.exists(um):
    out += ["## Real UM (f3) and allocator hook (f4) on the GPU", "", "```"]
    out += [l.rstrip() for l in open(um) if "UM " in l or "passed" in l or "failed" in l]
    out += ["```", ""]
nproc = os.path.join(G, tag + "_nproc.txt")
if os.path.exists(nproc):
    out += ["Host: `%s`" % " / ".join(l.strip() for l in open(nproc).readlines()[:1]), ""]
subprocess.run([sys.executable, os.path.join(ROOT, "tools", "summarize_profiles.py"), tag,
                "k_predict", "k_build_exec", "k_chain", "k_ingest", "k_build_prep"], check=False)
out += ["ncu launch list and --set full captures: `profiles/%s_ncu.md`." % tag, ""]
open(os.path.join(P, "%s_summary.md" % rnd), "w").write("\n".join(l for l in out if l is not None) + "\n")
print("\n".join(out))
