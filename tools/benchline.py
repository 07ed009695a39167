"""Print the headline, the roofline and the per-kernel breakdown of a bench log's JSON line."""
import json
import sys

for line in open(sys.argv[1]):
    if not line.startswith("{"):
        continue
    d = json.loads(line)
    print("value %.4g %s  ms/step %.4f  e2e %s" % (d["value"], d["unit"], d["ms_per_step"],
                                                   (d.get("e2e") or {}).get("value")))
    r = d.get("roofline") or {}
    print("roofline", {k: r.get(k) for k in ("kernel", "achieved", "frac", "avg_us")})
    print("step_roofline", {k: (d.get("step_roofline") or {}).get(k) for k in ("achieved_gbs", "frac")})
    for k, v in (d.get("kernels") or {}).items():
        print("  %-16s %7.2f us  %s" % (k, v.get("avg_us", 0), v.get("achieved_gbs", "")))
    if "verify" in d:
        print("verify", d["verify"].get("ok"))
