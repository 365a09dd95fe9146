"""Print the headline fields of a bench.py JSON line (dev helper)."""
import json
import sys

for line in open(sys.argv[1]):
    if not line.startswith("{"):
        continue
    d = json.loads(line)
    r = d.get("roofline") or {}
    print("value %.1f %s | ms/step %.4f | hit %.4f | p50 %.1f us | e2e %s | launches %s | clocks %s" % (
        d["value"], d["unit"], d["ms_per_step"], d.get("hit_ratio", 0), d.get("p50_batch_latency_us", 0),
        (d.get("e2e") or {}).get("value"), d.get("gpu_launches"), d.get("clocks")))
    for k, v in (r.get("kernels") or {}).items():
        print("  %-10s %.4f ms  %-9s achieved %.1f GB/s of %.1f -> %.3f" % (k, v["ms"], v["bound"], v["achieved"],
                                                                          v["peak"], v["frac"]))
    if r:
        print("  step roofline %.1f us -> step_frac %.3f; link 1GiB %.1f GB/s" % (
            r.get("step_roofline_us", 0), r.get("step_frac", 0), r.get("host_link_1GiB_gbs", 0)))
    if d.get("cpu_baseline"):
        print("  cpu:", d["cpu_baseline"]["value"], d["cpu_baseline"]["sample"])
