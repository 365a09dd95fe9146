"""Summarise A/B bench lines: tools/ab_summary.py gpurun_out/TAG_*.json (dev helper)."""
import json
import sys

for f in sys.argv[1:]:
    try:
        d = [json.loads(l) for l in open(f) if l.startswith("{")][0]
    except (IndexError, OSError, ValueError):
        print(f"{f}: no line")
        continue
    k = (d.get("roofline") or {}).get("kernels") or {}
    ks = "  ".join("%s %.1f" % (n.split("_")[0].upper(), v["ms"] * 1000) for n, v in k.items())
    st = d.get("stats") or {}
    print("%-28s %7.0f Mk/s  step %7.1f us  %s  ui_share %s hit %.4f" % (
        f.split("/")[-1], d["value"], d["ms_per_step"] * 1000, ks, d.get("ui_share_ppm", st.get("ui_share_ppm")),
        d.get("hit_ratio", 0)))
