"""one-line summaries of bench JSON files: python tools/bench_brief.py <files>"""
import json
import sys

for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).readline())
    except Exception as e:
        print(f, "ERR", e)
        continue
    r = d.get("roofline") or {}
    p = d.get("path") or {}
    e = d.get("e2e") or {}
    extra = {k: d[k] for k in ("delete_hit_rate",) if k in d}
    if "reads" in d:
        extra["reads"] = {k: round(v, 2) for k, v in d["reads"].items() if isinstance(v, float)}
    print(f"{f.split('/')[-1]:28s} value {d.get('value', 0):.4g} ms {d.get('ms_per_step', d.get('ms_per_cycle', 0)):.3f} "
          f"frac {r.get('frac', 0) or 0:.3f} path {p.get('frac_of_peak', 0) or 0:.3f} e2e {e.get('value', 0):.4g} {extra}")
