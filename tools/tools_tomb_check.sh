python -m pytest tests -m gpu -q -x 2>&1 | tail -3
summ='import json,sys
for l in sys.stdin:
    l=l.strip()
    if not l.startswith("{"): continue
    d=json.loads(l); r=d["roofline"]; p=d["path"]
    print(d["config"]["name"], d["config"].get("id_mode","compact"), "value=%.4g"%d["value"], "ms/step=%.3f"%d["ms_per_step"], "merge frac=%.3f"%r["frac"], "path_frac=%.3f"%p["frac_of_peak"], {k:round(v,3) for k,v in p["phase_ms"].items()})'
for t in "" "--tombstone"; do timeout 600 python bench.py --config c2 --steps 10 --warmup 3 --no-cpu-baseline $t 2>&1 | python -c "$summ"; done
