summ='import json,sys
for l in sys.stdin:
    l=l.strip()
    if not l.startswith("{"): continue
    d=json.loads(l); r=d["roofline"]; p=d["path"]
    print(d["config"]["name"], d["config"].get("input","ops"), "value=%.4g"%d["value"], "ms/step=%.3f"%d["ms_per_step"], "merge frac=%.3f"%r["frac"], "path_frac=%.3f"%p["frac_of_peak"], {k:round(v,3) for k,v in p["phase_ms"].items()}, "e2e=%.4g"%d["e2e"]["value"], "h2d=%d"%d["e2e"]["h2d_bytes_per_step"], d.get("checks"))'
for c in c2 c3; do
  for inp in ops records; do
    timeout 900 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --input $inp --checks 2>&1 | python -c "$summ" | tee -a gpurun_out/bench_records.txt
  done
done
