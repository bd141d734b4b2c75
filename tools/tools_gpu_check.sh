#!/bin/bash
# quick GPU iteration helper: tests + bench summaries (+ optional ncu launch lists)
set -o pipefail
summ='import json,sys
for l in sys.stdin:
    l=l.strip()
    if not l.startswith("{"): continue
    d=json.loads(l); r=d["roofline"]; p=d["path"]
    print(d["config"]["name"], "value=%.4g"%d["value"], "ms/step=%.3f"%d["ms_per_step"], "merge=%.3fms %.0fGB/s frac=%.3f"%(r["ms_per_launch"], r["achieved"], r["frac"]), "path_frac=%.3f"%p["frac_of_peak"], {k:round(v,3) for k,v in p["phase_ms"].items()}, "e2e=%.4g"%d["e2e"]["value"], "launches=%d"%d["gpu_launches"])'
timeout 600 python -m pytest tests -m gpu -q -x 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
for c in ${CONFIGS:-c2 c3}; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline 2>&1 | python -c "$summ" | tee -a gpurun_out/bench_summary.txt
done
if [ -n "$TRACE" ]; then
  for c in ${CONFIGS:-c2 c3}; do
    H2TAP_TRACE=1 timeout 300 python tools/tools_trace.py $c 2>&1 | grep "h2tap trace" | tail -3 > gpurun_out/trace_$c.txt
  done
fi
cat gpurun_out/pytest_gpu.txt
