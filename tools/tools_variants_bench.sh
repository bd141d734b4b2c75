#!/bin/bash
# build-variant sweep with the bench (device-resident batches): ms/step and phases per var/lib_*.so
summ='import json,sys
for l in sys.stdin:
    l=l.strip()
    if not l.startswith("{"): continue
    d=json.loads(l); p=d["path"]
    print("ms/step=%.3f"%d["ms_per_step"], {k:round(v,3) for k,v in p["phase_ms"].items()})'
for f in var/lib_*.so; do
  for c in ${CONFIGS:-c2}; do
    echo "$(basename $f .so) $c $(H2TAP_LIB=$f timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline 2>&1 | python -c "$summ")" >> gpurun_out/variants_bench.txt
  done
done
