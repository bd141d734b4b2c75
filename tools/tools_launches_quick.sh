#!/bin/bash
# launch list of a short bench run per config (per-kernel durations, serialised)
for c in ${CONFIGS:-c2 c3}; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
      --log-file gpurun_out/launches_$c.csv python bench.py --config $c --steps 1 --warmup 3 --no-cpu-baseline \
      > gpurun_out/launches_$c.log 2>&1
done
