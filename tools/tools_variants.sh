#!/bin/bash
# build-variant sweep: per-step device trace of each var/lib_*.so (H2TAP_LIB override)
for f in var/lib_*.so; do
  n=$(basename $f .so)
  for c in ${CONFIGS:-c3}; do
    echo "$n $c $(H2TAP_LIB=$f H2TAP_TRACE=1 timeout 300 python tools/tools_trace.py $c 2>&1 | grep 'h2tap trace' | tail -1)" >> gpurun_out/variants.txt
  done
done
