#!/bin/bash
# variant benches: tools/r2_var.sh <tag> "<variant> ..." "<config> ..."
tag=$1; out=gpurun_out/$tag; mkdir -p $out
for v in $2; do
  lib=""; [ $v != base ] && lib="H2TAP_LIB=build/libh2tap_$v.so"
  for c in $3; do env $lib timeout 300 python bench.py --config $c --steps 10 --no-cpu-baseline > $out/bench_${c}_$v.json 2> $out/bench_${c}_$v.err; done
done
