#!/bin/bash
tag=${1:-prof6}; out=gpurun_out/$tag; mkdir -p $out
for v in base nosplit; do
  lib=""; [ $v != base ] && lib="H2TAP_LIB=build/libh2tap_$v.so"
  for c in c3 c2; do env $lib timeout 300 python bench.py --config $c --steps 10 --no-cpu-baseline > $out/bench_${c}_$v.json 2> $out/bench_${c}_$v.err; done
done
tools/prof.sh $tag "c2 c3" "c2:k_merge3:3:1 c2:k_rows_fused:3:1 c3:k_merge3:3:1 c3:k_reduce_classify:3:1 c3:rs_coop:3:1"
