#!/bin/bash
# host+device step trace (H2TAP_TRACE=1): tools/r2_trace.sh <tag> "<config>:<input> ..."
out=gpurun_out/$1; mkdir -p $out
for ci in $2; do c=${ci%%:*}; i=${ci#*:}
H2TAP_TRACE=1 timeout 300 python bench.py --config $c --input $i --steps 4 --warmup 3 --no-cpu-baseline > $out/bench_${c}_$i.json 2> $out/trace_${c}_$i.txt
done
