#!/bin/bash
# evidence pass: ncu launch lists (c1 c2 c3) + ncu --set full of the dominant kernels -> gpurun_out/<tag>/
tag=${1:-evid}; out=gpurun_out/$tag; mkdir -p $out
tools/prof.sh $tag "c2 c3 c1" "c2:k_merge3:3:1 c3:k_merge3:3:1 c2:k_rows_fused:3:1 c3:rs_coop:3:1 c3:k_reduce_classify:3:1"
timeout 600 ncu --set full --clock-control none -k regex:k_dyn_cascade -c 1 -o $out/ncu_dyn_cascade python bench.py --replica dyn --node-deletes 200 --no-cpu-baseline --cycles 2 > $out/ncu_dyn.log 2>&1
ncu -i $out/ncu_dyn_cascade.ncu-rep --page details > $out/ncu_dyn_cascade.details.txt 2>/dev/null
ncu -i $out/ncu_dyn_cascade.ncu-rep --page raw --csv > $out/ncu_dyn_cascade.raw.csv 2>/dev/null
rm -f $out/ncu_dyn_cascade.ncu-rep
