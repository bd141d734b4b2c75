#!/bin/bash
# round-2 closing pass (part B): ncu launch lists + ncu --set full of the dominant kernels,
# compute-sanitizer memcheck / racecheck over the small GPU tests -> gpurun_out/<tag>/
tag=${1:-r2bev}; out=gpurun_out/$tag; mkdir -p $out
tools/prof.sh $tag "c2 c3 c1" "c2:k_merge3:3:1 c3:k_merge3:3:1 c2:k_rows_fused:3:1 c2:k_casc_cols_tma:3:1"
TOOLS="memcheck racecheck" tools/sanitize.sh $tag
