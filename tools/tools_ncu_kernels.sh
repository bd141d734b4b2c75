#!/bin/bash
# ncu --set full captures of individual hot-path kernels (one GPU), one report per kernel:
#   tools_ncu_kernels.sh <config> "<kernel>:<skip>:<count> ..." <prefix>
# Reports are reduced to text on the box (raw csv + details page); .ncu-rep files are
# kept only if KEEP=1 (gpurun brings back at most 64 MiB).
cfg=$1; list=$2; pre=$3
for spec in $list; do
  IFS=: read k s c <<< "$spec"
  out=gpurun_out/${pre}_$k
  timeout 600 ncu --set full --clock-control none --import-source on -k "regex:^$k\$" -s $s -c $c \
      -o $out python bench.py --config $cfg --steps 1 --warmup 3 --no-cpu-baseline > $out.log 2>&1
  ncu -i $out.ncu-rep --page raw --csv > $out.raw.csv 2>/dev/null
  ncu -i $out.ncu-rep --page details > $out.details.txt 2>/dev/null
  [ "$KEEP" = 1 ] || rm -f $out.ncu-rep
done
