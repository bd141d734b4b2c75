#!/bin/bash
# Profiling pass on the GPU box (one GPU): launch lists of the last applies and ncu --set full
# captures of named kernels, reduced to text under gpurun_out/<tag>/.
#   tools/prof.sh <tag> "<cfg> ..." "<cfg>:<kernel>:<skip>:<count> ..."
tag=$1; cfgs=$2; kern=$3
out=gpurun_out/$tag; mkdir -p $out
for c in $cfgs; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
      --csv --log-file $out/launches_$c.csv python bench.py --config $c --steps 2 --warmup 3 --no-cpu-baseline \
      > $out/launches_$c.log 2>&1
done
for spec in $kern; do
  IFS=: read c k s n <<< "$spec"
  f=$out/ncu_${c}_$k
  timeout 900 ncu --set full --clock-control none --import-source on -k "regex:^$k" -s $s -c $n \
      -o $f python bench.py --config $c --steps 1 --warmup 3 --no-cpu-baseline > $f.log 2>&1
  ncu -i $f.ncu-rep --page raw --csv > $f.raw.csv 2>/dev/null
  ncu -i $f.ncu-rep --page details > $f.details.txt 2>/dev/null
  ncu -i $f.ncu-rep --page source --csv > $f.source.csv 2>/dev/null
  [ "$KEEP" = 1 ] || rm -f $f.ncu-rep
done
