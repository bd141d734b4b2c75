#!/bin/bash
# usage: tools_ncu_one.sh <config> <kernel-regex> <skip> <count> <outname>
ncu --set full --clock-control none --cache-control ${CACHE:-all} --import-source on -k "regex:$2" -s $3 -c $4 -o gpurun_out/$5 \
    python bench.py --config $1 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/$5.log 2>&1
