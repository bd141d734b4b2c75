#!/bin/bash
# Round profile capture (one GPU): launch lists of the bench command + full ncu of the top kernel.
# Outputs in gpurun_out/; summarise locally with tools_profile_summary.py into profiles/.
for c in c2 c3; do
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
      --log-file gpurun_out/launches_$c.csv python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline \
      > gpurun_out/launches_$c.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k "regex:^k_merge3$" -s 2 -c 1 \
      -o gpurun_out/ncu_merge_$c python bench.py --config $c --steps 1 --warmup 3 --no-cpu-baseline \
      > gpurun_out/ncu_merge_$c.log 2>&1
done
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/gpu.txt
