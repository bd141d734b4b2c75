#!/bin/bash
# full ncu captures of the top kernels (one GPU); reports land in gpurun_out/
set -x
ncu --set full --clock-control none --import-source on -k 'regex:^(k_merge|k_reduce_classify|rs_onesweep|k_offsets_scan)$' \
    -s 18 -c 9 -o gpurun_out/prof_c3 python bench.py --config c3 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_c3.log 2>&1
ncu --set full --clock-control none --import-source on -k 'regex:^(k_merge|k_casc_cols|k_edge_prep|k_remap|k_offsets_old)$' \
    -s 4 -c 7 -o gpurun_out/prof_c2 python bench.py --config c2 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_c2.log 2>&1
ls -la gpurun_out
