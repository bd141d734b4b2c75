#!/bin/bash
# delta-store read-ahead placement (timing includes the read-ahead via h2tap_ds_join):
# H2TAP_RA = 0 (behind the scan), 1 (behind the merge launch), 2 (after the cycle), 3 (once the merge runs)
out=gpurun_out/$1; mkdir -p $out
for ra in 0 1 2 3; do for c in c3 c2; do
  H2TAP_RA=$ra timeout 300 python bench.py --config $c --input store --steps 10 --warmup 3 --no-cpu-baseline > $out/bench_${c}_ra$ra.json 2> $out/bench_${c}_ra$ra.err
done; done
for ra in 0 3; do H2TAP_RA=$ra H2TAP_TRACE=1 timeout 300 python bench.py --config c3 --input store --steps 3 --warmup 3 --no-cpu-baseline > $out/trace_c3_ra$ra.json 2> $out/trace_c3_ra$ra.txt; done
