#!/bin/bash
tag=${1:-spec1}; out=gpurun_out/$tag; mkdir -p $out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_store.py tests/test_gpu_records.py tests/test_gpu_sharded.py tests/test_gpu_sharded_mp.py tests/test_gpu_tombstone.py tests/test_gpu_dynamic.py -x -q > $out/pytest.txt 2>&1
for v in base nospec; do
  lib=""; [ $v != base ] && lib="H2TAP_LIB=build/libh2tap_$v.so"
  for c in c3 c2 c1; do env $lib timeout 300 python bench.py --config $c --steps 20 --no-cpu-baseline > $out/bench_${c}_$v.json 2> $out/bench_${c}_$v.err; done
done
