#!/bin/bash
tag=${1:-async1}; out=gpurun_out/$tag; mkdir -p $out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_store.py tests/test_gpu_records.py tests/test_gpu_sharded.py tests/test_gpu_sharded_mp.py tests/test_gpu_tombstone.py tests/test_gpu_dynamic.py -x -q > $out/pytest.txt 2>&1
for c in c3 c2 c1; do
  timeout 300 python bench.py --config $c --steps 20 --no-cpu-baseline > $out/bench_${c}_async.json 2> $out/bench_${c}_async.err
  timeout 300 python bench.py --config $c --steps 20 --no-cpu-baseline --sync-apply > $out/bench_${c}_sync.json 2> $out/bench_${c}_sync.err
done
