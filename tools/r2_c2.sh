#!/bin/bash
tag=${1:-c2a}; out=gpurun_out/$tag; mkdir -p $out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_tombstone.py tests/test_gpu_sharded.py tests/test_gpu_sharded_mp.py tests/test_gpu_records.py tests/test_gpu_store.py tests/test_gpu_fullsize.py -x -q > $out/pytest.txt 2>&1
for c in c2 c3; do timeout 300 python bench.py --config $c --steps 20 --no-cpu-baseline > $out/bench_${c}.json 2> $out/bench_${c}.err; done
H2TAP_TRACE=1 timeout 300 python bench.py --config c2 --steps 3 --warmup 3 --no-cpu-baseline --sync-apply 2> $out/trace_c2.err > /dev/null
