#!/bin/bash
# delta-store path: GPU tests + traces + benches (tools/r2_store.sh <tag>)
out=gpurun_out/$1; mkdir -p $out
timeout 900 python -m pytest tests/test_gpu_store.py tests/test_gpu_records.py -x -q > $out/pytest.txt 2>&1
tools/r2_trace.sh $1 "c3:store"
for c in c3 c2; do timeout 300 python bench.py --config $c --input store --steps 10 --warmup 3 --no-cpu-baseline > $out/bench_${c}_store_t.json 2> $out/bench_${c}_store_t.err; done
