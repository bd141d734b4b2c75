#!/bin/bash
tag=${1:-rec1}; out=gpurun_out/$tag; mkdir -p $out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_records.py tests/test_gpu_store.py -x -q > $out/pytest.txt 2>&1
timeout 600 python bench.py --config c3 --input records --no-cpu-baseline > $out/bench_c3_records.json 2> $out/bench_c3_records.err
timeout 600 python bench.py --config c3 --input store > $out/bench_c3_store.json 2> $out/bench_c3_store.err
timeout 600 python bench.py --config c2 --input records --no-cpu-baseline > $out/bench_c2_records.json 2> $out/bench_c2_records.err
timeout 600 python bench.py --config c2 --input store > $out/bench_c2_store.json 2> $out/bench_c2_store.err
