#!/bin/bash
# iteration pass: focused GPU tests, the C1/C2/C3 bench lines, device step traces -> gpurun_out/<tag>/
tag=${1:-iter}; tests=${2:-"tests/test_gpu_parity.py tests/test_gpu_tombstone.py tests/test_gpu_sharded.py"}
out=gpurun_out/$tag; mkdir -p $out
(time timeout 1500 python -m pytest $tests -x -q -m gpu) > $out/pytest_gpu.txt 2>&1
timeout 900 python bench.py --no-cpu-baseline > $out/bench_c2.json 2> $out/bench_c2.err
timeout 900 python bench.py --config c3 --no-cpu-baseline > $out/bench_c3.json 2> $out/bench_c3.err
timeout 300 python bench.py --config c1 --no-cpu-baseline > $out/bench_c1.json 2> $out/bench_c1.err
H2TAP_TRACE=1 timeout 600 python bench.py --no-cpu-baseline --steps 4 --warmup 3 --sync-apply > $out/trace_c2.json 2> $out/trace_c2.err
H2TAP_TRACE=1 timeout 600 python bench.py --config c3 --no-cpu-baseline --steps 4 --warmup 3 --sync-apply > $out/trace_c3.json 2> $out/trace_c3.err
