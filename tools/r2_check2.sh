#!/bin/bash
tag=${1:-r2check2}; out=gpurun_out/$tag; mkdir -p $out
timeout 900 python -m pytest tests/test_gpu_store.py tests/test_gpu_dynamic.py -x -q --durations=5 > $out/pytest.txt 2>&1
timeout 600 python bench.py --replica dyn --no-cpu-baseline > $out/bench_dyn.json 2> $out/bench_dyn.err
timeout 600 python bench.py --replica dyn --node-deletes 200 --no-cpu-baseline > $out/bench_dyn_nd.json 2> $out/bench_dyn_nd.err
timeout 600 python bench.py --config c3 --input store > $out/bench_c3_store.json 2> $out/bench_c3_store.err
timeout 600 python bench.py --config c3 --no-cpu-baseline > $out/bench_c3.json 2> $out/bench_c3.err
timeout 600 python bench.py --config c2 --no-cpu-baseline > $out/bench_c2.json 2> $out/bench_c2.err
PYTORCH_NO_CUDA_MEMORY_CACHING=1 timeout 1200 compute-sanitizer --tool initcheck --print-limit 20 --error-exitcode 9 \
    python -m pytest tests/test_gpu_parity.py -x -q -k "fig2 or tiny_fuzz or ldbc_shaped_small or node_ops" -p no:cacheprovider > $out/initcheck.txt 2>&1
echo "initcheck exit $?" >> $out/initcheck.txt
