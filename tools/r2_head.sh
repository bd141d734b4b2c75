#!/bin/bash
# HEAD check: smoke, every GPU test, the main bench lines -> gpurun_out/<tag>/
tag=${1:-head}; out=gpurun_out/$tag; mkdir -p $out
nvidia-smi > $out/nvidia_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $out/smoke.txt 2>&1
(time timeout 2400 python -m pytest tests -x -q -m gpu --durations=15) > $out/pytest_gpu.txt 2>&1
timeout 900 python bench.py > $out/bench_default.json 2> $out/bench_default.err
timeout 900 python bench.py --config c3 --no-cpu-baseline > $out/bench_c3.json 2> $out/bench_c3.err
timeout 300 python bench.py --config c1 --no-cpu-baseline > $out/bench_c1.json 2> $out/bench_c1.err
timeout 600 python bench.py --config c3 --input store --no-cpu-baseline > $out/bench_c3_store.json 2> $out/bench_c3_store.err
