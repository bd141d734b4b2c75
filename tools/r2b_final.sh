#!/bin/bash
# round-2 closing pass (part A): smoke, every GPU test, the bench lines -> gpurun_out/<tag>/
tag=${1:-r2b}; out=gpurun_out/$tag; mkdir -p $out
nvidia-smi > $out/nvidia_smi.txt 2>&1
lscpu > $out/host_lscpu.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $out/smoke.txt 2>&1
(time timeout 2400 python -m pytest tests -q -m gpu --durations=20) > $out/pytest_gpu_full.txt 2>&1
timeout 900 python bench.py > $out/bench_default.json 2> $out/bench_default.err
timeout 900 python bench.py --config c3 > $out/bench_c3.json 2> $out/bench_c3.err
timeout 300 python bench.py --config c1 --no-cpu-baseline > $out/bench_c1.json 2> $out/bench_c1.err
timeout 900 python bench.py --config c4 --steps 5 --no-cpu-baseline > $out/bench_c4.json 2> $out/bench_c4.err
timeout 600 python bench.py --config c3 --input store --no-cpu-baseline > $out/bench_c3_store.json 2> $out/bench_c3_store.err
timeout 600 python bench.py --config c2 --input store --no-cpu-baseline > $out/bench_c2_store.json 2> $out/bench_c2_store.err
timeout 600 python bench.py --config c3 --input records --no-cpu-baseline > $out/bench_c3_records.json 2> $out/bench_c3_records.err
timeout 600 python bench.py --replica dyn > $out/bench_dyn.json 2> $out/bench_dyn.err
timeout 900 python bench.py --impl reference > $out/bench_ref.json 2> $out/bench_ref.err
timeout 900 python bench.py --gpus 2 --dist-backend gloo --config c3 --steps 5 > $out/bench_g2_c3.json 2> $out/bench_g2_c3.err
