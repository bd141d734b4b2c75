#!/bin/bash
# round-2 GPU check: new tests, variant benches, dyn and store benches -> gpurun_out/<tag>/
tag=${1:-r2check}; out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.smoke()" > $out/smoke.txt 2>&1
timeout 1500 python -m pytest tests/test_gpu_store.py tests/test_gpu_dynamic.py tests/test_gpu_parity.py \
    tests/test_gpu_records.py tests/test_gpu_sharded.py tests/test_gpu_sharded_mp.py tests/test_gpu_tombstone.py \
    -x -q --durations=10 > $out/pytest.txt 2>&1
for v in base casc2 casc1 cascmain lookq1 lookq8 rowtile1k rowtile256 items12; do
  lib=""; [ $v != base ] && lib="H2TAP_LIB=build/libh2tap_$v.so"
  env $lib timeout 300 python bench.py --config c2 --steps 10 --no-cpu-baseline > $out/bench_c2_$v.json 2> $out/bench_c2_$v.err
  case $v in base|lookq1|lookq8)
    env $lib timeout 300 python bench.py --config c3 --steps 10 --no-cpu-baseline > $out/bench_c3_$v.json 2> $out/bench_c3_$v.err;;
  esac
done
timeout 600 python bench.py --replica dyn --no-cpu-baseline > $out/bench_dyn.json 2> $out/bench_dyn.err
timeout 600 python bench.py --replica dyn --node-deletes 200 --no-cpu-baseline > $out/bench_dyn_nd.json 2> $out/bench_dyn_nd.err
timeout 600 python bench.py --config c3 --input store > $out/bench_c3_store.json 2> $out/bench_c3_store.err
timeout 600 python bench.py --config c3 --input records --no-cpu-baseline > $out/bench_c3_records.json 2> $out/bench_c3_records.err
timeout 600 python bench.py --config c2 --input store > $out/bench_c2_store.json 2> $out/bench_c2_store.err
for v in base rslook16; do
  lib=""; [ $v != base ] && lib="H2TAP_LIB=build/libh2tap_$v.so"
  env $lib timeout 600 python bench.py --config c4 --steps 5 --no-cpu-baseline > $out/bench_c4_$v.json 2> $out/bench_c4_$v.err
done
