#!/bin/bash
# GPU tests of the apply paths + the store / records benches (tools/r2_check3.sh <tag>)
out=gpurun_out/$1; mkdir -p $out
timeout 1500 python -m pytest tests -m gpu -x -q > $out/pytest.txt 2>&1
for c in c3 c2; do
  timeout 300 python bench.py --config $c --input store --steps 10 --warmup 3 --no-cpu-baseline > $out/bench_${c}_store.json 2> $out/bench_${c}_store.err
  timeout 300 python bench.py --config $c --input records --steps 10 --warmup 3 --no-cpu-baseline > $out/bench_${c}_records.json 2> $out/bench_${c}_records.err
done
