#!/bin/bash
# compute-sanitizer tiers (memcheck, racecheck, synccheck, initcheck) over the small GPU
# parity tests: every kernel of the flat-op, delta-record, tombstone, dynamic and sharded
# paths at C1 size or smaller.  Exact allocations (no torch caching) so memcheck sees the
# real buffer ends.  Logs under gpurun_out/<tag>/.
tag=${1:-sanitize}; out=gpurun_out/$tag; mkdir -p $out
export PYTORCH_NO_CUDA_MEMORY_CACHING=1
SEL='tests/test_gpu_parity.py tests/test_gpu_records.py tests/test_gpu_tombstone.py tests/test_gpu_dynamic.py tests/test_gpu_sharded.py'
DESEL='--deselect tests/test_gpu_dynamic.py::test_full_size_sampled_rows --deselect tests/test_gpu_parity.py::test_rmat_c1_config'
for tool in ${TOOLS:-memcheck racecheck synccheck initcheck}; do
  extra=""
  [ $tool = memcheck ] && extra="--leak-check no"
  [ $tool = racecheck ] && extra="--racecheck-report hazard"
  timeout 3000 compute-sanitizer --tool $tool $extra --print-limit 100 --error-exitcode 9 \
      python -m pytest $SEL $DESEL -x -q -p no:cacheprovider > $out/$tool.txt 2>&1
  echo "$tool exit $?" >> $out/summary.txt
done
