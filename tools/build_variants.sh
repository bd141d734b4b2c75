#!/bin/bash
# build-variant experiments: build/libh2tap_<name>.so with extra -D flags (H2TAP_LIB=... selects one)
#   tools/build_variants.sh "name:-DFLAG=1 -DX=2" ...
for v in "$@"; do
  n=${v%%:*}; f=${v#*:}
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared \
      --expt-relaxed-constexpr $f -o build/libh2tap_$n.so paper_conf_edbt_jibrilabs23_b200/csrc/h2tap.cu &
done
wait
