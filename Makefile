# Build products (all in-tree so they travel to the GPU box with gpurun):
#   paper_conf_edbt_jibrilabs23_b200/libh2tap.so   product: sm_100a kernels + C ABI
#   oracle/liboracle.so, oracle/libo3.so            oracles O1, O3 (test infrastructure only)
#   synth/libsynth.so                               seeded input generators
NVCC ?= nvcc
PKG := paper_conf_edbt_jibrilabs23_b200
CSRC := $(PKG)/csrc
NVFLAGS := -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 \
           -Xcompiler -fPIC -shared --expt-relaxed-constexpr -Xptxas -v

all: lib oracle synth

lib: $(PKG)/libh2tap.so
$(PKG)/libh2tap.so: $(CSRC)/h2tap.cu $(CSRC)/kernels.cuh $(CSRC)/radix_sort.cuh $(CSRC)/dev_common.cuh $(CSRC)/dyn.cuh $(CSRC)/delta_store.cuh $(CSRC)/collective.cuh include/h2tap.h
	$(NVCC) $(NVFLAGS) -o $@ $(CSRC)/h2tap.cu 2> $(CSRC)/ptxas.log || (cat $(CSRC)/ptxas.log; false)

oracle: oracle/liboracle.so oracle/libo3.so
oracle/liboracle.so: oracle/o1_replay.cpp
	g++ -O2 -std=c++17 -fPIC -shared -o $@ $<
oracle/libo3.so: oracle/o3_alg2.cpp
	g++ -O2 -std=c++17 -fopenmp -fPIC -shared -o $@ $<

synth: synth/libsynth.so
synth/libsynth.so: synth/synth.c
	gcc -O2 -fopenmp -fPIC -shared -o $@ $<

clean:
	rm -f $(PKG)/libh2tap.so oracle/liboracle.so oracle/libo3.so synth/libsynth.so $(CSRC)/ptxas.log

.PHONY: all lib oracle synth clean
