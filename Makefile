# Build everything in-tree (the .so files travel to the GPU box with gpurun).
#   make            -> graphgen + oracle + CUDA library (sm_100a)
NVCC      ?= /usr/local/cuda/bin/nvcc
HOSTCC    := $(shell test -x /usr/bin/gcc && echo /usr/bin/gcc || echo gcc)
PKG       := paper_conf_ppopp_wangllwm00z25_b200
CUDA_ARCH := -gencode arch=compute_100a,code=sm_100a
NVFLAGS   := $(EXTRA) -O3 -std=c++17 $(CUDA_ARCH) -lineinfo -Xcompiler -fPIC,-O3,-Wall -Iinclude \
             --expt-relaxed-constexpr -Xptxas -warn-spills
CSRC      := $(wildcard $(PKG)/csrc/*.cu) $(wildcard $(PKG)/csrc/*.cuh) $(wildcard $(PKG)/csrc/*.h) include/gala.h

all: graphgen/libgraphgen.so oracle/liboracle.so $(PKG)/libgala.so

graphgen/libgraphgen.so: graphgen/graphgen.c
	$(HOSTCC) -O3 -fopenmp -fPIC -shared -Wall -Wextra -o $@ $< -lm

oracle/liboracle.so: oracle/gala_oracle.c
	$(HOSTCC) -O2 -fopenmp -fPIC -shared -Wall -Wextra -o $@ $<

$(PKG)/libgala.so: $(CSRC)
	$(NVCC) $(NVFLAGS) -shared -o $@ $(wildcard $(PKG)/csrc/*.cu) -ldl

clean:
	rm -f graphgen/libgraphgen.so oracle/liboracle.so $(PKG)/libgala.so

.PHONY: all clean
