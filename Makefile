# Native build: the product library (sm_100a CUDA + C-ABI), the seeded input generator and the
# CPU oracle (test infrastructure; built here, never linked into the product).
NVCC     ?= /usr/local/cuda/bin/nvcc
HOSTCC   := $(shell test -x /usr/bin/gcc && echo /usr/bin/gcc || echo gcc)
PKG      := paper_conf_ipps_cuissf17_b200
CSRC     := $(PKG)/csrc
ARCH     := -gencode arch=compute_100a,code=sm_100a
# TUNING=1 also compiles the kernels' alternative tile/stage variants (PP_*_VARIANT selects them)
TUNING   ?= 0
NVFLAGS  := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O2,-Wall -Iinclude -I$(CSRC) --expt-relaxed-constexpr \
            -DPP_TUNING_VARIANTS=$(TUNING)
CUSRC    := $(wildcard $(CSRC)/*.cu)
CPPSRC   := $(wildcard $(CSRC)/*.cpp)
HDRS     := $(wildcard $(CSRC)/*.h $(CSRC)/*.hpp $(CSRC)/*.cuh) include/ppipe.h

all: synth oracle ppipe example

synth: synth/libsynth.so
synth/libsynth.so: synth/synth.c
	$(HOSTCC) -O2 -fopenmp -fPIC -shared -o $@ $<

oracle: oracle/liboracle.so
oracle/liboracle.so: oracle/oracle.c
	$(HOSTCC) -O2 -ffp-contract=off -fno-fast-math -fopenmp -fPIC -shared -o $@ $<

ppipe: $(PKG)/libppipe.so
$(PKG)/libppipe.so: $(CUSRC) $(CPPSRC) $(HDRS)
	$(NVCC) $(NVFLAGS) -shared -o $@ $(CUSRC) $(CPPSRC) -lcudart -ldl

example: examples/stencil_offload
examples/stencil_offload: examples/stencil_offload.c include/ppipe.h $(PKG)/libppipe.so
	$(HOSTCC) -O2 -Iinclude -o $@ $< -L$(PKG) -lppipe -Wl,-rpath,'$$ORIGIN/../$(PKG)'

clean:
	rm -f synth/libsynth.so oracle/liboracle.so $(PKG)/libppipe.so

.PHONY: all synth oracle ppipe example clean
