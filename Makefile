# Builds the three native pieces in-tree (the .so files travel to the GPU box).
#   tracegen/libtracegen.so   seeded input generator (host C++, OpenMP)
#   oracle/liboracle.so       CPU oracle (test infrastructure only)
#   paper_conf_cgo_shensll18_b200/libcadv.so   the product: sm_100a CUDA + C-ABI
NVCC      ?= /usr/local/cuda/bin/nvcc
HOSTCXX   := /usr/bin/g++
ARCH      := -gencode arch=compute_100a,code=sm_100a
PKG       := paper_conf_cgo_shensll18_b200
CADV_SRC  := $(wildcard $(PKG)/csrc/*.cu) $(wildcard $(PKG)/csrc/*.cpp)
CADV_HDR  := $(wildcard $(PKG)/csrc/*.cuh) $(wildcard $(PKG)/csrc/*.h) include/cadv.h
NVFLAGS   := -ccbin $(HOSTCXX) $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
             -Iinclude --expt-relaxed-constexpr -Xptxas -v

all: tracegen/libtracegen.so oracle/liboracle.so $(PKG)/libcadv.so $(PKG)/producer/libcadv_demo.so

tracegen/libtracegen.so: tracegen/tracegen.cpp
	$(HOSTCXX) -O2 -std=c++17 -fopenmp -shared -fPIC -o $@ $<

oracle/liboracle.so: oracle/oracle.cpp
	$(HOSTCXX) -O2 -std=c++17 -fopenmp -shared -fPIC -o $@ $<

$(PKG)/libcadv.so: $(CADV_SRC) $(CADV_HDR)
	$(NVCC) $(NVFLAGS) -shared -o $@ $(CADV_SRC) -ldl 2> $(PKG)/ptxas.log || (cat $(PKG)/ptxas.log; exit 1)

# hand-instrumented demo kernels (device-side trace producer, include/cadv_record.cuh)
$(PKG)/producer/libcadv_demo.so: $(PKG)/producer/demo_kernels.cu include/cadv_record.cuh
	$(NVCC) $(NVFLAGS) -shared -o $@ $< 2> $(PKG)/producer/ptxas.log || (cat $(PKG)/producer/ptxas.log; exit 1)

clean:
	rm -f tracegen/libtracegen.so oracle/liboracle.so $(PKG)/libcadv.so $(PKG)/producer/libcadv_demo.so

.PHONY: all clean
