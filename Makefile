# Builds the three in-tree shared libraries (called by __graft_entry__.build()).
#   paper_conf_sigmod_merajispcksygnk16_b200/libblugby.so  — the product (C ABI, sm_100a kernels)
#   blugen/libblugen.so                                    — seeded input generator (host + device)
#   oracle/liboracle.so                                    — the CPU oracle (test infrastructure)
NVCC      ?= /usr/local/cuda/bin/nvcc
CXX       ?= g++
ARCH      := -gencode arch=compute_100a,code=sm_100a
NVFLAGS   := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -Wall -Iinclude \
             -Xptxas -warn-spills --expt-relaxed-constexpr
PKG       := paper_conf_sigmod_merajispcksygnk16_b200
CSRC      := $(PKG)/csrc
BLUGBY_SRCS := $(wildcard $(CSRC)/*.cu) $(wildcard $(CSRC)/*.cpp)
BLUGBY_HDRS := $(wildcard $(CSRC)/*.cuh) $(wildcard $(CSRC)/*.h) include/blu_gby.h $(CSRC)/jit_sources.h

all: $(PKG)/libblugby.so blugen/libblugen.so oracle/liboracle.so

# the NVRTC-specialised kernels are compiled at run time from the same device sources (jit.cpp)
$(CSRC)/jit_sources.h: $(CSRC)/blu_params.h $(CSRC)/blu_device.cuh tools/embed_sources.py
	python3 tools/embed_sources.py $@ $(CSRC)/blu_params.h $(CSRC)/blu_device.cuh

$(PKG)/libblugby.so: $(BLUGBY_SRCS) $(BLUGBY_HDRS)
	$(NVCC) $(NVFLAGS) -shared -o $@ $(BLUGBY_SRCS) -ldl

blugen/libblugen.so: blugen/csrc/gen.cu include/blu_gen.h
	$(NVCC) $(NVFLAGS) -shared -o $@ blugen/csrc/gen.cu

oracle/liboracle.so: oracle/blu_oracle.cpp oracle/sort_oracle.cpp include/blu_gen.h
	$(CXX) -O2 -std=c++17 -fPIC -shared -Wall -Iinclude -o $@ oracle/blu_oracle.cpp oracle/sort_oracle.cpp

clean:
	rm -f $(PKG)/libblugby.so blugen/libblugen.so oracle/liboracle.so

.PHONY: all clean
