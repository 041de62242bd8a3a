# Builds the three in-tree shared libraries (called by __graft_entry__.build()).
#   paper_conf_sigmod_merajispcksygnk16_b200/libblugby.so  — the product (C ABI, sm_100a kernels)
#   blugen/libblugen.so                                    — seeded input generator (host + device)
#   oracle/liboracle.so                                    — the CPU oracle (test infrastructure)
# Each libblugby source compiles to its own object (make -j builds them in parallel).
NVCC      ?= /usr/local/cuda/bin/nvcc
CXX       ?= g++
ARCH      := -gencode arch=compute_100a,code=sm_100a
NVFLAGS   := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -Wall -Iinclude \
             -Xptxas -warn-spills --expt-relaxed-constexpr
PKG       := paper_conf_sigmod_merajispcksygnk16_b200
CSRC      := $(PKG)/csrc
OBJDIR    := build/obj
BLUGBY_SRCS := $(wildcard $(CSRC)/*.cu) $(wildcard $(CSRC)/*.cpp)
BLUGBY_OBJS := $(patsubst $(CSRC)/%,$(OBJDIR)/%.o,$(BLUGBY_SRCS))
BLUGBY_HDRS := $(wildcard $(CSRC)/*.cuh) $(wildcard $(CSRC)/*.h) include/blu_gby.h include/blu_sort.h $(CSRC)/jit_sources.h
ORACLE_SRCS := oracle/blu_oracle.cpp oracle/sort_oracle.cpp oracle/kmv_oracle.cpp

all: $(PKG)/libblugby.so blugen/libblugen.so oracle/liboracle.so

# the NVRTC-specialised kernels are compiled at run time from the same device sources (jit.cpp)
$(CSRC)/jit_sources.h: $(CSRC)/blu_params.h $(CSRC)/blu_device.cuh tools/embed_sources.py
	python3 tools/embed_sources.py $@ $(CSRC)/blu_params.h $(CSRC)/blu_device.cuh

$(OBJDIR)/%.o: $(CSRC)/% $(BLUGBY_HDRS)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -x cu -c -o $@ $<

$(PKG)/libblugby.so: $(BLUGBY_OBJS)
	$(NVCC) $(ARCH) -shared -o $@ $(BLUGBY_OBJS) -ldl

blugen/libblugen.so: blugen/csrc/gen.cu include/blu_gen.h
	$(NVCC) $(NVFLAGS) -shared -o $@ blugen/csrc/gen.cu

oracle/liboracle.so: $(ORACLE_SRCS) include/blu_gen.h
	$(CXX) -O2 -std=c++17 -fPIC -shared -Wall -Iinclude -o $@ $(ORACLE_SRCS)

clean:
	rm -rf $(PKG)/libblugby.so blugen/libblugen.so oracle/liboracle.so $(OBJDIR)

.PHONY: all clean
