# Build every native artefact in-tree (the .so files travel to the GPU box with
# the gpurun snapshot). `make` is what __graft_entry__.build() runs.
#
#   tpchgen/libtpchgen.so                         seeded input generator (shared by oracle + CUDA path)
#   oracle/liboracle.so                           CPU oracle (test infrastructure only)
#   paper_conf_sigmod_paulhh16_b200/lib/libgpl.so the product: C-ABI + sm_100a kernels

NVCC     ?= /usr/local/cuda/bin/nvcc
CXX      := g++
CC       := gcc
ARCH     := -gencode arch=compute_100a,code=sm_100a
PKG      := paper_conf_sigmod_paulhh16_b200
CSRC     := $(PKG)/csrc
LIBGPL   := $(PKG)/lib/libgpl.so

CU_SRCS  := $(wildcard $(CSRC)/*.cu)
CPP_SRCS := $(wildcard $(CSRC)/*.cpp)
HDRS     := $(wildcard $(CSRC)/*.h $(CSRC)/*.cuh) include/gpl.h
OBJDIR   := build
CU_OBJS  := $(patsubst $(CSRC)/%.cu,$(OBJDIR)/%.cu.o,$(CU_SRCS))
CPP_OBJS := $(patsubst $(CSRC)/%.cpp,$(OBJDIR)/%.cpp.o,$(CPP_SRCS))

NVCCFLAGS := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
             -Iinclude -I$(CSRC) --expt-relaxed-constexpr -Xptxas -warn-spills
CXXFLAGS  := -O2 -std=c++17 -fPIC -fvisibility=hidden -Iinclude -I$(CSRC) -I/usr/local/cuda/include -Wall

all: tpchgen/libtpchgen.so oracle/liboracle.so $(LIBGPL)

tpchgen/libtpchgen.so: tpchgen/tpchgen.c
	$(CC) -O2 -fopenmp -shared -fPIC -Wall -o $@ $<

oracle/liboracle.so: oracle/oracle.cpp
	$(CXX) -O2 -std=c++17 -shared -fPIC -Wall -o $@ $<

$(OBJDIR)/%.cu.o: $(CSRC)/%.cu $(HDRS)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVCCFLAGS) -c $< -o $@

$(OBJDIR)/%.cpp.o: $(CSRC)/%.cpp $(HDRS)
	@mkdir -p $(OBJDIR)
	$(CXX) $(CXXFLAGS) -c $< -o $@

JIT_HDRS := $(CSRC)/common.h $(CSRC)/device_common.cuh $(CSRC)/pipeline_body.cuh

$(OBJDIR)/jit_sources.cpp: $(JIT_HDRS) tools/embed_sources.py
	@mkdir -p $(OBJDIR)
	python3 tools/embed_sources.py $@ $(JIT_HDRS)

$(OBJDIR)/jit_sources.o: $(OBJDIR)/jit_sources.cpp
	$(CXX) $(CXXFLAGS) -c $< -o $@

$(LIBGPL): $(CU_OBJS) $(CPP_OBJS) $(OBJDIR)/jit_sources.o
	@mkdir -p $(PKG)/lib
	$(NVCC) $(ARCH) -shared -o $@ $^ -cudart static -lpthread -ldl -lrt

clean:
	rm -rf $(OBJDIR) tpchgen/libtpchgen.so oracle/liboracle.so $(LIBGPL)

.PHONY: all clean
