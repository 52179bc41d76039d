# Builds the product library (CUDA, sm_100a) and the CPU oracle (test infra).
#   make            -> both
#   make lib        -> paper_conf_asplos_linzs23_b200/libdrgpum.so
#   make oracle     -> oracle/liboracle.so
NVCC      ?= /usr/local/cuda/bin/nvcc
CXX       ?= g++
ARCH      := -gencode arch=compute_100a,code=sm_100a
PKG       := paper_conf_asplos_linzs23_b200
CSRC      := $(PKG)/csrc
NVFLAGS   := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -O2 \
             -Xcompiler -fvisibility=hidden -Iinclude -Xptxas -v
LIB       := $(PKG)/libdrgpum.so
ORACLE    := oracle/liboracle.so
TRACEGEN  := tracegen/libtracegen.so

CU_SRCS   := $(wildcard $(CSRC)/*.cu)
CPP_SRCS  := $(wildcard $(CSRC)/*.cpp)
HDRS      := $(wildcard $(CSRC)/*.cuh) $(wildcard $(CSRC)/*.h) include/drgpum.h

all: lib oracle tracegen

lib: $(LIB)
oracle: $(ORACLE)
tracegen: $(TRACEGEN)

$(LIB): $(CU_SRCS) $(CPP_SRCS) $(HDRS)
	$(NVCC) $(NVFLAGS) -shared -o $@ $(CU_SRCS) $(CPP_SRCS) 2> build_ptxas.log || (cat build_ptxas.log; exit 1)

$(ORACLE): oracle/drgpum_oracle.cpp
	$(CXX) -O2 -std=c++17 -fPIC -shared -o $@ $<

# input generation on the device (C3-C5 at full size); not part of the library
$(TRACEGEN): tracegen/gen.cu
	$(NVCC) $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared -o $@ $<

clean:
	rm -f $(LIB) $(ORACLE) $(TRACEGEN) build_ptxas.log

.PHONY: all lib oracle tracegen clean
