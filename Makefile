# Build everything in-tree (the .so files travel to the GPU box with the gpurun snapshot).
#   make synth   -> synth/_synth.so          (input generators, host-only, g++/OpenMP)
#   make dgcl    -> $(PKG)/libdgcl.so        (C-ABI library: planner + runtime + sm_100a kernels)
PKG      := paper_conf_eurosys_cai0wmcy21_b200
CUDA     ?= /usr/local/cuda
NVCC     ?= $(CUDA)/bin/nvcc
CXX      := $(shell test -x /usr/bin/g++ && echo /usr/bin/g++ || echo g++)
GENCODE  := -gencode arch=compute_100a,code=sm_100a
NVFLAGS  := -O3 -std=c++17 $(GENCODE) -lineinfo -Xcompiler -fPIC -Xcompiler -Wall -Iinclude
CXXFLAGS := -O3 -std=c++17 -fPIC -fopenmp -Wall -Wextra -Iinclude -I$(CUDA)/include

CSRC     := $(PKG)/csrc
HOST_SRC := $(CSRC)/planner.cpp $(CSRC)/lowering.cpp $(CSRC)/api.cpp $(CSRC)/hostsim.cpp
HOST_OBJ := $(patsubst $(CSRC)/%.cpp,build/%.o,$(HOST_SRC))
CU_SRC   := $(CSRC)/executor.cu $(CSRC)/executor_tma.cu
CU_OBJ   := build/executor.o build/executor_tma.o
HDRS     := include/dgcl.h $(wildcard $(CSRC)/*.h) $(wildcard $(CSRC)/*.cuh)

.PHONY: all synth dgcl clean
all: synth dgcl
synth: synth/_synth.so
dgcl: $(PKG)/libdgcl.so

synth/_synth.so: synth/csrc/synth.cpp
	$(CXX) -O3 -std=c++17 -fPIC -shared -fopenmp -Wall $< -o $@

build/%.o: $(CSRC)/%.cpp $(HDRS)
	@mkdir -p build
	$(CXX) $(CXXFLAGS) -c $< -o $@

build/%.o: $(CSRC)/%.cu $(HDRS)
	@mkdir -p build
	$(NVCC) $(NVFLAGS) -Xptxas -v -c $< -o $@ 2> build/$*.ptxas.log || (cat build/$*.ptxas.log; false)

$(PKG)/libdgcl.so: $(HOST_OBJ) $(CU_OBJ)
	$(NVCC) $(GENCODE) -shared -Xcompiler -fPIC -Xcompiler -fopenmp -cudart static $^ -o $@

clean:
	rm -rf build synth/_synth.so $(PKG)/libdgcl.so
