# Build everything in-tree (the .so files travel to the GPU box with the gpurun snapshot).
NVCC      ?= nvcc
CC        := gcc
CXX       := g++
ARCH      := -gencode arch=compute_100a,code=sm_100a
NVFLAGS   := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fopenmp --expt-relaxed-constexpr
CFLAGS    := -O3 -fPIC -fopenmp -Wall -Wextra -std=c11
PKG       := paper_conf_icde_xing0wxl23_b200
CSRC      := $(PKG)/csrc

LT_CU     := $(wildcard $(CSRC)/*.cu)
LT_CPP    := $(wildcard $(CSRC)/*.cpp)
LT_H      := $(wildcard $(CSRC)/*.h $(CSRC)/*.cuh) include/lt.h

all: inputs oracle lt tools

tools: tools/gather_bench

tools/gather_bench: tools/gather_bench.cu
	$(NVCC) $(ARCH) -O3 -lineinfo $< -o $@

inputs: lt_inputs/libltgen.so
oracle: oracle/liboracle.so
lt: $(PKG)/liblt.so

lt_inputs/rmat_cpu.o: lt_inputs/rmat_cpu.c lt_inputs/ltgen.h lt_inputs/ltgen_common.h
	$(CC) $(CFLAGS) -c $< -o $@

lt_inputs/rmat_gpu.o: lt_inputs/rmat_gpu.cu lt_inputs/ltgen.h lt_inputs/ltgen_common.h
	$(NVCC) $(NVFLAGS) -c $< -o $@

lt_inputs/libltgen.so: lt_inputs/rmat_cpu.o lt_inputs/rmat_gpu.o
	$(NVCC) $(ARCH) -shared -Xcompiler -fopenmp $^ -o $@ -lgomp

# The oracle is plain C and shares nothing with the CUDA path (test infrastructure only).
oracle/liboracle.so: oracle/oracle.c oracle/oracle.h
	$(CC) -O2 -fPIC -fopenmp -Wall -Wextra -std=c11 -shared $< -o $@

$(CSRC)/%.o: $(CSRC)/%.cu $(LT_H)
	$(NVCC) $(NVFLAGS) -Iinclude -Xptxas -v -c $< -o $@ 2> $@.ptxas.txt || (cat $@.ptxas.txt; false)

$(CSRC)/%.o: $(CSRC)/%.cpp $(LT_H)
	$(CXX) -O3 -fPIC -std=c++17 -Wall -Wextra -Iinclude -I/usr/local/cuda/include -c $< -o $@

$(PKG)/liblt.so: $(LT_CU:.cu=.o) $(LT_CPP:.cpp=.o)
	$(NVCC) $(ARCH) -shared $^ -o $@ -ldl

# Experiment builds of liblt.so with compile-time switches (tools/variants/ is not shipped product):
#   make variant VTAG=nohint VDEFS="-DLT_PATH_HINT=0 -DLT_VIS_HINT=0"; run with LT_LIBRARY=tools/variants/liblt_nohint.so
variant: $(LT_CPP:.cpp=.o)
	mkdir -p tools/variants
	$(NVCC) $(NVFLAGS) $(VDEFS) -Iinclude -c $(CSRC)/lt_kernels.cu -o tools/variants/lt_kernels_$(VTAG).o
	$(NVCC) $(ARCH) -shared tools/variants/lt_kernels_$(VTAG).o $(LT_CPP:.cpp=.o) -o tools/variants/liblt_$(VTAG).so -ldl

clean:
	rm -f tools/gather_bench lt_inputs/*.o lt_inputs/*.so oracle/*.so $(CSRC)/*.o $(CSRC)/*.ptxas.txt $(PKG)/*.so

.PHONY: all inputs oracle lt tools clean variant
