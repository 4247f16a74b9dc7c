# Build the product library (sm_100a CUDA + C++ host, C ABI in include/gsword.h)
# and the CPU oracle (plain C, test infrastructure only).
NVCC     ?= nvcc
ARCH     := -gencode arch=compute_100a,code=sm_100a
PKG      := paper_journals_pacmmod_yelsg24_b200
CSRC     := $(PKG)/csrc
LIB      := $(PKG)/libgsword.so
ORACLE   := oracle/liboracle.so
XFLAGS   ?=
NVFLAGS  := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O3,-pthread -Xptxas -v --expt-relaxed-constexpr $(XFLAGS)

all: $(LIB) $(ORACLE)

variant:
	$(NVCC) $(NVFLAGS) -shared -o $(OUT) $(CSRC)/gsword_kernels.cu $(CSRC)/gsword_host.cpp 2> $(OUT).ptxas.log || (cat $(OUT).ptxas.log; false)

$(LIB): $(CSRC)/gsword_kernels.cu $(CSRC)/gsword_host.cpp $(CSRC)/internal.h $(CSRC)/device_util.cuh include/gsword.h
	$(NVCC) $(NVFLAGS) -shared -o $@ $(CSRC)/gsword_kernels.cu $(CSRC)/gsword_host.cpp 2> build_ptxas.log || (cat build_ptxas.log; false)

$(ORACLE): oracle/oracle.c
	gcc -O2 -std=c11 -Wall -Wextra -shared -fPIC -pthread -o $@ $<

clean:
	rm -f $(LIB) $(ORACLE) build_ptxas.log

.PHONY: all clean variant
