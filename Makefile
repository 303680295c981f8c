# Native build: every .so is built in-tree (they travel to the GPU box with gpurun).
#   graphgen/libgraphgen.so                 seeded input generators (CPU + CUDA)
#   oracle/liboracle.so                     plain-C CPU oracle (test infrastructure only)
#   paper_conf_sigmod_hu0l21_b200/libtc_b200.so   the product: C-ABI + sm_100a kernels
NVCC    ?= /usr/local/cuda/bin/nvcc
CC      ?= gcc
ARCH    := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -Wall -Xcompiler -ffp-contract=off \
           -Xptxas -v --expt-relaxed-constexpr
CFLAGS  := -O2 -std=c11 -fPIC -Wall -Wextra -ffp-contract=off

PKG := paper_conf_sigmod_hu0l21_b200
TC_SRCS := $(wildcard $(PKG)/csrc/*.cu)
TC_HDRS := $(wildcard $(PKG)/csrc/*.cuh) include/tc.h
TC_CPP  := $(wildcard $(PKG)/csrc/*.cpp)

all: graphgen/libgraphgen.so oracle/liboracle.so $(PKG)/libtc_b200.so

graphgen/libgraphgen.so: graphgen/graphgen_cpu.c graphgen/graphgen_cuda.cu graphgen/philox.h
	$(CC) $(CFLAGS) -c graphgen/graphgen_cpu.c -o graphgen/graphgen_cpu.o
	$(NVCC) $(ARCH) -O3 -Xcompiler -fPIC -c graphgen/graphgen_cuda.cu -o graphgen/graphgen_cuda.o
	$(NVCC) $(ARCH) -shared graphgen/graphgen_cpu.o graphgen/graphgen_cuda.o -o $@ -lpthread

oracle/liboracle.so: oracle/tc_oracle.c
	$(CC) $(CFLAGS) -pthread -shared oracle/tc_oracle.c -o $@ -lm

# one object per source (parallel make), then one shared library
TC_OBJS := $(patsubst $(PKG)/csrc/%.cu,build/%.o,$(TC_SRCS)) $(patsubst $(PKG)/csrc/%.cpp,build/%.cpp.o,$(TC_CPP))

build/%.o: $(PKG)/csrc/%.cu $(TC_HDRS) $(PKG)/csrc/internal.h $(PKG)/csrc/count_dev.cuh
	@mkdir -p build
	$(NVCC) $(NVFLAGS) -Iinclude -c $< -o $@ 2> build/$*.ptxas.log || (cat build/$*.ptxas.log; false)

build/%.cpp.o: $(PKG)/csrc/%.cpp $(TC_HDRS) $(PKG)/csrc/internal.h
	@mkdir -p build
	$(NVCC) $(NVFLAGS) -Iinclude -c $< -o $@

$(PKG)/libtc_b200.so: $(TC_OBJS)
	$(NVCC) $(ARCH) -shared $(TC_OBJS) -o $@ -ldl
	cat build/*.ptxas.log > $(PKG)/ptxas.log

clean:
	rm -rf build graphgen/*.o graphgen/*.so oracle/*.so $(PKG)/*.so

.PHONY: all clean
