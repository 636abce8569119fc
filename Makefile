# Builds every native artefact in-tree (the .so files travel to the GPU box
# with the gpurun snapshot).  `__graft_entry__.build()` runs `make`.
#
#   oracle/liboracle.so   CPU oracle (test infrastructure only)
#   synth/libsynth.so     seeded synthetic frames (tests + bench)
#   paper_conf_icpp_fanjzac15_b200/libsharp.so   the product: sm_100a kernels + C ABI

NVCC     ?= /usr/local/cuda/bin/nvcc
CUDA_HOME ?= /usr/local/cuda
HOSTCC   := /usr/bin/gcc
PKG      := paper_conf_icpp_fanjzac15_b200
ARCH     := -gencode arch=compute_100a,code=sm_100a

ORACLE_CFLAGS := -std=c11 -O2 -ffp-contract=off -fno-fast-math -fopenmp -fPIC -shared -Wall -Wextra
SYNTH_CFLAGS  := -std=c11 -O2 -fopenmp -fPIC -shared -Wall -Wextra

# --fmad=false: no implicit FMA contraction; every fused multiply-add in the
# kernels is an explicit __fmaf_rn / fma.rn (bit-exact parity, R15).
NVCC_FLAGS := $(ARCH) -O3 -lineinfo -std=c++17 --fmad=false -Xptxas -v \
              -Xcompiler -fPIC,-O2,-Wall -I include -I $(PKG)/csrc $(EXTRA_NVCC_FLAGS)

SHARP_SRCS := $(wildcard $(PKG)/csrc/*.cu) $(wildcard $(PKG)/csrc/*.cpp)
SHARP_HDRS := $(wildcard $(PKG)/csrc/*.cuh) $(wildcard $(PKG)/csrc/*.h) include/sharp.h

all: oracle/liboracle.so synth/libsynth.so $(PKG)/libsharp.so tests/c_abi_check

oracle/liboracle.so: oracle/oracle.c oracle/oracle.h
	$(HOSTCC) $(ORACLE_CFLAGS) -o $@ oracle/oracle.c -lm

synth/libsynth.so: synth/synth.c
	$(HOSTCC) $(SYNTH_CFLAGS) -o $@ synth/synth.c

$(PKG)/libsharp.so: $(SHARP_SRCS) $(SHARP_HDRS)
	$(NVCC) $(NVCC_FLAGS) -shared -o $@ $(SHARP_SRCS) 2> build/ptxas.log || (cat build/ptxas.log; false)

# The C ABI used from plain C (tests/test_gpu_c_abi.py runs it); links the
# oracle and the synthetic-input generator as test infrastructure.
tests/c_abi_check: tests/c_abi_check.c include/sharp.h oracle/oracle.h oracle/liboracle.so synth/libsynth.so $(PKG)/libsharp.so
	$(HOSTCC) -std=c11 -O2 -Wall -Wextra -I include -I $(CUDA_HOME)/include -o $@ tests/c_abi_check.c \
	  -L $(PKG) -lsharp -L oracle -loracle -L synth -lsynth -L $(CUDA_HOME)/lib64 -lcudart \
	  -Wl,-rpath,'$$ORIGIN/../$(PKG)' -Wl,-rpath,'$$ORIGIN/../oracle' -Wl,-rpath,'$$ORIGIN/../synth' \
	  -Wl,-rpath,$(CUDA_HOME)/lib64

$(shell mkdir -p build)

clean:
	rm -f oracle/liboracle.so synth/libsynth.so $(PKG)/libsharp.so tests/c_abi_check

.PHONY: all clean
