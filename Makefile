# Build everything in-tree (the .so files travel to the GPU box with gpurun).
#   make            -> generators, oracle, CUDA library
#   make host       -> generators + oracle only (no nvcc)
PY      ?= python
NVCC    ?= /usr/local/cuda/bin/nvcc
CC      := gcc
PKG     := paper_conf_icpp_wrightdtcc23_b200
CSRC    := $(PKG)/csrc
NCCL_DIR := $(shell $(PY) -c "import nvidia.nccl,os;print(os.path.dirname(nvidia.nccl.__file__) if nvidia.nccl.__file__ else list(nvidia.nccl.__path__)[0])" 2>/dev/null)
ARCH    := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := -O3 -std=c++17 $(ARCH) -lineinfo -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
           -Iinclude -I$(CSRC) -I$(NCCL_DIR)/include --expt-relaxed-constexpr
NVLINK  := -shared -cudart static -L$(NCCL_DIR)/lib -l:libnccl.so.2 \
           -Xlinker -rpath,$(NCCL_DIR)/lib

CU_SRCS := $(wildcard $(CSRC)/*.cu)
CU_OBJS := $(patsubst $(CSRC)/%.cu,build/%.o,$(CU_SRCS))
CU_HDRS := $(wildcard $(CSRC)/*.cuh $(CSRC)/*/*.cuh $(CSRC)/*.h include/*.h)

all: host $(PKG)/libnest.so

host: nestgen/libnestgen.so oracle/liboracle.so

nestgen/libnestgen.so: nestgen/nestgen.c
	$(CC) -O2 -fopenmp -fPIC -shared -o $@ $<

# The oracle: plain C, no FMA contraction, no fast-math; single-threaded except
# oracle_spmv_csr_f64_threads (OpenMP over rows, the all-cores CPU baseline).
oracle/liboracle.so: oracle/oracle.c
	$(CC) -O2 -ffp-contract=off -fno-fast-math -fopenmp -fPIC -shared -o $@ $< -lm

build/%.o: $(CSRC)/%.cu $(CU_HDRS)
	@mkdir -p build
	$(NVCC) $(NVFLAGS) -c $< -o $@

$(PKG)/libnest.so: $(CU_OBJS)
	$(NVCC) $(ARCH) $(NVLINK) -o $@ $(CU_OBJS)

# the C ABI from plain C (examples/spmv_c.c): gcc + libnest.so + the CUDA runtime
examples/spmv_c: examples/spmv_c.c include/nest.h $(PKG)/libnest.so
	$(CC) -O2 -Wall -Iinclude -I/usr/local/cuda/include -o $@ $< -L$(PKG) -lnest \
	    -Wl,-rpath,'$$ORIGIN/../$(PKG)' -L/usr/local/cuda/lib64 -lcudart -Wl,-rpath,/usr/local/cuda/lib64

clean:
	rm -rf build nestgen/libnestgen.so oracle/liboracle.so $(PKG)/libnest.so examples/spmv_c

.PHONY: all host clean
