# Build everything in-tree (the .so files travel to the GPU box with gpurun).
#   gen/libgnngen.so                       seeded input generators (shared by both sides)
#   oracle/liboracle.so                    fp64 CPU oracle (test infrastructure only)
#   paper_conf_ipps_fanwc23_b200/libgnnsparse.so   the product: C-ABI + sm_100a kernels
NVCC    ?= /usr/local/cuda/bin/nvcc
HOSTCC  ?= /usr/bin/gcc
PKG     := paper_conf_ipps_fanwc23_b200
ARCH    := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := -ccbin /usr/bin/g++ $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
           -Iinclude --expt-relaxed-constexpr -Xptxas -v
CUSRC   := $(wildcard $(PKG)/csrc/*.cu) $(wildcard $(PKG)/csrc/*.cpp)
CUHDR   := $(wildcard $(PKG)/csrc/*.cuh) include/gnn_sparse.h

all: gen/libgnngen.so oracle/liboracle.so $(PKG)/libgnnsparse.so

gen/libgnngen.so: gen/gen.c gen/gen.h
	$(HOSTCC) -O3 -fopenmp -fPIC -shared -o $@ gen/gen.c -lm

# no fast-math, no FMA contraction: the oracle must round exactly as written
oracle/liboracle.so: oracle/oracle.c oracle/oracle.h
	$(HOSTCC) -O2 -ffp-contract=off -fno-fast-math -fPIC -shared -o $@ oracle/oracle.c -lm

$(PKG)/libgnnsparse.so: $(CUSRC) $(CUHDR)
	$(NVCC) $(NVFLAGS) -shared -cudart static -o $@ $(CUSRC) 2> $(PKG)/ptxas.log || (cat $(PKG)/ptxas.log; exit 1)

# tuning variants: make variant TAG=x DEFS="-DGNN_SPMM_MINB=2 ..."  ->  build/libgnnsparse_x.so
variant: $(CUSRC) $(CUHDR)
	mkdir -p build
	$(NVCC) $(NVFLAGS) $(DEFS) -shared -cudart static -o build/libgnnsparse_$(TAG).so $(CUSRC) 2> build/ptxas_$(TAG).log || (cat build/ptxas_$(TAG).log; exit 1)

clean:
	rm -f gen/libgnngen.so oracle/liboracle.so $(PKG)/libgnnsparse.so

.PHONY: all clean variant
