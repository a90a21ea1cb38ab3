# Build everything in-tree (the .so files travel to the GPU box with gpurun).
#   gen/libgnngen.so                       seeded input generators (shared by both sides)
#   oracle/liboracle.so                    fp64 CPU oracle (test infrastructure only)
#   paper_conf_ipps_fanwc23_b200/libgnnsparse.so   the product: C-ABI + sm_100a kernels
# Translation units compile to objects in parallel (make -j), then link once.
NVCC    ?= /usr/local/cuda/bin/nvcc
HOSTCC  ?= /usr/bin/gcc
PKG     := paper_conf_ipps_fanwc23_b200
ARCH    := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := -ccbin /usr/bin/g++ $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC \
           -Xcompiler -fvisibility=hidden -Iinclude --expt-relaxed-constexpr -Xptxas -v
GITSHA  := $(shell git -C $(CURDIR) rev-parse --short=12 HEAD 2>/dev/null || echo unknown)$(shell git -C $(CURDIR) diff --quiet HEAD -- $(PKG)/csrc include 2>/dev/null || echo +dirty)
CUSRC   := $(wildcard $(PKG)/csrc/*.cu) $(wildcard $(PKG)/csrc/*.cpp)
CUHDR   := $(wildcard $(PKG)/csrc/*.cuh) include/gnn_sparse.h
OBJDIR  := $(if $(TAG),/tmp/gnn_obj_$(TAG),build/obj)
OBJS    := $(patsubst $(PKG)/csrc/%,$(OBJDIR)/%.o,$(CUSRC))

all: gen/libgnngen.so oracle/liboracle.so $(PKG)/libgnnsparse.so

gen/libgnngen.so: gen/gen.c gen/gen.h
	$(HOSTCC) -O3 -fopenmp -fPIC -shared -o $@ gen/gen.c -lm

# no fast-math, no FMA contraction: the oracle must round exactly as written
oracle/liboracle.so: oracle/oracle.c oracle/oracle.h
	$(HOSTCC) -O2 -ffp-contract=off -fno-fast-math -fopenmp -fPIC -shared -o $@ oracle/oracle.c -lm

$(OBJDIR)/%.o: $(PKG)/csrc/% $(CUHDR)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) $(DEFS) -c -o $@ $< 2> $@.ptxas.log || (cat $@.ptxas.log; exit 1)

# the version string carries the commit; rebuilt whenever HEAD moves
$(OBJDIR)/util.cu.o: $(PKG)/csrc/util.cu $(CUHDR) .git/HEAD $(wildcard .git/refs/heads/*)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) $(DEFS) -DGNN_GIT_SHA='"$(GITSHA)"' -c -o $@ $< 2> $@.ptxas.log || (cat $@.ptxas.log; exit 1)

$(PKG)/libgnnsparse.so: $(OBJS)
	$(NVCC) $(ARCH) -shared -cudart static -o $@ $(OBJS)
	cat $(OBJDIR)/*.ptxas.log > $(PKG)/ptxas.log

# tuning variants: make -j variant TAG=x DEFS="-DGNN_SPMM_REGS=80 ..." -> variants/libgnnsparse_x.so
# (variants/ travels to the GPU box; build/ does not)
variant: $(OBJS)
	@mkdir -p variants build
	$(NVCC) $(ARCH) -shared -cudart static -o variants/libgnnsparse_$(TAG).so $(OBJS)
	cat $(OBJDIR)/*.ptxas.log > build/ptxas_$(TAG).log

# measurement probes (tools/microbench.py), not part of the product
micro: variants/libgnnmicro.so
variants/libgnnmicro.so: tools/microbench.cu
	@mkdir -p variants
	$(NVCC) $(ARCH) -O3 -shared -Xcompiler -fPIC -o $@ $<

# lane-mapping experiment (tools/interleaved_ab.py), not part of the product
exp: variants/libgnnexp.so
variants/libgnnexp.so: tools/spmm_interleaved.cu $(PKG)/csrc/device.cuh
	@mkdir -p variants
	$(NVCC) $(ARCH) -O3 -std=c++17 -shared -Xcompiler -fPIC -Iinclude -o $@ $<

# SM-local traversal experiment (tools/locality_probe.py), not part of the product
locprobe: variants/liblocprobe.so
variants/liblocprobe.so: tools/locality_probe.cu
	@mkdir -p variants
	$(NVCC) $(ARCH) -O3 -lineinfo -shared -Xcompiler -fPIC -Xptxas -v -o $@ $<

clean:
	rm -rf gen/libgnngen.so oracle/liboracle.so $(PKG)/libgnnsparse.so build/obj*

.PHONY: all clean variant micro exp locprobe
