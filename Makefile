# Build everything in-tree (the .so files travel to the GPU box with the gpurun snapshot).
#   make            -> inputs + oracle + product CUDA library
#   make inputs     -> inputs/libgen.so        (seeded edge-list generators)
#   make oracle     -> oracle/liboracle.so     (CPU oracle; test infrastructure)
#   make gum        -> paper_conf_icde_menggltyz23_b200/libgum.so (C ABI + sm_100a kernels)
PKG      := paper_conf_icde_menggltyz23_b200
CUDA     ?= /usr/local/cuda
NVCC     := $(CUDA)/bin/nvcc
ARCH     := -gencode arch=compute_100a,code=sm_100a
NVFLAGS  := -O3 -std=c++17 $(ARCH) -lineinfo -Xcompiler -fPIC,-fopenmp,-O3 -Xptxas -v \
            -Iinclude --expt-relaxed-constexpr
GUM_SRCS := $(wildcard $(PKG)/csrc/*.cu) $(wildcard $(PKG)/csrc/*.cpp)
GUM_HDRS := $(wildcard $(PKG)/csrc/*.h) $(wildcard $(PKG)/csrc/*.cuh) include/gum.h

all: inputs oracle gum linkbench

linkbench: tools/linkbench/liblinkbench.so

tools/linkbench/liblinkbench.so: tools/linkbench/linkbench.cu
	$(NVCC) -O3 -std=c++17 $(ARCH) -Xcompiler -fPIC -shared -o $@ $<

inputs: inputs/libgen.so
oracle: oracle/liboracle.so
gum: $(PKG)/libgum.so

inputs/libgen.so: inputs/gen.c
	gcc -O3 -fopenmp -shared -fPIC -o $@ $<

oracle/liboracle.so: oracle/oracle.c
	gcc -O2 -fopenmp -shared -fPIC -o $@ $< -lm

$(PKG)/libgum.so: $(GUM_SRCS) $(GUM_HDRS)
	$(NVCC) $(NVFLAGS) -shared -o $@ $(GUM_SRCS) -lgomp 2> build/ptxas.log || (cat build/ptxas.log; false)
	@grep -E "error|warning" build/ptxas.log || true

$(shell mkdir -p build)

clean:
	rm -f inputs/libgen.so oracle/liboracle.so $(PKG)/libgum.so tools/linkbench/liblinkbench.so

.PHONY: all inputs oracle gum linkbench clean
