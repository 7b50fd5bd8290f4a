# Build everything in-tree (the .so files travel to the GPU box with gpurun).
#   make            -> product library + test-infrastructure libraries
NVCC      ?= nvcc
ARCH      := -gencode arch=compute_100a,code=sm_100a
NVFLAGS   := -O3 -std=c++17 $(ARCH) -lineinfo -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
             -Xptxas -v --cudart static
PKG       := paper_conf_sc_mandulakgfhs24_b200
LIB       := $(PKG)/liblmatch.so
SRCS      := $(PKG)/csrc/lmatch.cu
HDRS      := $(PKG)/csrc/kernels.cuh include/lmatch.h

all: $(LIB) oracle/liboracle.so graphgen/libgraphgen.so graphgen/libgraphgen_cuda.so

$(LIB): $(SRCS) $(HDRS)
	$(NVCC) $(NVFLAGS) -shared -Xlinker --exclude-libs=ALL $(SRCS) -o $@.tmp 2> $(PKG)/build.log || (cat $(PKG)/build.log; rm -f $@.tmp; exit 1)
	mv $@.tmp $@

# test infrastructure (never linked into the product)
oracle/liboracle.so: oracle/oracle.cpp
	g++ -O2 -std=c++17 -fopenmp -fPIC -shared $< -o $@

graphgen/libgraphgen.so: graphgen/graphgen.cpp graphgen/gg_common.h
	g++ -O3 -march=x86-64-v3 -ffp-contract=off -std=c++17 -fopenmp -fPIC -shared $< -o $@

sass: $(LIB)
	cuobjdump -sass $(LIB) > $(PKG)/liblmatch.sass

clean:
	rm -f $(LIB) oracle/liboracle.so graphgen/libgraphgen.so $(PKG)/build.log

.PHONY: all clean sass

graphgen/libgraphgen_cuda.so: graphgen/graphgen_cuda.cu graphgen/gg_common.h
	$(NVCC) -O3 -std=c++17 -fmad=false $(ARCH) -Xcompiler -fPIC -shared $< -o $@

# builder tooling (not product): TMA read-stream microbenchmark, built on demand
scripts/microbench_stream: scripts/microbench_stream.cu $(PKG)/csrc/kernels.cuh
	$(NVCC) -O3 -std=c++17 $(ARCH) -lineinfo $< -o $@
