# Build everything in-tree (the .so files travel to the GPU box with gpurun).
#   graphgen : seeded input generators (test/bench infrastructure)
#   oracle   : plain single-threaded CPU oracle (test infrastructure only)
#   hec      : libhec.so, the sm_100a CUDA hot path behind the C-ABI (include/hec.h)
NVCC    ?= nvcc
CC      := gcc
CUDA    ?= /usr/local/cuda
PKG     := paper_conf_ipps_gilbertabmr21_b200
ARCH    := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
           --expt-relaxed-constexpr -Iinclude
CU_SRC  := $(wildcard $(PKG)/csrc/*.cu)
CU_OBJ  := $(patsubst $(PKG)/csrc/%.cu,build/%.o,$(CU_SRC))
CU_HDR  := $(wildcard $(PKG)/csrc/*.cuh) include/hec.h

all: graphgen oracle hec

graphgen: graphgen/libgraphgen.so
graphgen/libgraphgen.so: graphgen/graphgen.c
	$(CC) -O3 -march=x86-64-v2 -fopenmp -fPIC -shared -o $@ $<

oracle: oracle/liboracle.so
oracle/liboracle.so: oracle/oracle.c oracle/oracle.h
	$(CC) -O2 -std=c11 -Wall -Wextra -fPIC -shared -o $@ oracle/oracle.c

hec: $(PKG)/libhec.so
build/%.o: $(PKG)/csrc/%.cu $(CU_HDR) Makefile
	@mkdir -p build
	$(NVCC) $(NVFLAGS) -Xptxas -v -c -o $@ $< 2> build/$*.ptxas.log || (cat build/$*.ptxas.log; exit 1)
$(PKG)/libhec.so: $(CU_OBJ)
	$(NVCC) $(ARCH) -shared -o $@ $(CU_OBJ) -lcudart
	@cat build/*.ptxas.log > $(PKG)/ptxas.log

clean:
	rm -rf build graphgen/libgraphgen.so oracle/liboracle.so $(PKG)/libhec.so

.PHONY: all graphgen oracle hec clean

# A/B variants for timing experiments: make variant V=name VFLAGS="-DFOO=1"
# -> build/variants/<name>/libhec.so (load with HEC_LIB_PATH)
variant:
	@mkdir -p build/variants/$(V)
	$(NVCC) $(NVFLAGS) $(VFLAGS) -shared -o build/variants/$(V)/libhec.so $(CU_SRC) -lcudart
.PHONY: variant
