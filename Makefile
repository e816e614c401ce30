# Build libtsg.so (sm_100a CUDA path) in-tree and liboracle.so (plain C, test infrastructure).
NVCC ?= nvcc
PKG := paper_conf_ppopp_niuljs0022_b200
SRC := $(wildcard $(PKG)/csrc/*.cu)
HDR := $(wildcard $(PKG)/csrc/*.cuh) include/tsg.h
ARCH := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-fvisibility=hidden -Iinclude --expt-relaxed-constexpr
OBJ := $(patsubst $(PKG)/csrc/%.cu,build/%.o,$(SRC))

all: $(PKG)/libtsg.so oracle/liboracle.so

build/%.o: $(PKG)/csrc/%.cu $(HDR)
	@mkdir -p build
	$(NVCC) $(NVFLAGS) $(EXTRA) -c $< -o $@

$(PKG)/libtsg.so: $(OBJ)
	$(NVCC) $(ARCH) -shared -o $@ $(OBJ) -lcudart

oracle/liboracle.so: oracle/tsg_oracle.c
	gcc -O2 -ffp-contract=off -fPIC -shared -std=c11 -fopenmp -o $@ $< -lm

ptxas: EXTRA = -Xptxas -v
ptxas: clean all

clean:
	rm -rf build $(PKG)/libtsg.so

.PHONY: all clean ptxas
