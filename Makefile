# Builds libmars.so (sm_100a CUDA kernels + C ABI) in-tree and the CPU oracle.
NVCC ?= /usr/local/cuda/bin/nvcc
PKG := paper_conf_icpp_lancl21_b200
SRC := $(PKG)/csrc
LIB := $(PKG)/libmars.so
CU := $(wildcard $(SRC)/*.cu)
OBJ := $(patsubst $(SRC)/%.cu,build/obj/%.o,$(CU))
HDR := $(wildcard $(SRC)/*.cuh) include/mars.h
ARCH := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
           -Xptxas -warn-spills -I include -DMARS_BUILD

all: $(LIB) oracle/liboracle.so oracle/liboracle_omp.so

build/obj/%.o: $(SRC)/%.cu $(HDR)
	@mkdir -p build/obj
	$(NVCC) $(NVFLAGS) -c $< -o $@

$(LIB): $(OBJ)
	$(NVCC) $(ARCH) -shared -o $@ $(OBJ) -ldl -lpthread -lrt

oracle/liboracle.so: oracle/mars_oracle.c
	gcc -O2 -std=c11 -fPIC -shared -fno-fast-math -ffp-contract=off -o $@ $< -lm

# the same source with -fopenmp: bench.py's multi-core cpu_baseline (bitwise = serial)
oracle/liboracle_omp.so: oracle/mars_oracle.c
	gcc -O2 -std=c11 -fPIC -shared -fno-fast-math -ffp-contract=off -fopenmp -o $@ $< -lm

clean:
	rm -rf build/obj $(LIB) oracle/liboracle.so oracle/liboracle_omp.so

.PHONY: all clean
