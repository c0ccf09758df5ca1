# Build of the native pieces.  `python -c "import __graft_entry__ as g; g.build()"` runs this.
NVCC    ?= nvcc
ARCH    := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xptxas -v -Iinclude
PKG     := paper_conf_icpp_liupw25_b200
SRCS    := $(wildcard $(PKG)/csrc/*.cu)
HDRS    := $(wildcard $(PKG)/csrc/*.cuh) include/gbdtmo.h
OBJS    := $(patsubst $(PKG)/csrc/%.cu,build/%.o,$(SRCS))

all: $(PKG)/libgbdtmo.so oracle/liboracle.so gen/libgbdtgen.so gen/libgbdtgen_cuda.so tools/microbench/libgbdtmo_peaks.so

build/%.o: $(PKG)/csrc/%.cu $(HDRS)
	@mkdir -p build
	$(NVCC) $(NVFLAGS) -c -o $@ $< 2> build/$*.ptxas.log || (cat build/$*.ptxas.log; false)

$(PKG)/libgbdtmo.so: $(OBJS)
	$(NVCC) $(ARCH) -shared -o $@ $(OBJS) -lcudart

oracle/liboracle.so: oracle/oracle.c oracle/oracle.h
	gcc -O2 -fopenmp -fPIC -shared -ffp-contract=off -o $@ oracle/oracle.c -lm

gen/libgbdtgen.so: gen/gen.c gen/gen_rng.h
	gcc -O2 -fopenmp -fPIC -shared -ffp-contract=off -o $@ gen/gen.c

gen/libgbdtgen_cuda.so: gen/gen_cuda.cu gen/gen_rng.h
	$(NVCC) $(ARCH) -O3 -lineinfo -Xcompiler -fPIC -shared -o $@ gen/gen_cuda.cu

# same-run roofline denominators for bench.py (measurement only, not the product path)
tools/microbench/libgbdtmo_peaks.so: tools/microbench/peaks.cu
	$(NVCC) $(ARCH) -O3 -lineinfo -Xcompiler -fPIC -shared -o $@ $<

clean:
	rm -rf build $(PKG)/libgbdtmo.so oracle/liboracle.so gen/libgbdtgen.so gen/libgbdtgen_cuda.so tools/microbench/libgbdtmo_peaks.so

.PHONY: all clean
