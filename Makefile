# Builds libbk.so (sm_100a CUDA + C++ runtime, C ABI), the oracle and the input generators.
NVCC   ?= nvcc
ARCH   := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := -std=c++17 -O3 -lineinfo $(ARCH) -Xcompiler -fPIC,-fvisibility=hidden -Xptxas -v
PKG    := paper_conf_ipps_mokhtaris14_b200
CSRC   := $(PKG)/csrc
OBJS   := build/kernels_stage.o build/kernels_compute.o build/kernels_partition.o build/kernels_baseline.o build/kernels_pattern.o build/kernels_kmer.o build/kernels_merge.o build/kernels_addr.o build/runtime_plan.o build/runtime_pipeline.o build/runtime_kernels.o build/runtime_api.o build/host_gather.o build/trace.o

all: $(PKG)/libbk.so oracle/libbkoracle.so gen/libbkgen.so baselines/libbkmt.so tests/user/libbkuser.so

build/%.o: $(CSRC)/%.cu $(CSRC)/bk_internal.cuh $(CSRC)/tma.cuh $(CSRC)/runtime.cuh $(CSRC)/host_gather.h $(CSRC)/trace.h include/bk.h
	@mkdir -p build
	$(NVCC) $(NVFLAGS) -c $< -o $@ 2> build/$*.ptxas.txt || (cat build/$*.ptxas.txt; false)

build/host_gather.o: $(CSRC)/host_gather.cpp $(CSRC)/host_gather.h $(CSRC)/bk_internal.cuh
	@mkdir -p build
	g++ -std=c++17 -O3 -march=x86-64-v3 -fPIC -fvisibility=hidden -Wall -I/usr/local/cuda/include -c $< -o $@

build/trace.o: $(CSRC)/trace.cpp $(CSRC)/trace.h
	@mkdir -p build
	g++ -std=c++17 -O2 -fPIC -fvisibility=hidden -Wall -I/usr/local/cuda/include -c $< -o $@

$(PKG)/libbk.so: $(OBJS)
	$(NVCC) -shared $(ARCH) -cudart static -o $@ $(OBJS) -lpthread -ldl

oracle/libbkoracle.so: oracle/oracle.c oracle/oracle.h
	gcc -O2 -ffp-contract=off -fPIC -shared -Wall -o $@ oracle/oracle.c -lm

gen/libbkgen.so: gen/gen.c gen/gen.h
	gcc -O2 -fopenmp -fPIC -shared -Wall -o $@ gen/gen.c -lm

# test-only user kernel for bk_run_user (a caller's own stage-4 kernel against include/bk.h)
tests/user/libbkuser.so: tests/user/user_kernels.cu include/bk.h
	$(NVCC) -std=c++17 -O3 $(ARCH) -Xcompiler -fPIC -shared -Iinclude -cudart static -o $@ $<

build/probe: tools/probe.cu
	@mkdir -p build
	$(NVCC) -O3 $(ARCH) -o $@ $<

clean:
	rm -rf build $(PKG)/libbk.so oracle/libbkoracle.so gen/libbkgen.so tests/user/libbkuser.so

.PHONY: all clean

baselines/libbkmt.so: baselines/cpu_mt.c
	gcc -O3 -march=x86-64-v3 -ffp-contract=off -fopenmp -fPIC -shared -o $@ $< -lm
