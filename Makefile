# Build every native artefact in-tree (the .so files travel to the GPU box with gpurun).
NVCC     ?= nvcc
ARCH     := -gencode arch=compute_100a,code=sm_100a
NVFLAGS  := -O3 -std=c++17 $(ARCH) -lineinfo -Xcompiler -fPIC -Xptxas -v --expt-relaxed-constexpr -ftz=false -prec-div=true -prec-sqrt=true
PKG      := paper_conf_ipps_jim11_b200
CSRC     := $(PKG)/csrc
CU_SRCS  := $(wildcard $(CSRC)/*.cu)
CPP_SRCS := $(wildcard $(CSRC)/*.cpp)
HDRS     := $(wildcard $(CSRC)/*.cuh) $(wildcard $(CSRC)/*.h) include/bmr.h
# nccl.h of the NCCL torch bundles (libnccl.so.2 itself is loaded at run time, csrc/comm.cu)
NCCL_INC ?= $(shell python3 -c "import nvidia.nccl, os; print(os.path.join(list(nvidia.nccl.__path__)[0], 'include'))" 2>/dev/null || echo /usr/include)
OBJS     := $(patsubst $(CSRC)/%.cu,build/%.o,$(CU_SRCS)) $(patsubst $(CSRC)/%.cpp,build/%.cpp.o,$(CPP_SRCS))

all: gen/libbmrgen.so oracle/liboracle.so gen/libbmrgen_cuda.so $(PKG)/libbmr.so

gen/libbmrgen.so: gen/gen_host.c gen/bmr_gen.h
	gcc -O2 -fPIC -shared -Wall -Wextra -o $@ gen/gen_host.c -lpthread -lm

oracle/liboracle.so: oracle/oracle.cpp
	g++ -O3 -std=c++17 -fPIC -shared -ffp-contract=off -Wall -Wextra -o $@ oracle/oracle.cpp

gen/libbmrgen_cuda.so: gen/gen_device.cu gen/bmr_gen.h
	$(NVCC) -O3 $(ARCH) -Xcompiler -fPIC -shared -o $@ gen/gen_device.cu

build/%.o: $(CSRC)/%.cu $(HDRS)
	@mkdir -p build
	$(NVCC) $(NVFLAGS) -Iinclude -I$(NCCL_INC) -c -o $@ $< 2> build/$*.ptxas.txt || (cat build/$*.ptxas.txt; false)

build/%.cpp.o: $(CSRC)/%.cpp $(HDRS)
	@mkdir -p build
	$(NVCC) -O2 -std=c++17 -Xcompiler -fPIC -Iinclude -c -o $@ $<

$(PKG)/libbmr.so: $(OBJS)
	$(NVCC) $(ARCH) -shared --cudart static -o $@ $(OBJS) -ldl

clean:
	rm -rf build gen/*.so oracle/*.so $(PKG)/*.so

.PHONY: all clean
