# Build everything in-tree (the .so files travel to the GPU box with gpurun).
#   make            -> libgts.so (CUDA, sm_100a) + oracle + input generators
PY       ?= python
PKG      := paper_conf_sigmod_0002apsk16_b200
CSRC     := $(PKG)/csrc
LIBDIR   := $(PKG)/lib
NVCC     ?= /usr/local/cuda/bin/nvcc
SITE     := $(shell $(PY) -c "import sysconfig;print(sysconfig.get_paths()['purelib'])")
NCCL_DIR := $(SITE)/nvidia/nccl
ARCH     := -gencode arch=compute_100a,code=sm_100a
NVFLAGS  := $(ARCH) -O3 -lineinfo -std=c++17 --expt-relaxed-constexpr -Xcompiler -fPIC,-fopenmp,-O3 \
            -Iinclude -I$(CSRC) -I$(NCCL_DIR)/include -Xptxas -v
CU_SRC   := $(CSRC)/context.cu $(CSRC)/comm.cu $(CSRC)/traverse.cu $(CSRC)/pagerank.cu $(CSRC)/wcc.cu
CPP_SRC  := $(CSRC)/builder.cpp $(CSRC)/capi.cpp
HDRS     := include/gts.h $(wildcard $(CSRC)/*.h) $(wildcard $(CSRC)/*.cuh)
OBJDIR   := build/obj
CU_OBJ   := $(patsubst $(CSRC)/%.cu,$(OBJDIR)/%.o,$(CU_SRC))
CPP_OBJ  := $(patsubst $(CSRC)/%.cpp,$(OBJDIR)/%.o,$(CPP_SRC))

all: $(LIBDIR)/libgts.so oracle/liboracle.so oracle/liboracle_omp.so inputs/libgtsgen.so

$(OBJDIR)/%.o: $(CSRC)/%.cu $(HDRS)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -c $< -o $@ 2> $@.ptxas.log || (cat $@.ptxas.log; false)

$(OBJDIR)/%.o: $(CSRC)/%.cpp $(HDRS)
	@mkdir -p $(OBJDIR)
	g++ -O3 -std=c++17 -fPIC -fopenmp -Iinclude -I$(CSRC) -I/usr/local/cuda/include -c $< -o $@

$(LIBDIR)/libgts.so: $(CU_OBJ) $(CPP_OBJ)
	@mkdir -p $(LIBDIR)
	$(NVCC) $(ARCH) -shared -o $@ $^ -Xcompiler -fopenmp -L$(NCCL_DIR)/lib -l:libnccl.so.2 \
	    -Xlinker -rpath,$(NCCL_DIR)/lib

oracle/liboracle.so: oracle/oracle.c
	gcc -O2 -fPIC -shared -o $@ $<

oracle/liboracle_omp.so: oracle/oracle.c
	gcc -O2 -fopenmp -fPIC -shared -o $@ $<

inputs/libgtsgen.so: inputs/gen.c
	gcc -O3 -march=x86-64-v2 -fopenmp -fPIC -shared -o $@ $< -lm

clean:
	rm -rf build $(LIBDIR) oracle/liboracle.so oracle/liboracle_omp.so inputs/libgtsgen.so

.PHONY: all clean
