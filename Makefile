# Builds every native artefact in-tree (the .so files travel to the GPU box).
#   paper_conf_ipps_kurtysps23_b200/lib/librdm.so   product: CUDA sm_100a + C ABI
#   synth/libsynth.so                                seeded input generators
#   oracle/liboracle.so                              CPU fp64 oracle (test infrastructure)
PY        ?= python
NVCC      ?= /usr/local/cuda/bin/nvcc
SITE      := $(shell $(PY) -c "import sysconfig;print(sysconfig.get_paths()['purelib'])")
NCCL_DIR  ?= $(SITE)/nvidia/nccl
ARCH      := -gencode arch=compute_100a,code=sm_100a
NVFLAGS   := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -Wall \
             -I$(NCCL_DIR)/include -Iinclude --expt-relaxed-constexpr -Xptxas -v
PKG       := paper_conf_ipps_kurtysps23_b200
SRC       := $(PKG)/csrc
OBJDIR    := build/obj
CU_SRCS   := $(wildcard $(SRC)/*.cu)
CPP_SRCS  := $(wildcard $(SRC)/*.cpp)
OBJS      := $(patsubst $(SRC)/%.cu,$(OBJDIR)/%.o,$(CU_SRCS)) $(patsubst $(SRC)/%.cpp,$(OBJDIR)/%.o,$(CPP_SRCS))
LIB       := $(PKG)/lib/librdm.so

all: $(LIB) synth/libsynth.so oracle/liboracle.so

$(OBJDIR)/%.o: $(SRC)/%.cu $(wildcard $(SRC)/*.h) include/rdm.h
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -c $< -o $@ 2> $@.log || (cat $@.log; false)

$(OBJDIR)/%.o: $(SRC)/%.cpp $(wildcard $(SRC)/*.h) include/rdm.h
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -x cu -c $< -o $@ 2> $@.log || (cat $@.log; false)

$(LIB): $(OBJS)
	@mkdir -p $(PKG)/lib
	$(NVCC) $(ARCH) -shared -o $@ $(OBJS) -L$(NCCL_DIR)/lib -l:libnccl.so.2 \
	    -Xlinker -rpath=$(NCCL_DIR)/lib

synth/libsynth.so: synth/gen.cpp
	g++ -O3 -fopenmp -fPIC -shared -std=c++17 $< -o $@

oracle/liboracle.so: oracle/spmm.c
	gcc -O2 -fopenmp -fPIC -shared -std=c11 $< -o $@

clean:
	rm -rf build $(LIB) synth/libsynth.so oracle/liboracle.so

.PHONY: all clean
