# Build the CUDA product library and the CPU oracle (test infrastructure).
# `python -c "import __graft_entry__ as g; g.build()"` runs `make all`.

NVCC     ?= /usr/local/cuda/bin/nvcc
CXX      ?= g++
PKG      := paper_conf_icpp_liuwc21_b200
CSRC     := $(PKG)/csrc
LIB      := $(PKG)/libfastpso.so
ORACLE   := oracle/liboracle.so
NCCL_INC ?= $(shell python -c "import os, nvidia.nccl as m; print(os.path.join(list(m.__path__)[0], 'include'))" 2>/dev/null)

ARCH     := -gencode arch=compute_100a,code=sm_100a
NVFLAGS  := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O3,-Wall \
            -Xptxas -v -I include -I $(CSRC) $(if $(NCCL_INC),-I $(NCCL_INC) -DPSO_HAVE_NCCL_H=1,)
NVFLAGS  += $(EXTRA)
CU_SRCS  := $(wildcard $(CSRC)/*.cu)
CPP_SRCS := $(wildcard $(CSRC)/*.cpp)
HDRS     := $(wildcard $(CSRC)/*.cuh) $(wildcard $(CSRC)/*.h) include/fastpso.h

.PHONY: all lib oracle clean
all: oracle lib
lib: $(LIB)
oracle: $(ORACLE)

$(ORACLE): oracle/pso_oracle.cpp oracle/pso_oracle.h
	$(CXX) -O3 -std=c++17 -ffp-contract=off -fno-fast-math -fPIC -shared -Wall -o $@ $<

OBJDIR   := build/obj
CU_OBJS  := $(patsubst $(CSRC)/%.cu,$(OBJDIR)/%.o,$(CU_SRCS))
CPP_OBJS := $(patsubst $(CSRC)/%.cpp,$(OBJDIR)/%.o,$(CPP_SRCS))

$(OBJDIR)/%.o: $(CSRC)/%.cu $(HDRS)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -c -o $@ $< 2> $@.log || (cat $@.log; exit 1)

$(OBJDIR)/%.o: $(CSRC)/%.cpp $(HDRS)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -c -o $@ $< 2> $@.log || (cat $@.log; exit 1)

$(LIB): $(CU_OBJS) $(CPP_OBJS)
	$(NVCC) $(ARCH) -shared -o $@ $^ -ldl
	cat $(OBJDIR)/*.log > $(PKG)/build.log

clean:
	rm -rf $(LIB) $(ORACLE) $(PKG)/build.log $(OBJDIR)
