# Build every native artefact in-tree (the .so files travel to the GPU box with gpurun).
#   gen/libfgrgen.so                               seeded workload generator (C, shared plumbing)
#   oracle/liboracle.so                            plain CPU oracle (C, test infrastructure only)
#   paper_conf_date_liulzclly22_b200/libfastgr.so  the product: CUDA kernels + C ABI (sm_100a)
PY      ?= python
NVCC    ?= /usr/local/cuda/bin/nvcc
CC      ?= gcc
SITE    := $(shell $(PY) -c "import nvidia.nccl,os;print(os.path.dirname(nvidia.nccl.__path__[0]))" 2>/dev/null)
NCCL_INC := $(SITE)/nccl/include
NCCL_LIB := $(SITE)/nccl/lib
PKG     := paper_conf_date_liulzclly22_b200
CSRC    := $(PKG)/csrc
ARCH    := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := $(EXTRA) -O3 -std=c++17 $(ARCH) -lineinfo -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
           -Iinclude -I$(NCCL_INC) --expt-relaxed-constexpr -Xptxas -v
CFLAGS  := -O2 -std=c11 -fPIC -Wall -Wextra -Wno-unused-parameter

KERN_SRC := $(wildcard $(CSRC)/*.cu)
KERN_HDR := $(wildcard $(CSRC)/*.cuh) include/fastgr.h
BUILD   ?= build
LIB     ?= $(PKG)/libfastgr.so
KERN_OBJ := $(patsubst $(CSRC)/%.cu,$(BUILD)/%.o,$(KERN_SRC))

all: gen/libfgrgen.so oracle/liboracle.so $(LIB)

gen/libfgrgen.so: gen/fgr_gen.c
	$(CC) $(CFLAGS) -shared -o $@ $< -lm

oracle/liboracle.so: oracle/fgr_oracle.c oracle/fgr_oracle.h
	$(CC) $(CFLAGS) -shared -o $@ oracle/fgr_oracle.c -lm

$(BUILD)/%.o: $(CSRC)/%.cu $(KERN_HDR)
	@mkdir -p $(BUILD)
	$(NVCC) $(NVFLAGS) -c -o $@ $< 2> $(BUILD)/$*.ptxas.txt || (cat $(BUILD)/$*.ptxas.txt; false)

$(LIB): $(KERN_OBJ)
	$(NVCC) $(ARCH) -shared -o $@ $(KERN_OBJ) -L$(NCCL_LIB) -l:libnccl.so.2 \
	    -Xlinker -rpath=$(NCCL_LIB) -Xcompiler -fPIC

clean:
	rm -rf build gen/libfgrgen.so oracle/liboracle.so $(PKG)/libfastgr.so

.PHONY: all clean
