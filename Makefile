# Builds every native artefact in-tree (the .so files travel to the GPU box
# with the gpurun snapshot; they are git-ignored).
#   oracle/liboracle.so                         plain C oracle (test infra)
#   kcgen/libkcgen.so                           input generator (host C + CUDA)
#   paper_conf_icde_ahmady0gcz23_b200/lib/libkcore.so   the C-ABI hot path
PY      ?= python
NVCC    ?= /usr/local/cuda/bin/nvcc
ARCH    := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -O3 --expt-relaxed-constexpr
NCCL_DIR := $(shell $(PY) -c "import nvidia.nccl,os;print(list(nvidia.nccl.__path__)[0])" 2>/dev/null)
PKG     := paper_conf_icde_ahmady0gcz23_b200

KCORE_SRC := $(wildcard $(PKG)/csrc/*.cu) $(wildcard $(PKG)/csrc/*.cuh) $(wildcard include/*.h)

all: oracle/liboracle.so kcgen/libkcgen.so $(PKG)/lib/libkcore.so $(PKG)/lib/libkcore_trace.so

oracle/liboracle.so: oracle/kcore_oracle.c
	gcc -O2 -std=c11 -shared -fPIC $< -o $@

kcgen/libkcgen.so: kcgen/csrc/kcgen_host.c kcgen/csrc/kcgen_device.cu kcgen/csrc/kcgen_rng.h kcgen/include/kcgen.h
	gcc -O2 -std=c11 -fPIC -c kcgen/csrc/kcgen_host.c -o kcgen/kcgen_host.o
	$(NVCC) $(NVFLAGS) -c kcgen/csrc/kcgen_device.cu -o kcgen/kcgen_device.o
	$(NVCC) $(ARCH) -shared kcgen/kcgen_host.o kcgen/kcgen_device.o -o $@ -lm
	rm -f kcgen/kcgen_host.o kcgen/kcgen_device.o

$(PKG)/lib/libkcore.so: $(KCORE_SRC)
	mkdir -p $(PKG)/lib
	$(NVCC) $(NVFLAGS) -Xptxas -v -Iinclude -I$(NCCL_DIR)/include -shared \
	    $(PKG)/csrc/kcore.cu $(PKG)/csrc/kcore_mg.cu $(PKG)/csrc/kcore_extract.cu $(PKG)/csrc/kcore_mpm.cu $(PKG)/csrc/kcore_testhooks.cu $(PKG)/csrc/kcore_mgd.cu -o $@ \
	    -L$(NCCL_DIR)/lib -l:libnccl.so.2 -Xlinker -rpath=$(NCCL_DIR)/lib 2> $(PKG)/lib/ptxas.log || (cat $(PKG)/lib/ptxas.log; false)

# the same library with the per-phase / per-CTA trace compiled in (tools/cta_trace.py)
$(PKG)/lib/libkcore_trace.so: $(KCORE_SRC)
	mkdir -p $(PKG)/lib
	$(NVCC) $(NVFLAGS) -DKC_TRACE=1 -Iinclude -I$(NCCL_DIR)/include -shared \
	    $(PKG)/csrc/kcore.cu $(PKG)/csrc/kcore_mg.cu $(PKG)/csrc/kcore_extract.cu $(PKG)/csrc/kcore_mpm.cu $(PKG)/csrc/kcore_testhooks.cu $(PKG)/csrc/kcore_mgd.cu -o $@ \
	    -L$(NCCL_DIR)/lib -l:libnccl.so.2 -Xlinker -rpath=$(NCCL_DIR)/lib

clean:
	rm -f oracle/liboracle.so kcgen/libkcgen.so $(PKG)/lib/libkcore.so $(PKG)/lib/libkcore_trace.so

.PHONY: all clean
