# Builds the three native libraries in-tree (the .so files travel to the GPU
# box with the gpurun snapshot; they are git-ignored).
#   paper_conf_isca_shaharbs16_b200/libapointer.so  -- the product (CUDA, sm_100a)
#   paper_conf_isca_shaharbs16_b200/libapointer_hash.so -- N4 ablation: hash-table page table
#   oracle/liboracle.so                             -- CPU oracle (test infrastructure)
#   synth/libsynth.so                               -- seeded input generators
NVCC    ?= /usr/local/cuda/bin/nvcc
HOSTCC  := $(shell test -x /usr/bin/gcc && echo /usr/bin/gcc || echo gcc)
PKG     := paper_conf_isca_shaharbs16_b200
CSRC    := $(PKG)/csrc
ARCH    := -gencode arch=compute_100a,code=sm_100a
# -rdc=true: the out-of-line fault path (deref_slow and friends) is called
# through the ABI, so values a hot loop keeps live across a possible fault stay
# in callee-saved registers and are saved only inside the fault path (a
# whole-program call made ptxas spill them at their definition, on the hit
# path).  -maxrregcount=64 sizes those ABI functions for every caller (the
# paper's 64 registers per thread); kernels keep their own
# __launch_bounds__ budgets.
NVFLAGS := -O3 -std=c++17 $(ARCH) -lineinfo -Xcompiler -fPIC -Xcompiler -Wall \
           -Iinclude -I$(CSRC) --expt-relaxed-constexpr -rdc=true -maxrregcount=64
CFLAGS  := -O2 -fopenmp -fPIC -Wall -Wextra -std=c11

CU_SRCS := $(wildcard $(CSRC)/*.cu)
CU_HDRS := $(wildcard $(CSRC)/*.cuh) $(wildcard include/*.h) $(wildcard include/ap/*.cuh)

all: synth/libsynth.so oracle/liboracle.so $(PKG)/libapointer.so $(PKG)/libapointer_hash.so \
     tools/atomic_ceiling

synth/libsynth.so: synth/synth.c
	$(HOSTCC) $(CFLAGS) -shared $< -o $@ -lm

oracle/liboracle.so: oracle/oracle.c
	$(HOSTCC) $(CFLAGS) -shared $< -o $@ -lm

$(PKG)/libapointer.so: $(CU_SRCS) $(CU_HDRS)
	$(NVCC) $(NVFLAGS) -shared $(CU_SRCS) -o $@ -lcuda

# N4 ablation: the paper's hash-table page table instead of the dense PTE array
$(PKG)/libapointer_hash.so: $(CU_SRCS) $(CU_HDRS)
	$(NVCC) $(NVFLAGS) -DAP_PT_HASH -shared $(CU_SRCS) -o $@ -lcuda

# the M2r ceiling (bench.py runs it in the same session as the kernels it bounds)
tools/atomic_ceiling: tools/atomic_ceiling.cu
	$(NVCC) -O3 $(ARCH) $< -o $@

host: synth/libsynth.so oracle/liboracle.so

sass: $(PKG)/libapointer.so
	/usr/local/cuda/bin/cuobjdump -sass $< > build_sass.txt

clean:
	rm -f synth/libsynth.so oracle/liboracle.so $(PKG)/libapointer.so $(PKG)/libapointer_hash.so \
	      tools/atomic_ceiling

.PHONY: all host clean sass
