# Builds the CUDA library (sm_100a), the native input generator, and the CPU
# oracle (test infrastructure; built so the checker exists, never linked into libbc).
NVCC ?= nvcc
PKG := paper_conf_sc_mclaughlinb14_b200
ARCH := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := -O3 -std=c++17 -lineinfo $(ARCH) -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
           -Iinclude -Xptxas -v
SRCS := $(PKG)/csrc/bc_api.cu $(PKG)/csrc/bc_kernels.cuh include/bc.h

all: $(PKG)/libbc.so $(PKG)/libgraphgen.so oracle/liboracle.so

$(PKG)/libbc.so: $(SRCS)
	$(NVCC) $(NVFLAGS) -shared -o $@ $(PKG)/csrc/bc_api.cu 2> $(PKG)/csrc/ptxas.log || (cat $(PKG)/csrc/ptxas.log; false)
	@grep -E "registers|spill" $(PKG)/csrc/ptxas.log | sed 's/^ptxas info    : //' | sort -u | head -20

$(PKG)/libgraphgen.so: $(PKG)/graphgen_native.c
	gcc -O2 -std=c99 -fPIC -shared -pthread -o $@ $<

oracle/liboracle.so: oracle/brandes_oracle.c
	gcc -O2 -std=c99 -fPIC -shared -pthread -o $@ $<

clean:
	rm -f $(PKG)/libbc.so $(PKG)/libgraphgen.so oracle/liboracle.so

.PHONY: all clean
