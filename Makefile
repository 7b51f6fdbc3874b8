# Builds the CUDA library (sm_100a), the native input generator, and the CPU
# oracle (test infrastructure; built so the checker exists, never linked into libbc).
NVCC ?= nvcc
PKG := paper_conf_sc_mclaughlinb14_b200
ARCH := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := -O3 -std=c++17 -lineinfo $(ARCH) -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
           -Iinclude -Xptxas -v
CSRC := $(PKG)/csrc
HDRS := $(CSRC)/bc_kernels.cuh $(CSRC)/bc_fast.cuh $(CSRC)/bc_batch.cuh $(CSRC)/bc_group.cuh include/bc.h
# one translation unit per level store (compiled in parallel: make -j)
UNITS := bc_api bc_batch bc_group bc_inst_directed bc_inst_levels bc_inst_gcodes bc_inst_scodes
OBJS := $(UNITS:%=build/%.o)

all: $(PKG)/libbc.so $(PKG)/libgraphgen.so $(PKG)/libbcprobe.so oracle/liboracle.so

build/%.o: $(CSRC)/%.cu $(HDRS)
	@mkdir -p build
	$(NVCC) $(NVFLAGS) -c -o $@ $< 2> build/$*.ptxas.log || (cat build/$*.ptxas.log; false)

$(PKG)/libbc.so: $(OBJS)
	$(NVCC) $(ARCH) -shared -o $@ $(OBJS)
	@cat $(UNITS:%=build/%.ptxas.log) > $(CSRC)/ptxas.log
	@grep -E "registers|spill" $(CSRC)/ptxas.log | sed 's/^ptxas info    : //' | sort -u | head -20

# measurement helper for bench.py (L2 read ceiling), not part of the method
$(PKG)/libbcprobe.so: $(CSRC)/l2probe.cu
	$(NVCC) -O3 -std=c++17 $(ARCH) -Xcompiler -fPIC -Xcompiler -fvisibility=hidden -shared -o $@ $<

$(PKG)/libgraphgen.so: $(PKG)/graphgen_native.c
	gcc -O2 -std=c99 -fPIC -shared -pthread -o $@ $<

oracle/liboracle.so: oracle/brandes_oracle.c
	gcc -O2 -std=c99 -fPIC -shared -pthread -o $@ $<

clean:
	rm -rf build $(PKG)/libbc.so $(PKG)/libgraphgen.so $(PKG)/libbcprobe.so oracle/liboracle.so

.PHONY: all clean

# Tuning experiments: make variant VARIANT=name VFLAGS="-DBC_MINB512=3" builds
# build/<name>/libbc.so (load it with BC_LIBBC=build/<name>/libbc.so).
variant:
	@mkdir -p build/$(VARIANT)
	@for u in $(UNITS); do $(NVCC) $(NVFLAGS) $(VFLAGS) -c -o build/$(VARIANT)/$$u.o $(CSRC)/$$u.cu 2> build/$(VARIANT)/$$u.ptxas.log & done; wait
	$(NVCC) $(ARCH) -shared -o build/$(VARIANT)/libbc.so $(UNITS:%=build/$(VARIANT)/%.o)
	@cat build/$(VARIANT)/*.ptxas.log > build/$(VARIANT)/ptxas.log

.PHONY: variant
