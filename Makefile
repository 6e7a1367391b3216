# Build every native artefact in-tree (they travel to the GPU box with gpurun).
NVCC   ?= /usr/local/cuda/bin/nvcc
PKG    := paper_conf_iiswc_yudhakzs20_b200
ARCH   := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := -O3 -lineinfo -std=c++17 $(ARCH) -Xcompiler -fPIC -Xcompiler -fvisibility=hidden --expt-relaxed-constexpr
OBJDIR := build/obj

LP_SRCS := $(wildcard $(PKG)/csrc/*.cu)
LP_OBJS := $(patsubst $(PKG)/csrc/%.cu,$(OBJDIR)/%.o,$(LP_SRCS))
LP_HDRS := $(wildcard $(PKG)/csrc/*.cuh $(PKG)/csrc/*.h include/*.h)

all: oracle/liboracle.so lpsynth/libsynth.so $(PKG)/liblp.so examples/tmm_protect

oracle/liboracle.so: oracle/lp_oracle.c
	gcc -O2 -std=c11 -ffp-contract=off -fno-fast-math -shared -fPIC -o $@ $<

lpsynth/libsynth.so: lpsynth/synth.cu
	$(NVCC) $(NVFLAGS) -Xcompiler -fvisibility=default -shared -o $@ $<

$(OBJDIR)/%.o: $(PKG)/csrc/%.cu $(LP_HDRS)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -Iinclude -Xptxas -v -c -o $@ $< 2> $(OBJDIR)/$*.ptxas.txt || (cat $(OBJDIR)/$*.ptxas.txt; false)

$(PKG)/liblp.so: $(LP_OBJS)
	$(NVCC) $(ARCH) -shared -o $@ $(LP_OBJS)

# a pure-C client of the C ABI (no Python, no torch)
examples/tmm_protect: examples/tmm_protect.c include/liblp.h $(PKG)/liblp.so
	gcc -O2 -std=c11 -Wall -Iinclude -I/usr/local/cuda/include $< -L$(PKG) -llp -L/usr/local/cuda/lib64 -lcudart \
	    -Wl,-rpath,'$$ORIGIN/../$(PKG)' -Wl,-rpath,/usr/local/cuda/lib64 -o $@

clean:
	rm -rf build oracle/liboracle.so lpsynth/libsynth.so $(PKG)/liblp.so examples/tmm_protect

.PHONY: all clean
