# Build: libfusedpat (the product, sm_100a), liboracle (host C, test infrastructure),
# libsynth_{host,cuda} (seeded input generators).  `make -j` or __graft_entry__.build().
NVCC     ?= nvcc
CC       := gcc
ARCH     := -gencode arch=compute_100a,code=sm_100a
NVFLAGS  := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC --expt-relaxed-constexpr
# FP_EXPERIMENTAL=1 also builds the measured-but-never-chosen CSR variants 10, 12, 14, 15
ifeq ($(FP_EXPERIMENTAL),1)
NVFLAGS  += -DFP_EXPERIMENTAL_VARIANTS
endif
CFLAGS   := -O2 -fPIC -shared -fopenmp -ffp-contract=off -std=c11 -Wall
PKG      := paper_conf_ppopp_asharitbrcks15_b200
CSRC     := $(PKG)/csrc
OBJDIR   := build/obj
FP_SRCS  := $(wildcard $(CSRC)/*.cu)
FP_OBJS  := $(patsubst $(CSRC)/%.cu,$(OBJDIR)/%.o,$(FP_SRCS))
FP_HDRS  := $(wildcard $(CSRC)/*.cuh) include/fusedpat.h

all: fusedpat oracle synth

fusedpat: $(PKG)/libfusedpat.so
oracle: oracle/liboracle.so
synth: synth/libsynth_host.so synth/libsynth_cuda.so

$(OBJDIR)/%.o: $(CSRC)/%.cu $(FP_HDRS)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -Iinclude -Xptxas -v -c -o $@ $< 2> $@.ptxas.log || (cat $@.ptxas.log; exit 1)

$(PKG)/libfusedpat.so: $(FP_OBJS)
	$(NVCC) $(ARCH) -shared -o $@ $(FP_OBJS) -lnccl -lcudart
	@cat $(OBJDIR)/*.ptxas.log > $(PKG)/ptxas.log

oracle/liboracle.so: oracle/oracle.c
	$(CC) $(CFLAGS) -o $@ $< -lm

synth/libsynth_host.so: synth/synth_host.c synth/synth_core.h
	$(CC) $(CFLAGS) -o $@ $< -lm

synth/libsynth_cuda.so: synth/synth_cuda.cu synth/synth_core.h
	$(NVCC) $(NVFLAGS) -shared -o $@ $<

clean:
	rm -rf $(OBJDIR) $(PKG)/libfusedpat.so oracle/liboracle.so synth/libsynth_host.so synth/libsynth_cuda.so

.PHONY: all fusedpat oracle synth clean
