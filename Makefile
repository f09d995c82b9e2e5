# Builds libpasta.so (sm_100a) in-tree and the CPU oracle.  `make -j` from the repo root.
NVCC      ?= /usr/local/cuda/bin/nvcc
ARCH      := -gencode arch=compute_100a,code=sm_100a
NVFLAGS   := -O3 -std=c++17 $(ARCH) -lineinfo -Xcompiler -fPIC -Xcompiler -Wall \
             --expt-relaxed-constexpr -Xptxas -v
PKG       := paper_conf_iiswc_lilwlob20_b200
SRCDIR    := $(PKG)/csrc
BUILDDIR  := build
SRCS      := $(wildcard $(SRCDIR)/*.cu)
OBJS      := $(patsubst $(SRCDIR)/%.cu,$(BUILDDIR)/%.o,$(SRCS))
LIB       := $(PKG)/lib/libpasta.so
ORACLE    := oracle/liboracle.so

all: $(LIB) $(ORACLE)

$(BUILDDIR)/%.o: $(SRCDIR)/%.cu $(SRCDIR)/internal.cuh include/pasta.h
	@mkdir -p $(BUILDDIR)
	$(NVCC) $(NVFLAGS) -c $< -o $@ 2> $(BUILDDIR)/$*.ptxas.log || (cat $(BUILDDIR)/$*.ptxas.log; false)

$(LIB): $(OBJS)
	@mkdir -p $(PKG)/lib
	$(NVCC) $(ARCH) -shared -o $@ $(OBJS) -cudart static

$(ORACLE): oracle/oracle.c
	gcc -O2 -ffp-contract=off -fPIC -shared -o $@ $< -lm

clean:
	rm -rf $(BUILDDIR) $(LIB) $(ORACLE)

.PHONY: all clean
