# libkgs (CUDA path, sm_100a), the oracle (plain C, test infrastructure) and the input generator.
NVCC ?= nvcc
ARCH := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := -O3 -std=c++17 $(ARCH) -lineinfo -Xcompiler -fPIC \
           --expt-relaxed-constexpr -Xptxas -v
PKG := paper_conf_icde_yangajtw19_b200
CSRC := $(PKG)/csrc
LIB := $(PKG)/libkgs.so
OBJS := $(CSRC)/api.o $(CSRC)/prep.o $(CSRC)/engine.o $(CSRC)/vpart.o $(CSRC)/relabel.o $(CSRC)/load.o \
        $(CSRC)/vpquery.o

all: $(LIB) oracle/liboracle.so synth/libkgs_synth.so

$(CSRC)/%.o: $(CSRC)/%.cu $(CSRC)/kgs_internal.h include/kgs.h
	$(NVCC) $(NVFLAGS) -c $< -o $@ 2> $@.ptxas.log || (cat $@.ptxas.log; exit 1)

$(LIB): $(OBJS)
	$(NVCC) $(ARCH) -shared -o $@ $(OBJS) -ldl

oracle/liboracle.so: oracle/oracle.c
	gcc -O2 -fPIC -shared -ffp-contract=off -fno-fast-math -o $@ $< -lm

synth/libkgs_synth.so: synth/kgs_synth.c
	gcc -O2 -fopenmp -fPIC -shared -ffp-contract=off -o $@ $< -lm

clean:
	rm -f $(OBJS) $(CSRC)/*.ptxas.log $(LIB) oracle/liboracle.so synth/libkgs_synth.so

.PHONY: all clean
