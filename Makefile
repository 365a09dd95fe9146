# Build every native artefact in-tree (they travel to the GPU box with gpurun).
NVCC    ?= /usr/local/cuda/bin/nvcc
ARCH    := -gencode arch=compute_100a,code=sm_100a
PKG     := paper_conf_eurosys_xiellwgrs22_b200
CFLAGS  := -O2 -fPIC -shared -fopenmp -Wall -Wextra
NVFLAGS := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-Wall -shared -cudart static -Iinclude

all: workload/libflgen.so oracle/libfleche_oracle.so $(PKG)/libfleche.so

workload/libflgen.so: workload/gen.c
	gcc $(CFLAGS) -o $@ $< -lm

oracle/libfleche_oracle.so: oracle/oracle.cpp
	g++ -std=c++17 -O2 -fPIC -shared -Wall -Wextra -o $@ $<

$(PKG)/libfleche.so: $(wildcard $(PKG)/csrc/*.cu $(PKG)/csrc/*.cuh $(PKG)/csrc/*.cpp) include/fleche.h
	$(NVCC) $(NVFLAGS) -Xptxas -v -o $@ $(PKG)/csrc/fleche.cu 2> $(PKG)/ptxas.log || (cat $(PKG)/ptxas.log; exit 1)

clean:
	rm -f workload/libflgen.so oracle/libfleche_oracle.so $(PKG)/libfleche.so

.PHONY: all clean

# timing-experiment build (tools only; semantics-breaking knobs behind FLECHE_EXP_MODE)
$(PKG)/libfleche_exp.so: $(wildcard $(PKG)/csrc/*.cu $(PKG)/csrc/*.cuh) include/fleche.h
	$(NVCC) $(NVFLAGS) -DFLECHE_EXPERIMENTS -o $@ $(PKG)/csrc/fleche.cu
