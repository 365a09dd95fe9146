# Build every native artefact in-tree (they travel to the GPU box with gpurun).
# libfleche.so is linked from four translation units compiled in parallel (make -j):
# the host side and three kernel groups (fns.h).
NVCC    ?= /usr/local/cuda/bin/nvcc
ARCH    := -gencode arch=compute_100a,code=sm_100a
PKG     := paper_conf_eurosys_xiellwgrs22_b200
CSRC    := $(PKG)/csrc
BUILD   := build
CFLAGS  := -O2 -fPIC -shared -fopenmp -Wall -Wextra
NVFLAGS := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-Wall -Iinclude
HDRS    := $(wildcard $(CSRC)/*.cuh $(CSRC)/*.h) include/fleche.h
UNITS   := fleche k_query k_miss k_misc
OBJS    := $(UNITS:%=$(BUILD)/%.o)
MAKEFLAGS += -j4

all: workload/libflgen.so oracle/libfleche_oracle.so $(PKG)/libfleche.so

workload/libflgen.so: workload/gen.c
	gcc $(CFLAGS) -o $@ $< -lm

oracle/libfleche_oracle.so: oracle/oracle.cpp
	g++ -std=c++17 -O2 -fPIC -shared -Wall -Wextra -o $@ $<

$(BUILD)/%.o: $(CSRC)/%.cu $(HDRS)
	@mkdir -p $(BUILD)
	$(NVCC) $(NVFLAGS) $(EXTRA) -Xptxas -v -c -o $@ $< 2> $(BUILD)/$*.ptxas.log || (cat $(BUILD)/$*.ptxas.log; exit 1)

$(PKG)/libfleche.so: $(OBJS)
	$(NVCC) $(ARCH) -shared -cudart static -o $@ $(OBJS)
	cat $(UNITS:%=$(BUILD)/%.ptxas.log) > $(PKG)/ptxas.log

clean:
	rm -rf $(BUILD) workload/libflgen.so oracle/libfleche_oracle.so $(PKG)/libfleche.so $(PKG)/libfleche_exp.so

.PHONY: all clean

# timing-experiment build (tools only; semantics-breaking knobs behind FLECHE_EXPERIMENTS)
$(PKG)/libfleche_exp.so: $(wildcard $(CSRC)/*.cu) $(HDRS)
	@mkdir -p $(BUILD)/exp
	for u in $(UNITS); do $(NVCC) $(NVFLAGS) -DFLECHE_EXPERIMENTS -c -o $(BUILD)/exp/$$u.o $(CSRC)/$$u.cu || exit 1; done
	$(NVCC) $(ARCH) -shared -cudart static -o $@ $(UNITS:%=$(BUILD)/exp/%.o)

# A/B variant build: make variant V=name EXTRA="-DFL_KQ_PROBE=16" -> $(PKG)/libfleche_name.so
# (select at run time with FLECHE_LIB=libfleche_name.so)
variant:
	@mkdir -p $(BUILD)/v_$(V)
	for u in $(UNITS); do $(NVCC) $(NVFLAGS) $(EXTRA) -c -o $(BUILD)/v_$(V)/$$u.o $(CSRC)/$$u.cu & done; wait
	$(NVCC) $(ARCH) -shared -cudart static -o $(PKG)/libfleche_$(V).so $(UNITS:%=$(BUILD)/v_$(V)/%.o)
