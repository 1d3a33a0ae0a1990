# Build of the B200-native library (libpdl.so, sm_100a) and the CPU oracle
# (oracle/liboracle.so, gcc only).  `python -c "import __graft_entry__ as g; g.build()"`
# runs this.
NVCC      ?= /usr/local/cuda/bin/nvcc
CXX       ?= g++
PKG       := paper_conf_ipps_sandrieserbp11_b200
CSRC      := $(PKG)/csrc
BUILD     := build
ARCH      := -gencode arch=compute_100a,code=sm_100a
NVFLAGS   := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden -Xptxas -v --expt-relaxed-constexpr
CXXFLAGS  := -O2 -std=c++17 -fPIC -fvisibility=hidden -Wall -Wextra -Wno-unused-parameter

HOST_SRC  := $(CSRC)/pdl_xml.cpp $(CSRC)/pdl_model.cpp $(CSRC)/pdl_map.cpp
CU_SRC    := $(CSRC)/pdl_runtime.cu $(CSRC)/pdl_devices.cu $(CSRC)/pdl_exec.cu $(CSRC)/pdl_xchg.cu $(CSRC)/k_dgemm.cu $(CSRC)/k_tf32.cu $(CSRC)/k_tf32_2sm.cu $(CSRC)/k_ozaki.cu $(CSRC)/k_ozaki2.cu
HOST_OBJ  := $(patsubst $(CSRC)/%.cpp,$(BUILD)/%.o,$(HOST_SRC))
CU_OBJ    := $(patsubst $(CSRC)/%.cu,$(BUILD)/%.o,$(CU_SRC))
HDRS      := $(wildcard $(CSRC)/*.h $(CSRC)/*.hpp $(CSRC)/*.cuh) include/libpdl.h

LIB       := $(PKG)/libpdl.so
ORACLE    := oracle/liboracle.so

all: $(LIB) $(ORACLE)

examples: examples/dgemm_c_abi

# measurement tools (peaks, tensor-core behaviour, green-context splits)
TOOLS := tools/microbench tools/tc_microbench tools/tc_probe tools/fp64_mix_probe tools/green_probe tools/cluster_probe tools/feed_probe
tools: $(TOOLS)

tools/%: tools/%.cu
	$(NVCC) $(ARCH) -O3 -lineinfo -std=c++17 -o $@ $< -lcuda

examples/dgemm_c_abi: examples/dgemm_c_abi.c include/libpdl.h $(LIB)
	gcc -O2 -Wall -o $@ $< -L$(PKG) -lpdl -Wl,-rpath,'$$ORIGIN/../$(PKG)' -lm

$(BUILD):
	mkdir -p $(BUILD)

$(BUILD)/%.o: $(CSRC)/%.cpp $(HDRS) | $(BUILD)
	$(CXX) $(CXXFLAGS) -c $< -o $@

$(BUILD)/%.o: $(CSRC)/%.cu $(HDRS) | $(BUILD)
	$(NVCC) $(NVFLAGS) -c $< -o $@ 2> $(BUILD)/$*.ptxas.txt || (cat $(BUILD)/$*.ptxas.txt; exit 1)

$(LIB): $(HOST_OBJ) $(CU_OBJ)
	$(NVCC) $(ARCH) -shared -cudart static -o $@ $^ -lrt -ldl -lpthread

$(ORACLE): oracle/oracle.c
	gcc -O3 -fopenmp -ffp-contract=off -fno-fast-math -shared -fPIC -o $@ $< -lm

clean:
	rm -rf $(BUILD) $(LIB) $(ORACLE) examples/dgemm_c_abi $(TOOLS)

.PHONY: all clean examples tools
