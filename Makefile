# Build of the B200-native GPApriori library (sm_100a only) and of the test-side C helpers.
#   make            -> paper_conf_cluster_zhangzb11a_b200/libgpapriori.so, oracle/liboracle.so, gen/libgen.so
PY        ?= python
NVCC      ?= /usr/local/cuda/bin/nvcc
CXX       ?= g++
CC        ?= gcc
NCCL_DIR  ?= $(shell $(PY) -c "import os, nvidia.nccl as n; print(os.path.dirname(n.__file__) if n.__file__ else list(n.__path__)[0])" 2>/dev/null)
PKG       := paper_conf_cluster_zhangzb11a_b200
CSRC      := $(PKG)/csrc
BUILD     := build
ARCH      := -gencode arch=compute_100a,code=sm_100a
NVFLAGS   := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -Wall -Iinclude -I$(CSRC) -I$(NCCL_DIR)/include
CXXFLAGS  := -O2 -g -fPIC -std=c++17 -Wall -Wextra -Iinclude -I$(CSRC) -I/usr/local/cuda/include -I$(NCCL_DIR)/include
LIB       := $(PKG)/libgpapriori.so

CU_SRCS   := $(wildcard $(CSRC)/kernels/*.cu)
CPP_SRCS  := $(wildcard $(CSRC)/runtime/*.cpp)
CU_OBJS   := $(patsubst $(CSRC)/kernels/%.cu,$(BUILD)/k_%.o,$(CU_SRCS))
CPP_OBJS  := $(patsubst $(CSRC)/runtime/%.cpp,$(BUILD)/r_%.o,$(CPP_SRCS))
HDRS      := $(wildcard $(CSRC)/kernels/*.cuh) include/gpapriori.h $(CSRC)/common.h $(CSRC)/kernels.h $(CSRC)/runtime/internal.h $(CSRC)/runtime/pool.h

all: $(LIB) oracle/liboracle.so gen/libgen.so examples/gpa_mine_fimi

$(BUILD):
	mkdir -p $(BUILD)

$(BUILD)/k_%.o: $(CSRC)/kernels/%.cu $(HDRS) | $(BUILD)
	$(NVCC) $(NVFLAGS) -Xptxas -v -c $< -o $@ 2> $(BUILD)/k_$*.ptxas.txt || (cat $(BUILD)/k_$*.ptxas.txt; false)

$(BUILD)/r_%.o: $(CSRC)/runtime/%.cpp $(HDRS) | $(BUILD)
	$(CXX) $(CXXFLAGS) -c $< -o $@

$(LIB): $(CU_OBJS) $(CPP_OBJS)
	$(NVCC) $(ARCH) -shared -o $@ $^ -L$(NCCL_DIR)/lib -l:libnccl.so.2 -Xlinker -rpath=$(NCCL_DIR)/lib -lpthread

oracle/liboracle.so: oracle/apriori_oracle.c
	$(CC) -O2 -shared -fPIC -Wall -o $@ $< -lpthread

gen/libgen.so: gen/quest.c
	$(CC) -O2 -shared -fPIC -Wall -o $@ $< -lm -lpthread

examples/gpa_mine_fimi: examples/gpa_mine_fimi.c include/gpapriori.h $(LIB)
	$(CC) -O2 -std=c11 -D_POSIX_C_SOURCE=200809L -Wall -Iinclude -o $@ $< -L$(PKG) -lgpapriori -Wl,-rpath,'$$ORIGIN/../$(PKG)'

clean:
	rm -rf $(BUILD) $(LIB) oracle/liboracle.so gen/libgen.so examples/gpa_mine_fimi

.PHONY: all clean
