# Builds the product library (CUDA sm_100a + C++ host runtime) and the CPU oracle.
#   make            -> paper_conf_asplos_strati0k25_b200/libpccheck.so, oracle/liboracle.so
PKG      := paper_conf_asplos_strati0k25_b200
CSRC     := $(PKG)/csrc
BUILD    := build
CUDA     ?= /usr/local/cuda
PY       ?= python
NCCL_DIR := $(shell $(PY) -c "import nvidia.nccl, os; print(os.path.dirname(nvidia.nccl.__path__[0]) + '/nccl')" 2>/dev/null)
NVCC     := $(CUDA)/bin/nvcc
ARCH     := -gencode arch=compute_100a,code=sm_100a
NVFLAGS  := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-fvisibility=hidden -Xptxas -v -I$(NCCL_DIR)/include
CXXFLAGS := -O2 -g -fPIC -std=c++17 -msse4.2 -Wall -Wno-unused-function -I$(CUDA)/include -I$(NCCL_DIR)/include \
            -DPCC_NCCL_LIBDIR=\"$(NCCL_DIR)/lib\" -fvisibility=hidden
HDRS     := $(wildcard $(CSRC)/*.hpp $(CSRC)/*.cuh include/*.h)

OBJS := $(BUILD)/kernels.o $(BUILD)/runtime.o $(BUILD)/commit.o $(BUILD)/kapi.o $(BUILD)/host_api.o

all: $(PKG)/libpccheck.so oracle/liboracle.so

$(BUILD):
	mkdir -p $(BUILD)

$(BUILD)/kernels.o: $(CSRC)/kernels.cu $(HDRS) | $(BUILD)
	$(NVCC) $(NVFLAGS) -c $< -o $@ 2> $(BUILD)/ptxas.log || (cat $(BUILD)/ptxas.log; false)

$(BUILD)/%.o: $(CSRC)/%.cpp $(HDRS) | $(BUILD)
	g++ $(CXXFLAGS) -c $< -o $@

$(PKG)/libpccheck.so: $(OBJS)
	g++ -shared -o $@ $(OBJS) -L$(CUDA)/lib64 -lcudart_static -ldl -lpthread -lrt -Wl,--exclude-libs,ALL

oracle/liboracle.so: oracle/pcc_oracle.c
	gcc -O2 -Wall -shared -fPIC -o $@ $<

clean:
	rm -rf $(BUILD) $(PKG)/libpccheck.so oracle/liboracle.so

.PHONY: all clean
