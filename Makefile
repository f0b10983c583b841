# Builds libgsh.so (sm_100a) in-tree and the CPU oracle (test infrastructure).
NVCC ?= /usr/local/cuda/bin/nvcc
ARCH := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := -O3 -std=c++17 $(ARCH) -lineinfo -Xcompiler -fPIC -Xcompiler -fvisibility=hidden -Iinclude
SRC_DIR := paper_conf_icde_caic24_b200/csrc
OBJ_DIR := build/obj
LIB := paper_conf_icde_caic24_b200/lib/libgsh.so
CU := $(wildcard $(SRC_DIR)/*.cu)
OBJ := $(patsubst $(SRC_DIR)/%.cu,$(OBJ_DIR)/%.o,$(CU))
HDR := $(wildcard $(SRC_DIR)/*.cuh) $(wildcard $(SRC_DIR)/*.h) include/gsh.h

all: $(LIB) oracle/liboracle.so

$(OBJ_DIR)/%.o: $(SRC_DIR)/%.cu $(HDR)
	@mkdir -p $(OBJ_DIR)
	$(NVCC) $(NVFLAGS) -Xptxas -v -c $< -o $@ 2> $(OBJ_DIR)/$*.ptxas.txt || (cat $(OBJ_DIR)/$*.ptxas.txt; false)

$(LIB): $(OBJ)
	@mkdir -p $(dir $(LIB))
	$(NVCC) $(ARCH) -shared -cudart static -o $@ $(OBJ) -ldl

oracle/liboracle.so: oracle/join_oracle.c
	gcc -O2 -std=c11 -shared -fPIC -pthread $< -o $@

clean:
	rm -rf build $(LIB) oracle/liboracle.so

.PHONY: all clean
