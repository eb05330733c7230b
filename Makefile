# Native build: libdasp.so (product, sm_100a) + the test-side helper libraries.
NVCC      ?= /usr/local/cuda/bin/nvcc
ARCH      := -gencode arch=compute_100a,code=sm_100a
NVFLAGS   := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-fopenmp -Xptxas -v
CXXFLAGS  := -O3 -std=c++17 -fPIC -fopenmp -Wall -Wextra
PKG       := paper_conf_sc_lu023_b200
SRC       := $(PKG)/csrc
OBJ       := build

all: $(PKG)/libdasp.so oracle/liboracle.so synth/libsynth.so

$(OBJ):
	mkdir -p $(OBJ)

$(OBJ)/builder.o: $(SRC)/builder.cpp $(SRC)/format.hpp include/dasp.h | $(OBJ)
	g++ $(CXXFLAGS) -c $< -o $@

$(OBJ)/kernels.o: $(SRC)/kernels.cu $(SRC)/kernels.cuh | $(OBJ)
	$(NVCC) $(NVFLAGS) -c $< -o $@ 2> $(OBJ)/kernels.ptxas.txt || (cat $(OBJ)/kernels.ptxas.txt; false)

$(OBJ)/api.o: $(SRC)/api.cu $(SRC)/kernels.cuh $(SRC)/gpu_builder.cuh $(SRC)/format.hpp include/dasp.h | $(OBJ)
	$(NVCC) $(NVFLAGS) -c $< -o $@

$(OBJ)/gpu_builder.o: $(SRC)/gpu_builder.cu $(SRC)/gpu_builder.cuh $(SRC)/format.hpp include/dasp.h | $(OBJ)
	$(NVCC) $(NVFLAGS) -c $< -o $@ 2> $(OBJ)/gpu_builder.ptxas.txt || (cat $(OBJ)/gpu_builder.ptxas.txt; false)

$(PKG)/libdasp.so: $(OBJ)/builder.o $(OBJ)/kernels.o $(OBJ)/gpu_builder.o $(OBJ)/api.o
	$(NVCC) $(ARCH) -shared -o $@ $^ -Xcompiler -fopenmp -lgomp

oracle/liboracle.so: oracle/oracle.c
	gcc -O2 -ffp-contract=off -fno-fast-math -fopenmp -fPIC -shared -o $@ $< -lm

synth/libsynth.so: synth/synth.c
	gcc -O2 -fopenmp -fPIC -shared -o $@ $< -lm

clean:
	rm -rf $(OBJ) $(PKG)/libdasp.so oracle/liboracle.so synth/libsynth.so

.PHONY: all clean

# experiment builds: one build/libdasp_<VAR=value[+VAR=value]>.so per EXPVARS entry (comma-separated
# -D settings applied to every translation unit); select one with DASP_LIB=<path> (dasp.py)
EXPVARS ?= DASP_NARROW_IL=1
exp:
	for v in $(EXPVARS); do \
	  t=$$(echo $$v | tr , +); d="-D$$(echo $$v | sed 's/,/ -D/g')"; mkdir -p $(OBJ)/exp_$$t; \
	  g++ $(CXXFLAGS) $$d -c $(SRC)/builder.cpp -o $(OBJ)/exp_$$t/builder.o && \
	  $(NVCC) $(NVFLAGS) $$d -c $(SRC)/kernels.cu -o $(OBJ)/exp_$$t/kernels.o 2> $(OBJ)/exp_$$t/kernels.ptxas.txt && \
	  $(NVCC) $(NVFLAGS) $$d -c $(SRC)/gpu_builder.cu -o $(OBJ)/exp_$$t/gpu_builder.o 2> /dev/null && \
	  $(NVCC) $(NVFLAGS) $$d -c $(SRC)/api.cu -o $(OBJ)/exp_$$t/api.o && \
	  $(NVCC) $(ARCH) -shared -o $(OBJ)/libdasp_$$t.so $(OBJ)/exp_$$t/*.o -Xcompiler -fopenmp -lgomp || exit 1; \
	done

.PHONY: exp
