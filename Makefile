# libpm.so (CUDA path, sm_100a) and the CPU oracle's libpm_oracle.so.
NVCC ?= nvcc
ARCH := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -Wall --expt-relaxed-constexpr
PKG := paper_conf_ipps_yangin17_b200
SRCS := $(wildcard $(PKG)/csrc/*.cu)
HDRS := $(wildcard $(PKG)/csrc/*.cuh) include/pm.h

all: $(PKG)/libpm.so oracle/libpm_oracle.so

$(PKG)/libpm.so: $(SRCS) $(HDRS)
	$(NVCC) $(NVFLAGS) -shared -cudart static -o $@ $(SRCS)

oracle/libpm_oracle.so: oracle/pm_oracle.c
	gcc -O2 -fopenmp -shared -fPIC -std=c11 -o $@ $<

ptxas:
	$(NVCC) $(NVFLAGS) -Xptxas -v -c $(PKG)/csrc/k_sad.cu -o /tmp/k_sad.o
	$(NVCC) $(NVFLAGS) -Xptxas -v -c $(PKG)/csrc/k_search.cu -o /tmp/k_search.o

clean:
	rm -f $(PKG)/libpm.so oracle/libpm_oracle.so

.PHONY: all clean ptxas
