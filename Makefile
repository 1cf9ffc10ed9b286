# libctaclust: sm_100a only (SASS, no PTX fallback); oracle: plain gcc.
NVCC ?= nvcc
PTXLOG ?= build_ptxas.log
PKG := paper_conf_asplos_lis0l0c17_b200
SRC := $(PKG)/csrc
LIB := $(PKG)/libctaclust.so
NVFLAGS := -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -lineinfo \
           -Xcompiler -fPIC -Xcompiler -Wall -Xptxas -v --expt-relaxed-constexpr -I include $(CC_DEFS)
HDRS := $(wildcard $(SRC)/*.cuh) include/ctaclust.h

all: $(LIB) oracle/liboracle.so oracle/liboracle_omp.so

$(LIB): $(SRC)/ctaclust.cu $(SRC)/cc_comm.cu $(HDRS)
	$(NVCC) $(NVFLAGS) -shared -o $@ $(SRC)/ctaclust.cu $(SRC)/cc_comm.cu -ldl 2> $(PTXLOG) || (cat $(PTXLOG); exit 1)

oracle/liboracle.so: oracle/oracle.c
	gcc -O2 -fPIC -shared -std=c11 -o $@ $<

# the same oracle with its OpenMP pragmas live: all-core timing (bench.py cpu_baseline) only
oracle/liboracle_omp.so: oracle/oracle.c
	gcc -O2 -fPIC -shared -std=c11 -fopenmp -o $@ $<

clean:
	rm -f $(LIB) oracle/liboracle.so oracle/liboracle_omp.so build_ptxas.log

.PHONY: all clean
