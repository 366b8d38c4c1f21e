# Build the product library (CUDA sm_100a) and the oracle (plain C).
NVCC      ?= nvcc
ARCH      := -gencode arch=compute_100a,code=sm_100a
# nccl.h for the run-time-loaded NCCL entry points (types only; libnccl.so.2 is dlopen'ed):
# the header of the NCCL torch ships, else the system one
NCCL_INC  ?= $(shell python3 -c "import nvidia.nccl, os; print(os.path.join(list(nvidia.nccl.__path__)[0], 'include'))" 2>/dev/null || echo /usr/include)
NVFLAGS   := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -O2 --expt-relaxed-constexpr -I$(NCCL_INC)
PKG       := paper_conf_ipps_overmanpmm13_b200
SRC       := $(PKG)/csrc
LIB       := $(PKG)/libafmm_p2p.so
CU_SRCS   := $(SRC)/afmm_p2p.cu $(SRC)/peak.cu $(SRC)/tree_build.cu $(SRC)/step.cu $(SRC)/balance.cpp $(SRC)/finegrained.cpp
CU_HDRS   := $(SRC)/nccl_api.h $(SRC)/p2p_kernel.cuh $(SRC)/worklist.inc $(SRC)/worklist_dev.cuh include/afmm_p2p.h include/afmm_tree.h include/afmm_step.h include/afmm_balance.h
ORACLE    := oracle/liboracle.so

all: $(LIB) $(ORACLE)

$(LIB): $(CU_SRCS) $(CU_HDRS)
	$(NVCC) $(NVFLAGS) -Xptxas -v -shared -o $@ $(CU_SRCS) -ldl 2> $(PKG)/ptxas.log || (cat $(PKG)/ptxas.log; false)
	@grep -E "registers|spill" $(PKG)/ptxas.log | grep -E "p2p_kernel|tree" -A0 | head -20 || true

$(ORACLE): oracle/oracle.c
	gcc -O2 -fopenmp -ffp-contract=off -fno-fast-math -fPIC -shared -std=c11 -o $@ $< -lm

# plain-C caller of the C ABI (no Python): examples/c_abi_demo.c
DEMO      := examples/c_abi_demo
$(DEMO): examples/c_abi_demo.c $(LIB) include/afmm_p2p.h include/afmm_tree.h
	gcc -O2 -std=c11 -Wall -Iinclude -I/usr/local/cuda/include -o $@ $< -L$(PKG) -lafmm_p2p \
	    -L/usr/local/cuda/lib64 -lcudart -lm -Wl,-rpath,'$$ORIGIN/../$(PKG)' -Wl,-rpath,/usr/local/cuda/lib64
demo: $(DEMO)

sass: $(LIB)
	cuobjdump -sass $(LIB) > $(PKG)/sass.txt

clean:
	rm -f $(LIB) $(ORACLE) $(PKG)/ptxas.log $(DEMO)

.PHONY: all clean sass demo
