# Build: `make` (all), `make gen oracle` (CPU-only pieces), `make accmg` (CUDA product library).
# nvcc cross-compiles sm_100a without a GPU.
NVCC     ?= /usr/local/cuda/bin/nvcc
CC       := gcc
CXX      := g++
PKG      := paper_conf_icpp_komodamnm13_b200
CSRC     := $(PKG)/csrc
NCCL_INC ?= $(shell python -c "import nvidia.nccl, os; print(os.path.join(list(nvidia.nccl.__path__)[0], 'include'))" 2>/dev/null)
ARCH     := -gencode arch=compute_100a,code=sm_100a
NVFLAGS  := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O2,-Wall -Xptxas -v \
            --expt-relaxed-constexpr -Iinclude -I$(CSRC) $(if $(NCCL_INC),-I$(NCCL_INC),)
CUFILES  := $(wildcard $(CSRC)/*.cu)
CPPFILES := $(wildcard $(CSRC)/*.cpp)
HDRS     := $(wildcard $(CSRC)/*.h $(CSRC)/*.cuh include/*.h)
OBJDIR   := build/obj
CUOBJS   := $(patsubst $(CSRC)/%.cu,$(OBJDIR)/%.o,$(CUFILES))
CPPOBJS  := $(patsubst $(CSRC)/%.cpp,$(OBJDIR)/%.cpp.o,$(CPPFILES))

.PHONY: all gen oracle accmg clean
all: gen oracle accmg

gen: gen/libaccgen.so
gen/libaccgen.so: gen/accgen.c
	$(CC) -O2 -fopenmp -shared -fPIC -Wall -o $@ $<

# The oracle: plain C, no FMA contraction, shares nothing with the product tree.
oracle: oracle/liboracle.so
oracle/liboracle.so: oracle/oracle.c
	$(CC) -O2 -ffp-contract=off -mfma -fopenmp -shared -fPIC -Wall -o $@ $< -lm

accmg: $(PKG)/libaccmg.so
$(OBJDIR)/%.o: $(CSRC)/%.cu $(HDRS)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -c -o $@ $< 2> $(OBJDIR)/$*.ptxas.txt || (cat $(OBJDIR)/$*.ptxas.txt; false)
$(OBJDIR)/%.cpp.o: $(CSRC)/%.cpp $(HDRS)
	@mkdir -p $(OBJDIR)
	$(CXX) -O2 -std=c++17 -fPIC -Wall -Iinclude -I$(CSRC) -I/usr/local/cuda/include \
	    $(if $(NCCL_INC),-I$(NCCL_INC),) -c -o $@ $<
$(PKG)/libaccmg.so: $(CUOBJS) $(CPPOBJS)
	$(NVCC) $(ARCH) -shared -o $@ $^ -lcudart_static -ldl -lrt -lpthread

clean:
	rm -rf build gen/libaccgen.so oracle/liboracle.so $(PKG)/libaccmg.so
