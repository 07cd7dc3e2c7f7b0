# Builds paper_conf_asplos_cowanmmsx23_b200/libmsccl_b200.so (C ABI in include/msccl.h)
# for sm_100a. No fast-math / ftz: reductions must round exactly like the oracle.
NVCC    ?= nvcc
ARCH    ?= -gencode arch=compute_100a,code=sm_100a
PKG     := paper_conf_asplos_cowanmmsx23_b200
SRC     := $(PKG)/csrc
OBJDIR  ?= build/obj
EXTRA   ?=
NVFLAGS := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -Wall -diag-suppress 177 -Iinclude -I$(SRC) $(EXTRA)
CXXSRCS := $(wildcard $(SRC)/*.cpp)
CUSRCS  := $(wildcard $(SRC)/*.cu)
OBJS    := $(patsubst $(SRC)/%.cpp,$(OBJDIR)/%.o,$(CXXSRCS)) $(patsubst $(SRC)/%.cu,$(OBJDIR)/%.o,$(CUSRCS))
HDRS    := $(wildcard $(SRC)/*.h) $(wildcard $(SRC)/*.cuh) include/msccl.h
LIB     ?= $(PKG)/libmsccl_b200.so

all: $(LIB)

$(OBJDIR)/%.o: $(SRC)/%.cpp $(HDRS)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -c $< -o $@

$(OBJDIR)/%.o: $(SRC)/%.cu $(HDRS)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -Xptxas -v -c $< -o $@ 2> $(OBJDIR)/$*.ptxas.txt || (cat $(OBJDIR)/$*.ptxas.txt; exit 1)

$(LIB): $(OBJS)
	$(NVCC) $(ARCH) -shared -o $@ $(OBJS)

clean:
	rm -rf build $(LIB)

.PHONY: all clean
