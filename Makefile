# Builds every native artefact in-tree (the .so files travel to the GPU box with
# the gpurun snapshot; they are git-ignored).
#
#   paper_conf_ipps_li0ptz24_b200/libtc.so   the product: C-ABI + sm_100a kernels
#   tcgen/libtcgen.so                        seeded input generators (host)
#   oracle/libtcoracle.so                    CPU oracle (test infrastructure)

NVCC      ?= /usr/local/cuda/bin/nvcc
CXX       ?= g++
PKG       := paper_conf_ipps_li0ptz24_b200
ARCH      := -gencode arch=compute_100a,code=sm_100a
NVFLAGS   := $(NVEXTRA) -O3 -std=c++17 $(ARCH) -lineinfo -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
             -Iinclude --expt-relaxed-constexpr -Xptxas -v
CXXFLAGS  := -O3 -std=c++17 -fPIC -pthread

CU_SRC    := $(wildcard $(PKG)/csrc/*.cu)
CU_HDR    := $(wildcard $(PKG)/csrc/*.cuh) include/tc.h
CU_OBJ    := $(patsubst $(PKG)/csrc/%.cu,build/%.o,$(CU_SRC))

all: $(PKG)/libtc.so tcgen/libtcgen.so oracle/libtcoracle.so

build/%.o: $(PKG)/csrc/%.cu $(CU_HDR)
	@mkdir -p build
	$(NVCC) $(NVFLAGS) -c $< -o $@ 2> build/$*.ptxas.txt || (cat build/$*.ptxas.txt; false)

$(PKG)/libtc.so: $(CU_OBJ)
	$(NVCC) $(ARCH) -shared -o $@ $(CU_OBJ) -cudart static

tcgen/libtcgen.so: tcgen/tcgen.cpp include/tcgen.h
	$(CXX) $(CXXFLAGS) -Iinclude -shared $< -o $@

oracle/libtcoracle.so: oracle/tc_oracle.cpp
	$(CXX) $(CXXFLAGS) -shared $< -o $@

clean:
	rm -rf build $(PKG)/libtc.so tcgen/libtcgen.so oracle/libtcoracle.so

.PHONY: all clean
