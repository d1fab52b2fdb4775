# Builds every native artefact in-tree (they travel to the GPU box with gpurun).
#   libra.so     — the product: C-ABI + sm_100a kernels (include/ra.h)
#   libragen.so  — seeded input generator (host threads + CUDA), shared by tests
#   liboracle.so — the CPU oracle (test infrastructure only)

NVCC      ?= /usr/local/cuda/bin/nvcc
CC        ?= gcc
ARCH      := -gencode arch=compute_100a,code=sm_100a
NVFLAGS   := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-fvisibility=hidden -shared \
             -Xptxas -v --expt-relaxed-constexpr
PKG       := paper_conf_ipps_wudwcyc12_b200

RA_SRCS   := $(wildcard $(PKG)/csrc/*.cu) $(wildcard $(PKG)/csrc/*.cpp)
RA_HDRS   := $(wildcard $(PKG)/csrc/*.cuh) $(wildcard $(PKG)/csrc/*.h) include/ra.h

all: ragen/libragen.so oracle/liboracle.so $(PKG)/libra.so

ragen/libragen.so: ragen/ragen.cu ragen/ragen_core.h
	$(NVCC) $(ARCH) -O3 -std=c++17 -Xcompiler -fPIC -shared -o $@ ragen/ragen.cu

oracle/liboracle.so: oracle/oracle.c
	$(CC) -O2 -std=c11 -fPIC -shared -Wall -Wextra -o $@ oracle/oracle.c

$(PKG)/libra.so: $(RA_SRCS) $(RA_HDRS)
	$(NVCC) $(NVFLAGS) -Iinclude -o $@ $(RA_SRCS) -lpthread 2> $(PKG)/ptxas.log || (cat $(PKG)/ptxas.log; exit 1)
	@grep -E "registers|spill" $(PKG)/ptxas.log | sed 's/^ptxas info    ://' | head -40

# diagnostics builds of the product library with extra compile-time flags:
#   make variant NAME=wd FLAGS=-DRA_MO_WATCHDOG   ->  build/libra_wd.so  (RA_LIB_PATH=...)
variant: $(RA_SRCS) $(RA_HDRS)
	mkdir -p build
	$(NVCC) $(NVFLAGS) $(FLAGS) -Iinclude -o build/libra_$(NAME).so $(RA_SRCS) -lpthread 2> build/ptxas_$(NAME).log || (cat build/ptxas_$(NAME).log; exit 1)

clean:
	rm -f ragen/libragen.so oracle/liboracle.so $(PKG)/libra.so $(PKG)/ptxas.log

.PHONY: all clean variant
