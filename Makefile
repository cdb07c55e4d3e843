# Builds the CUDA library (sm_100a), the generator twin and the C oracle.
NVCC      ?= /usr/local/cuda/bin/nvcc
ARCH      := -gencode arch=compute_100a,code=sm_100a
NVFLAGS   := -O3 -std=c++17 $(ARCH) -lineinfo -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
             --expt-relaxed-constexpr -diag-suppress 177 -cudart static
PKG       := paper_conf_sigmod_shahvaranij16_b200
NCCL_HOME ?= $(shell python -c "import nvidia.nccl, os; print(os.path.dirname(nvidia.nccl.__file__) if nvidia.nccl.__file__ else list(nvidia.nccl.__path__)[0])" 2>/dev/null)
CSRC      := $(wildcard $(PKG)/csrc/*.cu)
HDRS      := $(wildcard $(PKG)/csrc/*.cuh) include/hbt.h
OBJDIR    := build/obj
OBJS      := $(patsubst $(PKG)/csrc/%.cu,$(OBJDIR)/%.o,$(CSRC))

all: $(PKG)/libhbt.so gen/libhbtgen.so oracle/liboracle.so tools/libhbtprobe.so

$(OBJDIR)/%.o: $(PKG)/csrc/%.cu $(HDRS)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -I$(NCCL_HOME)/include -Xcompiler -DHBT_BUILDING -c $< -o $@

$(PKG)/libhbt.so: $(OBJS)
	$(NVCC) $(ARCH) -shared -cudart static -o $@ $(OBJS) -L$(NCCL_HOME)/lib -l:libnccl.so.2 \
	  -Xlinker -rpath -Xlinker $(NCCL_HOME)/lib

gen/libhbtgen.so: gen/gen.cu
	$(NVCC) -O3 -std=c++17 $(ARCH) -Xcompiler -fPIC -shared -cudart static -o $@ $<

tools/libhbtprobe.so: tools/probe.cu
	$(NVCC) -O3 -std=c++17 $(ARCH) -Xcompiler -fPIC -shared -cudart static -o $@ $<

oracle/liboracle.so: oracle/oracle.c oracle/oracle.h
	gcc -std=c11 -O2 -fPIC -shared -fopenmp -o $@ oracle/oracle.c

clean:
	rm -rf build $(PKG)/libhbt.so gen/libhbtgen.so oracle/liboracle.so tools/libhbtprobe.so

.PHONY: all clean
