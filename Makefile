# Builds the three native artefacts in-tree (they travel to the GPU box with the snapshot).
#   gen/libvista_gen.so      seeded input generators (shared by both sides; no method arithmetic)
#   oracle/liboracle.so      fp64 CPU oracle (test infrastructure only)
#   paper_conf_sigmod_nakandalak20_b200/libvista.so   the product: sm_100a kernels + C-ABI
NVCC ?= /usr/local/cuda/bin/nvcc
CXX ?= g++
CC ?= gcc
PKG := paper_conf_sigmod_nakandalak20_b200
CSRC := $(PKG)/csrc
CU_SRCS := $(wildcard $(CSRC)/*.cu)
CPP_SRCS := $(wildcard $(CSRC)/*.cpp)
HDRS := $(wildcard $(CSRC)/*.cuh) $(wildcard $(CSRC)/*.h) include/vista.h gen/vista_gen.h
ARCH := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := -O3 -std=c++17 $(ARCH) -lineinfo -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
           -Iinclude -Igen -I$(CSRC) --expt-relaxed-constexpr -Xptxas -O3
OBJDIR := build/obj

all: gen/libvista_gen.so oracle/liboracle.so $(PKG)/libvista.so

gen/libvista_gen.so: gen/vista_gen.c gen/vista_gen.h
	$(CC) -O2 -fPIC -shared -o $@ gen/vista_gen.c -lm -lpthread

oracle/liboracle.so: oracle/oracle.cpp oracle/oracle.h $(OBJDIR)/vista_gen.o
	$(CXX) -O2 -std=c++17 -fPIC -shared -o $@ oracle/oracle.cpp $(OBJDIR)/vista_gen.o -lm -lpthread

CU_OBJS := $(patsubst $(CSRC)/%.cu,$(OBJDIR)/%.o,$(CU_SRCS))
CPP_OBJS := $(patsubst $(CSRC)/%.cpp,$(OBJDIR)/%.cpp.o,$(CPP_SRCS))

$(OBJDIR)/%.o: $(CSRC)/%.cu $(HDRS)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -c -o $@ $<

$(OBJDIR)/%.cpp.o: $(CSRC)/%.cpp $(HDRS)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -x cu -c -o $@ $<

$(OBJDIR)/vista_gen.o: gen/vista_gen.c gen/vista_gen.h
	@mkdir -p $(OBJDIR)
	$(CC) -O2 -fPIC -fvisibility=hidden -c -o $@ gen/vista_gen.c

$(PKG)/libvista.so: $(CU_OBJS) $(CPP_OBJS) $(OBJDIR)/vista_gen.o
	$(NVCC) $(ARCH) -shared -o $@ $^ -lcudart -ldl -lpthread

clean:
	rm -rf build gen/libvista_gen.so oracle/liboracle.so $(PKG)/libvista.so

.PHONY: all clean
