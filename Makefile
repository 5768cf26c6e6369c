# Build libgsw.so (CUDA, sm_100a) + the C generator and oracle libraries (CPU).
NVCC ?= nvcc
PKG := paper_conf_ppopp_menglts19_b200
CSRC := $(PKG)/csrc
CU := $(wildcard $(CSRC)/*.cu)
HDR := $(wildcard $(CSRC)/*.cuh $(CSRC)/*.h) include/gsw.h
NCCL_INC ?= $(shell python3 -c "import nvidia.nccl, os; print(os.path.join(list(nvidia.nccl.__path__)[0], 'include'))" 2>/dev/null)
NVFLAGS := -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 \
           -Xcompiler -fPIC -Iinclude -I$(CSRC) -I$(NCCL_INC) --expt-relaxed-constexpr -Xptxas -v
LIB := $(PKG)/libgsw.so
OBJDIR := build/obj
OBJ := $(patsubst $(CSRC)/%.cu,$(OBJDIR)/%.o,$(CU))

all: $(LIB) gen/libgswgen.so oracle/liboracle.so cpu_baselines/libompbase.so

$(OBJDIR)/%.o: $(CSRC)/%.cu $(HDR)
	@mkdir -p $(OBJDIR)
	$(NVCC) $(NVFLAGS) -c $< -o $@ 2> $(OBJDIR)/$*.ptxas.txt || (cat $(OBJDIR)/$*.ptxas.txt; exit 1)

$(LIB): $(OBJ)
	$(NVCC) -gencode arch=compute_100a,code=sm_100a -shared -o $@ $(OBJ) -lcudart -ldl

gen/libgswgen.so: gen/gen.c
	gcc -O3 -fopenmp -fPIC -shared -o $@ $< -lm

oracle/liboracle.so: oracle/oracle.c
	gcc -O2 -fopenmp -fPIC -shared -o $@ $< -lm

cpu_baselines/libompbase.so: cpu_baselines/omp_bfs.c
	gcc -O3 -fopenmp -fPIC -shared -o $@ $<

# A/B variant of the library with another number of resident CTAs per SM for the persistent
# kernels (register budget 65536 / (256 * MINB)): build/var_m$(MINB)/libgsw.so, loaded with
# GSW_LIB_PATH=... for side-by-side timing
MINB ?= 3
variant:
	@mkdir -p build/var_m$(MINB)
	$(NVCC) $(NVFLAGS) -DGSW_MINB=$(MINB) -shared -o build/var_m$(MINB)/libgsw.so $(CU) -lcudart -ldl \
	    2> build/var_m$(MINB)/ptxas.txt || (tail -20 build/var_m$(MINB)/ptxas.txt; exit 1)

# A/B variant with arbitrary -D flags: make flagvariant VNAME=pb VFLAGS=-DGSW_PULL_BOUNDS=1
VNAME ?= x
VFLAGS ?=
flagvariant:
	@mkdir -p build/var_$(VNAME)
	$(NVCC) $(NVFLAGS) $(VFLAGS) -shared -o build/var_$(VNAME)/libgsw.so $(CU) -lcudart -ldl \
	    2> build/var_$(VNAME)/ptxas.txt || (tail -20 build/var_$(VNAME)/ptxas.txt; exit 1)

clean:
	rm -rf build $(LIB) gen/libgswgen.so oracle/liboracle.so cpu_baselines/libompbase.so

.PHONY: all clean
