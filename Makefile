# Build every native artefact in-tree (the .so files travel to the GPU box with gpurun).
NVCC      ?= nvcc
PKG       := paper_conf_asplos_finglertyshar23_b200
CSRC      := $(PKG)/csrc
LIB       := $(PKG)/liblake_linnos.so
ORACLE    := oracle/liblake_oracle.so
TRACESIM  := $(PKG)/inputs/libtracesim.so
ARCH      := -gencode arch=compute_100a,code=sm_100a
# --fmad=false: no implicit mul+add contraction anywhere (FP32 path is bit-exact, R15)
NVFLAGS   := $(ARCH) -O3 -lineinfo -std=c++17 --fmad=false -Xcompiler -fPIC,-O2 \
             -Xptxas -v --expt-relaxed-constexpr
SRCS      := $(CSRC)/api.cu $(CSRC)/digitize.cu $(CSRC)/mlp_fp32.cu $(CSRC)/mlp_tc.cu $(CSRC)/group.cu $(CSRC)/capture.cu $(CSRC)/sort.cu $(CSRC)/server.cu $(CSRC)/mlp_family.cu $(CSRC)/deferred.cu
HDRS      := $(wildcard $(CSRC)/*.h $(CSRC)/*.cuh) include/lake_linnos.h include/lake_mlp.h
OBJS      := $(patsubst $(CSRC)/%.cu,build/%.o,$(SRCS))

all: $(LIB) $(ORACLE) $(TRACESIM)

build/%.o: $(CSRC)/%.cu $(HDRS)
	@mkdir -p build
	$(NVCC) $(NVFLAGS) -c $< -o $@ 2> build/$*.ptxas.log || (cat build/$*.ptxas.log; false)

$(LIB): $(OBJS)
	$(NVCC) $(ARCH) -shared -o $@ $(OBJS) -lcudart

$(ORACLE): oracle/lake_oracle.c
	gcc -std=gnu99 -O2 -mfma -ffp-contract=off -fno-fast-math -fopenmp -shared -fPIC -o $@ $< -lm

$(TRACESIM): $(PKG)/inputs/tracesim.c
	gcc -std=gnu99 -O2 -shared -fPIC -o $@ $<

clean:
	rm -rf build $(LIB) $(ORACLE) $(TRACESIM)

.PHONY: all clean

# timeline-trace build (development only; not loaded by the product path)
TRACE_LIB := build/trace/liblake_linnos_trace.so
trace: $(TRACE_LIB)
$(TRACE_LIB): $(SRCS) $(HDRS)
	@mkdir -p build/trace
	$(NVCC) $(NVFLAGS) -DLAKE_TRACE -shared -o $@ $(SRCS) -lcudart 2> build/trace/ptxas.log || (cat build/trace/ptxas.log; false)
.PHONY: trace

# A/B variants of the fused kernel (development): make variant VAR=name DEFS="-D..."
variant:
	@mkdir -p build/var/$(VAR)
	$(NVCC) $(NVFLAGS) $(DEFS) -shared -o build/var/$(VAR)/liblake_linnos.so $(SRCS) -lcudart 2> build/var/$(VAR)/ptxas.log || (cat build/var/$(VAR)/ptxas.log; false)
.PHONY: variant
