# Build of the sdag library (libsdag.so, sm_100a) and the CPU oracle.
# `make -j` or __graft_entry__.build().
NVCC    ?= nvcc
PY      ?= python
PKG     := paper_conf_ipps_rawatvsrps19_b200
SRC     := $(PKG)/csrc
BUILD   := build
LIBDIR  := $(PKG)/lib
LIB     := $(LIBDIR)/libsdag.so
ARCH    := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -Wall -Iinclude -I$(SRC) -I$(BUILD) \
           --expt-relaxed-constexpr
CU_SRCS := k_jacobi7 k_lap25 k_smooth27 k_hypterm k_rhs4 k_toys runtime jit p2p profile
CC_SRCS := spec analysis registry dist capi program fission
OBJS    := $(addprefix $(BUILD)/,$(addsuffix .o,$(CU_SRCS) $(CC_SRCS)))
HDRS    := $(wildcard $(SRC)/*.hpp $(SRC)/*.cuh) include/sdag.h

all: $(LIB) oracle

$(BUILD)/specs_embed.inc: $(wildcard $(PKG)/specs/*.sdag) tools/embed_specs.py
	@mkdir -p $(BUILD)
	$(PY) tools/embed_specs.py $@ $(PKG)/specs

$(BUILD)/%.o: $(SRC)/%.cu $(HDRS)
	@mkdir -p $(BUILD)
	$(NVCC) $(NVFLAGS) -c $< -o $@

$(BUILD)/registry.o: $(BUILD)/specs_embed.inc

$(BUILD)/jit_embed.inc: $(SRC)/sweep.cuh tools/embed_text.py
	@mkdir -p $(BUILD)
	$(PY) tools/embed_text.py $@ kSweepSrc $(SRC)/sweep.cuh

$(BUILD)/jit_star_embed.inc: $(SRC)/star.cuh tools/embed_text.py
	@mkdir -p $(BUILD)
	$(PY) tools/embed_text.py $@ kStarSrc $(SRC)/star.cuh

$(BUILD)/jit.o: $(BUILD)/jit_embed.inc $(BUILD)/jit_star_embed.inc

$(BUILD)/%.o: $(SRC)/%.cpp $(HDRS)
	@mkdir -p $(BUILD)
	$(NVCC) $(NVFLAGS) -c $< -o $@

$(LIB): $(OBJS)
	@mkdir -p $(LIBDIR)
	$(NVCC) $(ARCH) -shared -o $@.tmp $(OBJS) -ldl -lpthread
	mv $@.tmp $@

oracle:
	$(PY) -c "import oracle; oracle.build()"

clean:
	rm -rf $(BUILD) $(LIB) oracle/liboracle.so

.PHONY: all oracle clean
