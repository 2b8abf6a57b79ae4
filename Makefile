# libugraph.so -- sm_100a only.  No --use_fast_math: IEEE div/sqrt, explicit _rn intrinsics
# keep every message rounded once (R11).
NVCC    ?= /usr/local/cuda/bin/nvcc
PKG     := paper_conf_asplos_0001lslwlgslllw23_b200
SRC     := $(PKG)/csrc
BUILD   := build
LIB     := $(PKG)/libugraph.so
ARCH    := -gencode arch=compute_100a,code=sm_100a
NVFLAGS := $(ARCH) -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -prec-div=true -prec-sqrt=true -fmad=true \
           -Iinclude -I$(SRC) -Xptxas -v $(EXTRA)
CU      := $(wildcard $(SRC)/*.cu)
CPP     := $(wildcard $(SRC)/*.cpp)
OBJ     := $(patsubst $(SRC)/%.cu,$(BUILD)/%.o,$(CU)) $(patsubst $(SRC)/%.cpp,$(BUILD)/%.o,$(CPP))
HDR     := $(wildcard $(SRC)/*.h $(SRC)/*.cuh) include/ug.h

all: $(LIB) oracle/libugoracle.so

$(BUILD)/%.o: $(SRC)/%.cu $(HDR)
	@mkdir -p $(BUILD)
	$(NVCC) $(NVFLAGS) -c $< -o $@ > $(BUILD)/$*.ptxas.log 2>&1 || (cat $(BUILD)/$*.ptxas.log; false)

$(BUILD)/%.o: $(SRC)/%.cpp $(HDR)
	@mkdir -p $(BUILD)
	$(NVCC) $(NVFLAGS) -x cu -c $< -o $@ > $(BUILD)/$*.ptxas.log 2>&1 || (cat $(BUILD)/$*.ptxas.log; false)

$(LIB): $(OBJ)
	$(NVCC) $(ARCH) -shared -o $@ $(OBJ) -ldl

oracle/libugoracle.so: oracle/ug_oracle.c
	gcc -O2 -ffp-contract=off -fno-fast-math -fPIC -shared -o $@ $< -lm

clean:
	rm -rf $(BUILD) $(LIB) oracle/libugoracle.so

.PHONY: all clean
