#!/bin/bash
# build an experiment variant of libbat.so: tools/build_variant.sh NAME "-DFLAG=..." -> paper_.../libbat_NAME.so
set -e
cd "$(dirname "$0")/../paper_conf_asplos_0017wzlxszh0w26_b200"
make -s BUILD=build_$1 EXTRA_NVFLAGS="$2" build_$1/api.o build_$1/plan.o build_$1/sched.o build_$1/k_gemm.o build_$1/k_attn.o build_$1/k_misc.o build_$1/k_f32.o
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o libbat_$1.so build_$1/*.o -Xlinker --version-script=csrc/exports.map
echo built libbat_$1.so
