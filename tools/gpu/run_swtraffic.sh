#!/bin/bash
# SwiGLU GEMM DRAM traffic vs rasterisation group (pair M-tiles) and L2 hints (1: evict_last weights,
# 3: + evict_first act stores): configs[2] step time + ncu dram bytes of one gate/up launch
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/sw2_$tag.json 2>gpurun_out/sw2_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/sw2_$tag.json
}
for cfg in "g16h1 BAT_GEMM_GROUP_SWIGLU=16 BAT_GEMM_HINTS=1" "g32h1 BAT_GEMM_GROUP_SWIGLU=32 BAT_GEMM_HINTS=1" "g64h1 BAT_GEMM_GROUP_SWIGLU=64 BAT_GEMM_HINTS=1" "g16h3 BAT_GEMM_GROUP_SWIGLU=16 BAT_GEMM_HINTS=3" "g32h3 BAT_GEMM_GROUP_SWIGLU=32 BAT_GEMM_HINTS=3"; do
  set -- $cfg; tag=$1; shift
  run ${tag}_a "$@"; run ${tag}_b "$@"
  env "$@" BAT_PROFILE_RANGE=1 timeout 600 ncu --profile-from-start off --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
    --clock-control none -k regex:gemm2_tc_kernel --launch-skip 2 --launch-count 1 --csv \
    python bench.py --steps 1 --warmup 1 --plans 2 --no-cpu-baseline --no-extras --corpus 16384 2>/dev/null | grep -E 'dram__bytes|gpu__time' | awk -F'","' -v t=$tag '{print t, $(NF-2), $(NF-1), $NF}'
done
