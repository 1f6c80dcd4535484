#!/bin/bash
# GEMM epilogue A/B on configs[2]: 8 epilogue warps (default) vs 4 (libbat_e4.so), fused RMSNorm
# on / off, SwiGLU on the CTA-pair kernel; then the fused-norm + kernel parity tests
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
L4=BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_e4.so
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/fu_$tag.json 2>gpurun_out/fu_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/fu_$tag.json
}
for rep in 1 2; do
  run e8_fuse_$rep X=1
  run e8_nofuse_$rep BAT_FUSED_NORM=0
  run e8_fuse_pair_$rep BAT_GEMM_SWIGLU_PAIR=1 BAT_GEMM_GROUP_SWIGLU=4
  run e8_nofuse_pair_$rep BAT_FUSED_NORM=0 BAT_GEMM_SWIGLU_PAIR=1 BAT_GEMM_GROUP_SWIGLU=4
  run e4_nofuse_$rep $L4 BAT_FUSED_NORM=0
done
timeout 1200 python -m pytest tests/test_gpu_fused_norm.py tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x -p no:cacheprovider 2>&1 | tail -5
