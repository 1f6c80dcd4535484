#!/bin/bash
# GEMM epilogue warps for the residual (O, down) and QKV GEMMs: 4 (default) vs 8 with one staging buffer
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
P=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200
for v in r8 q8; do BAT_LIB=$P/libbat_$v.so timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -p no:cacheprovider -k "gemm" 2>&1 | tail -1; done
timeout 300 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_fused_norm.py -q -x -p no:cacheprovider 2>&1 | tail -1
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/ew_$tag.json 2>gpurun_out/ew_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/ew_$tag.json
}
for rep in 1 2; do
  run base_$rep X=1
  run r8_$rep BAT_LIB=$P/libbat_r8.so
  run q8_$rep BAT_LIB=$P/libbat_q8.so
done
