#!/bin/bash
# after the epilogue fixes: 8 epilogue warps for QKV + a4 (libbat_q8.so) and one staging buffer /
# one more ring stage for SwiGLU (libbat_s1.so) vs default, configs[2], same box
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
P=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200
for v in q8 s1; do BAT_LIB=$P/libbat_$v.so timeout 300 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_fused_epilogues.py -q -x -p no:cacheprovider -k "gemm or stage" 2>&1 | tail -1; done
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/e2_$tag.json 2>gpurun_out/e2_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/e2_$tag.json
}
for rep in 1 2; do
  run base_$rep X=1
  run q8_$rep BAT_LIB=$P/libbat_q8.so
  run s1_$rep BAT_LIB=$P/libbat_s1.so
done
