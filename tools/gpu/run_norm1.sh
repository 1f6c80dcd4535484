#!/bin/bash
# fused ln2 through the O GEMM with h_old prefetched 4 chunks ahead: BAT_FUSED_NORM=1 vs d (default) vs 0
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
timeout 600 python -m pytest tests/test_gpu_fused_epilogues.py tests/test_gpu_kernels.py -q -x -p no:cacheprovider 2>&1 | tail -2
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/n1_$tag.json 2>gpurun_out/n1_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/n1_$tag.json
}
for rep in 1 2; do
  run d_$rep X=1
  run both_$rep BAT_FUSED_NORM=1
  run none_$rep BAT_FUSED_NORM=0
done
