#!/bin/bash
# RMSNorm ln1 fused into the down GEMM epilogue (BAT_FUSED_NORM=d) vs standalone (0) vs both (1)
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
timeout 600 python -m pytest tests/test_gpu_fused_epilogues.py -q -x -p no:cacheprovider 2>&1 | tail -2
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/nd_$tag.json 2>gpurun_out/nd_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/nd_$tag.json
}
for rep in 1 2 3; do
  run none_$rep BAT_FUSED_NORM=0
  run d_$rep BAT_FUSED_NORM=d
done
for rep in 1 2; do
  run g16_$rep BAT_GEMM_GROUP_SWIGLU=16
  run g1_$rep BAT_GEMM_GROUP_SWIGLU=1
done
