#!/bin/bash
# rasterisation group of the QKV / O / down pair GEMMs (BAT_GEMM_GROUP_M, default 1), configs[2]
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/gm_$tag.json 2>gpurun_out/gm_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/gm_$tag.json
}
for rep in 1 2; do
  run g1_$rep X=1
  run g2_$rep BAT_GEMM_GROUP_M=2
  run g4_$rep BAT_GEMM_GROUP_M=4
done
