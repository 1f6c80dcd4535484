#!/bin/bash
# same-box A/B of the attention MMA issue: per-MMA elect (default) vs batched (libbat_bi.so) vs batched +
# 4/16 FMA-pipe exp2 pairs (libbat_p4.so); three interleaved reps each, configs[2]
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
P=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200
BAT_LIB=$P/libbat_bi.so timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -p no:cacheprovider -k attention 2>&1 | tail -1
BAT_LIB=$P/libbat_p4.so timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -p no:cacheprovider -k attention 2>&1 | tail -1
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/bi_$tag.json 2>gpurun_out/bi_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/bi_$tag.json
}
for rep in 1 2 3; do
  run base_$rep X=1
  run bi_$rep BAT_LIB=$P/libbat_bi.so
  run p4_$rep BAT_LIB=$P/libbat_p4.so
done
