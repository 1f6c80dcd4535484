#!/bin/bash
# batched MMA issue x FMA-pipe exp2 share (BAT_POLY_PAIRS of 16) vs the default, configs[2], same box
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
P=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200
for v in bip6 bip8; do BAT_LIB=$P/libbat_$v.so timeout 300 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_attn_rescale.py -q -x -p no:cacheprovider -k "attention" 2>&1 | tail -1; done
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/bp_$tag.json 2>gpurun_out/bp_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/bp_$tag.json
}
for rep in 1 2; do
  run base_$rep X=1
  run bip4_$rep BAT_LIB=$P/libbat_bip4.so
  run bip6_$rep BAT_LIB=$P/libbat_bip6.so
  run bip8_$rep BAT_LIB=$P/libbat_bip8.so
done
