#!/bin/bash
# fused ln1 producer: xg stores after the h_new TMA flush (libbat_xo.so) vs default, configs[2]
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
P=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200
BAT_LIB=$P/libbat_xo.so timeout 600 python -m pytest tests/test_gpu_fused_epilogues.py -q -x -p no:cacheprovider -k norm 2>&1 | tail -1
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/xo_$tag.json 2>gpurun_out/xo_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/xo_$tag.json
}
for rep in 1 2 3; do
  run base_$rep X=1
  run xo_$rep BAT_LIB=$P/libbat_xo.so
done
