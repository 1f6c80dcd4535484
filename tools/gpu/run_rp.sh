#!/bin/bash
# relaxed P hand-off (libbat_rp.so) vs default, configs[2], same box
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
P=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200
BAT_LIB=$P/libbat_rp.so timeout 300 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_attn_rescale.py -q -x -p no:cacheprovider -k attention 2>&1 | tail -1
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/rp_$tag.json 2>gpurun_out/rp_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/rp_$tag.json
}
for rep in 1 2 3; do
  run base_$rep X=1
  run rp_$rep BAT_LIB=$P/libbat_rp.so
done
