#!/bin/bash
# next-tile row lookups prefetched (plan per-row record) vs the previous build
# previous build (libbat_prev.so), configs[2], same box; then the GEMM / fused / parity tests
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
P=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/pf_$tag.json 2>gpurun_out/pf_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/pf_$tag.json
}
for rep in 1 2 3; do
  run new_$rep X=1
  run prev_$rep BAT_LIB=$P/libbat_prev.so
done
timeout 900 python -m pytest tests/test_gpu_fused_epilogues.py tests/test_gpu_parity.py tests/test_gpu_plan_device.py tests/test_gpu_pic.py tests/test_gpu_multidisc.py -q -x -p no:cacheprovider 2>&1 | tail -2
