#!/bin/bash
# batched MMA issue: attention parity, timelines, configs[2] A/B h64 vs v1
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -p no:cacheprovider -k attention 2>&1 | tail -3
BAT_ATTN=v1 timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -p no:cacheprovider -k attention 2>&1 | tail -3
H64=1 B=8 NU=8192 NI=20 ORDER=UP timeout 300 python tools/attn_timeline.py 2>&1 | sed -n 1,26p | cut -c1-250
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/h_$tag.json 2>gpurun_out/h_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/h_$tag.json
}
for rep in 1 2; do
  run h64b_$rep X=1
  run v1b_$rep BAT_ATTN=v1
done
