#!/bin/bash
# h64 attention kernel: layer-level parity first (hard timeout: a deadlock must not hang the box),
# then the GEMM / fused-norm tests, then configs[2] A/B against the round-1 kernel (BAT_ATTN=v1)
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -p no:cacheprovider -k attention 2>&1 | tail -15
echo "attn-kernel-tests rc=$?"
timeout 600 python -m pytest tests/test_gpu_attn_fullbatch.py tests/test_gpu_attn_rescale.py -q -x -p no:cacheprovider 2>&1 | tail -8
timeout 600 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_fused_norm.py tests/test_gpu_parity.py -q -x -p no:cacheprovider 2>&1 | tail -8
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/h_$tag.json 2>gpurun_out/h_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/h_$tag.json
}
for rep in 1 2; do
  run h64_$rep X=1
  run v1_$rep BAT_ATTN=v1
done
BAT_ATTN_ITEMS=gpurun_out/items_h64.txt BAT_ATTN_LAYER=5 timeout 300 python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-extras --corpus 16384 > /dev/null 2> gpurun_out/items_h64.err
python tools/attn_items.py gpurun_out/items_h64.txt
