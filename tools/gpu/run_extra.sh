#!/bin/bash
# new-feature GPU tests + extra model-shape bench lines
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests/test_gpu_multidisc.py tests/test_gpu_fp32.py tests/test_gpu_parity.py tests/test_gpu_serving.py tests/test_gpu_attn_variants.py -q -x -s -p no:cacheprovider > gpurun_out/extra_tests.log 2>&1
echo "tests exit $?"; grep -E "worst|passed|failed|Error" gpurun_out/extra_tests.log | tail -25
timeout 600 python bench.py --model llama3-1b --steps 6 --warmup 3 --no-cpu-baseline > gpurun_out/bench_llama.json 2> gpurun_out/bench_llama.err
echo "llama exit $?"; tail -c 1500 gpurun_out/bench_llama.json; tail -2 gpurun_out/bench_llama.err
timeout 900 python bench.py --model qwen2-7b --n-user 2048 --n-items 200 --batch 16 --corpus 4096 --steps 4 --warmup 3 --no-cpu-baseline > gpurun_out/bench_7b.json 2> gpurun_out/bench_7b.err
echo "7b exit $?"; tail -c 1500 gpurun_out/bench_7b.json; tail -2 gpurun_out/bench_7b.err
