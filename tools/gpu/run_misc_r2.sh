#!/bin/bash
# compute-sanitizer over the round-2 GPU paths + other model shapes' bench lines
cd $GRAFT_REPO_ROOT
S=/usr/local/cuda/bin/compute-sanitizer
{
for tool in memcheck racecheck synccheck; do
  echo "=== $tool"
  timeout 1200 $S --tool $tool --print-limit 20 python -m pytest -q -p no:cacheprovider -x \
    tests/test_gpu_parity.py tests/test_gpu_pic.py tests/test_gpu_score.py "tests/test_gpu_kernels.py::test_attention_layer_small_gqa6" \
    "tests/test_gpu_dist.py::test_cold_pipeline_one_batch_ahead_overlaps_and_serves_identically" 2>&1 | grep -E "ERROR SUMMARY|passed|failed|Error" | tail -5
done
} > gpurun_out/r2_sanitizer.txt 2>&1
timeout 1200 python bench.py --model qwen2-7b --batch 16 --steps 3 --warmup 2 --no-cpu-baseline --no-extras --corpus 65536 > gpurun_out/r2_bench_7b.json 2> gpurun_out/r2_bench_7b.err
timeout 1200 python bench.py --model llama3-1b --steps 3 --warmup 2 --no-cpu-baseline --no-extras --corpus 65536 > gpurun_out/r2_bench_llama.json 2> gpurun_out/r2_bench_llama.err
cat gpurun_out/r2_sanitizer.txt; tail -c 400 gpurun_out/r2_bench_7b.json; tail -c 300 gpurun_out/r2_bench_7b.err; tail -c 400 gpurun_out/r2_bench_llama.json
