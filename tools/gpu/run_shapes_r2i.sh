#!/bin/bash
# other model shapes on the final code: Qwen2-7B per-GPU share of configs[4] and the Llama3-1B head shape
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
timeout 1200 python bench.py --model qwen2-7b --batch 16 --steps 3 --warmup 2 --no-cpu-baseline --no-extras --corpus 65536 > gpurun_out/r2i_bench_7b.json 2> gpurun_out/r2i_bench_7b.err
python tools/bench_line.py 7b gpurun_out/r2i_bench_7b.json
timeout 1200 python bench.py --model llama3-1b --steps 3 --warmup 2 --no-cpu-baseline --no-extras --corpus 65536 > gpurun_out/r2i_bench_llama.json 2> gpurun_out/r2i_bench_llama.err
python tools/bench_line.py llama gpurun_out/r2i_bench_llama.json
