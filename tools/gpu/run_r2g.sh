#!/bin/bash
# round 2: full GPU tests, smoke, default bench (configs[2]) + reference arm
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2g_gputests.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2g_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2g_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r2g_smoke.log
timeout 1800 python bench.py > gpurun_out/r2g_bench.json 2> gpurun_out/r2g_bench.err; echo "bench rc=$?" >> gpurun_out/r2g_bench.err
tail -3 gpurun_out/r2g_gputests.log; tail -2 gpurun_out/r2g_smoke.log; tail -2 gpurun_out/r2g_bench.err; head -c 1500 gpurun_out/r2g_bench.json
# 2 ranks sharing the one GPU at a medium corpus: the N>1 bench path (placement, staged pulls, routing)
BAT_BENCH_SHARED_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 4 --warmup 3 --corpus 32768 --batch 32 --no-extras --no-cpu-baseline > gpurun_out/r2g_bench2.json 2> gpurun_out/r2g_bench2.err; echo "bench2 rc=$?" >> gpurun_out/r2g_bench2.err
tail -2 gpurun_out/r2g_bench2.err; head -c 1200 gpurun_out/r2g_bench2.json
