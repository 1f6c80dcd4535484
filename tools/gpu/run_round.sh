#!/bin/bash
# One GPU session: build check, -m gpu tests, smoke, bench (N=1), ncu launch list, ncu full
# capture of the attention + GEMM kernels.  Usage: run_round.sh TAG
TAG=${1:-r1}
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/gpu_$TAG.txt
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider --durations=8 > gpurun_out/tests_$TAG.log 2>&1
echo "tests exit $?"; tail -15 gpurun_out/tests_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
echo "smoke exit $?"; tail -2 gpurun_out/smoke_$TAG.log
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
echo "bench exit $?"; head -c 4000 gpurun_out/bench_$TAG.json; tail -3 gpurun_out/bench_$TAG.err
ARGS="--steps 2 --warmup 1 --no-cpu-baseline --plans 1 --corpus 2048"
BAT_PROFILE_RANGE=1 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/launches_$TAG.csv python bench.py $ARGS > gpurun_out/ncu_list_$TAG.out 2>&1
echo "list exit $?"
BAT_PROFILE_RANGE=1 timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off -k regex:"attn|gemm" -c 8 -o gpurun_out/full_$TAG python bench.py $ARGS > gpurun_out/ncu_full_$TAG.out 2>&1
echo "full exit $?"
