#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
ARGS="--steps 2 --warmup 1 --no-cpu-baseline --plans 1 --corpus 2048"
BAT_PROFILE_RANGE=1 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/launches_r1b.csv python bench.py $ARGS > gpurun_out/ncu_list.out 2>&1
echo "list exit $?"
BAT_PROFILE_RANGE=1 timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off -k regex:"attn_tc|gemm_tc" -c 5 -o gpurun_out/full_r1 python bench.py $ARGS > gpurun_out/ncu_full.out 2>&1
echo "full exit $?"
timeout 900 python bench.py > gpurun_out/bench_r1.json 2> gpurun_out/bench_r1.err
echo "bench exit $?"; cat gpurun_out/bench_r1.json | head -c 3000
