#!/bin/bash
TAG=${1:-r1f}
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
ARGS="--steps 2 --warmup 1 --no-cpu-baseline --plans 1 --corpus 2048"
BAT_PROFILE_RANGE=1 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/launches_$TAG.csv python bench.py $ARGS > gpurun_out/ncu_list_$TAG.out 2>&1
echo "list exit $?"
BAT_PROFILE_RANGE=1 timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off -k regex:"attn|gemm|rmsnorm|stage" -c 9 -o gpurun_out/full_$TAG python bench.py $ARGS > gpurun_out/ncu_full_$TAG.out 2>&1
echo "full exit $?"
