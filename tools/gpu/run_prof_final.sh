#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
ARGS="--steps 2 --warmup 1 --no-cpu-baseline --plans 1 --corpus 2048"
BAT_PROFILE_RANGE=1 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/launches_r1f.csv python bench.py $ARGS > gpurun_out/ncu_list_r1f.out 2>&1
echo "list exit $?"
BAT_PROFILE_RANGE=1 timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off -k regex:"attn|gemm|rmsnorm|stage" -c 9 -o gpurun_out/full_r1f python bench.py $ARGS > gpurun_out/ncu_full_r1f.out 2>&1
echo "full exit $?"
