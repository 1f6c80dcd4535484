#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
export BAT_PROFILE_RANGE=1
ARGS="--steps 1 --warmup 1 --no-cpu-baseline --plans 1 --corpus 2048"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off --csv --log-file gpurun_out/launches_r1.csv python bench.py $ARGS > gpurun_out/ncu_list.out 2>&1
echo "list exit $?"
timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off -k regex:attn_tc -c 1 -o gpurun_out/attn_r1 python bench.py $ARGS > gpurun_out/ncu_attn.out 2>&1
echo "attn exit $?"
timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off -k regex:gemm_tc -c 4 -o gpurun_out/gemm_r1 python bench.py $ARGS > gpurun_out/ncu_gemm.out 2>&1
echo "gemm exit $?"
ls -la gpurun_out
