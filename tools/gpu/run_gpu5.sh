#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
export BAT_PROFILE_RANGE=1
ARGS="--steps 1 --warmup 1 --no-cpu-baseline --plans 1 --corpus 2048"
timeout 900 ncu --set full --import-source on --clock-control none --profile-from-start off -k regex:attn_tc -c 1 -o gpurun_out/attn_r4 python bench.py $ARGS > gpurun_out/ncu_attn4.out 2>&1
echo "attn exit $?"
