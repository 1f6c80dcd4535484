#!/bin/bash
# round 2 profiles of the default bench (configs[2] batch 64, 262,144-item corpus): launch list of the timed
# region + one --set full capture of the first launch of each hot kernel
cd $GRAFT_REPO_ROOT
export BAT_PROFILE_RANGE=1
timeout 1500 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_r2.csv python bench.py --steps 1 --warmup 1 --plans 2 --no-cpu-baseline --no-extras > gpurun_out/r2_prof_bench1.log 2>&1
timeout 1500 ncu --profile-from-start off --set full --clock-control none --import-source on \
  -k regex:"gemm_tc_kernel|gemm2_tc_kernel|attn_tc_kernel" -c 6 -o gpurun_out/full_r2 \
  python bench.py --steps 1 --warmup 1 --plans 2 --no-cpu-baseline --no-extras > gpurun_out/r2_prof_bench2.log 2>&1
ls -la gpurun_out/launches_r2.csv gpurun_out/full_r2.ncu-rep
