#!/bin/bash
# DRAM bytes per launch of the CTA-pair GEMMs (O, down) vs their rasterisation group
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for g in 1 4 8 32; do
BAT_GEMM_GROUP_M=$g BAT_PROFILE_RANGE=1 timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none --profile-from-start off -k regex:"gemm2" -c 6 --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --plans 1 --corpus 2048 > gpurun_out/dt_ncu_$g.csv 2>/dev/null
echo "ncu g=$g exit $?"
done
