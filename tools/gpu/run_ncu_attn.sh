#!/bin/bash
# ncu --set full of the attention kernel (one launch) on the configs[1] IP batch, v2 and v1
cd $GRAFT_REPO_ROOT
for v in v2 v1; do
  BAT_ATTN=$v timeout 600 ncu --set full --clock-control none --import-source on -k regex:attn_ -s 2 -c 1 \
    -o gpurun_out/attn_$v python tools/attn_layer_run.py > gpurun_out/ncu_attn_$v.log 2>&1
done
ls -la gpurun_out/*.ncu-rep
