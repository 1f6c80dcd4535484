#!/bin/bash
# attention timelines v2 vs v1 (tools/attn_timeline.py), configs[1] IP batch
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
ORDER=IP timeout 300 python tools/attn_timeline.py > gpurun_out/tl2_v2.txt 2>&1
BAT_ATTN=v1 ORDER=IP timeout 300 python tools/attn_timeline.py > gpurun_out/tl2_v1.txt 2>&1
head -30 gpurun_out/tl2_v2.txt; tail -4 gpurun_out/tl2_v2.txt; head -3 gpurun_out/tl2_v1.txt; tail -4 gpurun_out/tl2_v1.txt
