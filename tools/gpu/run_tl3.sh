#!/bin/bash
# long full-tile items: UP with |U| = 8192 cached (64 full prefix k-tiles per item), v2 vs v1
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
B=8 NU=8192 NI=20 ORDER=UP timeout 300 python tools/attn_timeline.py > gpurun_out/tl3_v2.txt 2>&1
BAT_ATTN=v1 B=8 NU=8192 NI=20 ORDER=UP timeout 300 python tools/attn_timeline.py > gpurun_out/tl3_v1.txt 2>&1
for f in gpurun_out/tl3_v2.txt gpurun_out/tl3_v1.txt; do echo $f; head -1 $f; sed -n 20,30p $f | cut -c1-200; tail -3 $f; done
