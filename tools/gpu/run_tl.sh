#!/bin/bash
# attention timeline + per-item records (tools/attn_timeline.py)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
for o in IP UP; do ORDER=$o timeout 300 python tools/attn_timeline.py > gpurun_out/tl_$o.txt 2>&1; echo "$o exit $?"; head -3 gpurun_out/tl_$o.txt; tail -4 gpurun_out/tl_$o.txt; done
