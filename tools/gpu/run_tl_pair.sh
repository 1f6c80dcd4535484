#!/bin/bash
# double-buffered attention timeline (tools/attn_timeline_pair.py), debug build guards against hangs
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
for o in IP; do BAT_ATTN=pair ORDER=$o timeout 120 python tools/attn_timeline_pair.py > gpurun_out/tlpair_$o.txt 2>&1; echo "$o exit $?"; cat gpurun_out/tlpair_$o.txt | head -80; done
