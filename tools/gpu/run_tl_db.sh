#!/bin/bash
# double-buffered attention timeline (tools/attn_timeline_db.py), debug build guards against hangs
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
for o in IP; do ORDER=$o timeout 300 python tools/attn_timeline_db.py > gpurun_out/tldb_$o.txt 2>&1; echo "$o exit $?"; cat gpurun_out/tldb_$o.txt | head -80; done
