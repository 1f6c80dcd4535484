#!/bin/bash
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
H64=1 B=8 NU=8192 NI=20 ORDER=UP timeout 300 python tools/attn_timeline.py 2>&1 | sed -n 1,30p | cut -c1-250
H64=1 B=64 NU=512 NI=100 ORDER=IP timeout 300 python tools/attn_timeline.py 2>&1 | sed -n 1,30p | cut -c1-250
