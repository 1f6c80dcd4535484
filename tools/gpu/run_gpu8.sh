#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 300 python -m pytest tests -m gpu -q -x -p no:cacheprovider --timeout 120 --timeout-method=thread 2>&1 | tail -3
timeout 300 python tools/attn_timeline.py 2>&1 | grep -E "stage\+attention|^   [3456] "
ORDER=UP timeout 300 python tools/attn_timeline.py 2>&1 | grep -E "stage\+attention"
