#!/bin/bash
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
nproc
timeout 1500 python -m pytest tests/test_gpu_fullsize.py -q -s -x -p no:cacheprovider --durations=5 2>&1 | grep -E "worst|passed|failed|Error|assert|slowest|s call" | head -30
