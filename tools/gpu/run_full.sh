#!/bin/bash
# full-size sampled parity (tests/test_gpu_fullsize.py)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
nproc
timeout 2400 python -m pytest tests/test_gpu_fullsize.py -q -s -x -p no:cacheprovider --durations=5 > gpurun_out/full.log 2>&1
echo "exit $?"
grep -E "worst|passed|failed|Error|assert|slowest|s call" gpurun_out/full.log | head -30
