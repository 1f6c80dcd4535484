#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 300 python -m pytest tests/test_gpu_serving.py -q -x -s -p no:cacheprovider 2>&1 | tail -5
timeout 900 python tools/serve_trace.py > gpurun_out/serve_trace.json 2> gpurun_out/serve_trace.err
echo "serve exit $?"; cat gpurun_out/serve_trace.json | tail -7; tail -3 gpurun_out/serve_trace.err
