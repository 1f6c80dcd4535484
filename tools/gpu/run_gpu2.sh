#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 300 python -m pytest tests -m gpu -q -x -p no:cacheprovider --timeout 150 --timeout-method=thread > gpurun_out/gpu2_tests.log 2>&1
echo "tests exit $?" >> gpurun_out/gpu2_tests.log
tail -3 gpurun_out/gpu2_tests.log
timeout 600 python bench.py --steps 5 --warmup 3 --cpu-budget 10 > gpurun_out/bench2.json 2> gpurun_out/bench2.err
echo "bench exit $?"
cat gpurun_out/bench2.json; tail -20 gpurun_out/bench2.err
