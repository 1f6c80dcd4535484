#!/bin/bash
# round 2: full GPU tests, smoke, default bench (configs[2]) + reference arm
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2f_gputests.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2f_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2f_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r2f_smoke.log
timeout 1800 python bench.py > gpurun_out/r2f_bench.json 2> gpurun_out/r2f_bench.err; echo "bench rc=$?" >> gpurun_out/r2f_bench.err
tail -3 gpurun_out/r2f_gputests.log; tail -2 gpurun_out/r2f_smoke.log; tail -2 gpurun_out/r2f_bench.err; head -c 1500 gpurun_out/r2f_bench.json
