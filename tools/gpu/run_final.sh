#!/bin/bash
# end-of-round validation: every GPU test, smoke, the default bench line
TAG=${1:-final}
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 2000 python -m pytest tests -m gpu -q -p no:cacheprovider --durations=5 > gpurun_out/tests_$TAG.log 2>&1
echo "tests exit $?"; tail -12 gpurun_out/tests_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
echo "smoke exit $?"; tail -1 gpurun_out/smoke_$TAG.log
timeout 900 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
echo "bench exit $?"; python -c "import json;d=json.loads(open('gpurun_out/bench_$TAG.json').read().strip().splitlines()[-1]);print(d['value'], d['e2e']['value'], d['roofline']['frac'], d['attention']['tflops'], d['mfu'], d['clocks'])"
