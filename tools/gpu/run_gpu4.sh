#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 300 python -m pytest tests -m gpu -q -x -p no:cacheprovider --timeout 120 --timeout-method=thread > gpurun_out/gpu4_tests.log 2>&1
echo "tests exit $?"
tail -15 gpurun_out/gpu4_tests.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench4.json 2> gpurun_out/bench4.err
echo "bench exit $?"
python -c "
import json; d=json.load(open('gpurun_out/bench4.json'))
print('value',d['value'],'ms/step',d['ms_per_step'],'alg TF',d['algorithmic_tflops'])
print('attn',d['attention'])
for k,v in d['kernels'].items(): print(k, v)
"
tail -5 gpurun_out/bench4.err
