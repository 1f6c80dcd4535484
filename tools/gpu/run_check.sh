#!/bin/bash
# full check: GPU test suite + default bench line
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout 1200 --timeout-method=thread -rs -s > gpurun_out/chk_tests.log 2>&1
echo "tests exit $?"; grep -E "worst|passed|failed|Error" gpurun_out/chk_tests.log | tail -12
timeout 600 python bench.py ${BENCH_ARGS} > gpurun_out/chk_bench.json 2> gpurun_out/chk_bench.err
echo "bench exit $?"
python - <<'PY'
import json
d=json.load(open('gpurun_out/chk_bench.json'))
print('value %.1f req/s  ms/step %.2f  e2e %s clocks %s' % (d['value'], d['ms_per_step'], d['e2e']['value'], d['clocks']))
print('roofline', d['roofline'])
for k,v in d['kernels'].items(): print('  %-13s %7.3f ms  %s TF/s' % (k, v['ms_per_step'], None if v['tflops'] is None else round(v['tflops'])))
PY
tail -3 gpurun_out/chk_bench.err
