#!/bin/bash
# attention-kernel iteration: kernel tests + bench table
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 300 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py -q -x -p no:cacheprovider --timeout 120 --timeout-method=thread > gpurun_out/ta_tests.log 2>&1
echo "tests exit $?"; tail -3 gpurun_out/ta_tests.log; grep -E "worst|excess" gpurun_out/ta_tests.log | head -5
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/ta_bench.json 2> gpurun_out/ta_bench.err
echo "bench exit $?"
python - <<'PY'
import json
d=json.load(open('gpurun_out/ta_bench.json'))
print('value %.1f req/s  ms/step %.2f  clocks %s' % (d['value'], d['ms_per_step'], d['clocks']))
for k,v in d['kernels'].items(): print('  %-13s %7.3f ms  %s TF/s' % (k, v['ms_per_step'], None if v['tflops'] is None else round(v['tflops'])))
PY
tail -3 gpurun_out/ta_bench.err
