#!/bin/bash
# GPU tests + a short bench with the per-kernel table
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 400 python -m pytest tests -m "gpu and not slow" -q -x -p no:cacheprovider --timeout 150 --timeout-method=thread > gpurun_out/tb_tests.log 2>&1
echo "tests exit $?"; tail -3 gpurun_out/tb_tests.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/tb_bench.json 2> gpurun_out/tb_bench.err
echo "bench exit $?"
python - <<'PY'
import json
d=json.load(open('gpurun_out/tb_bench.json'))
print('value %.1f req/s  e2e %.1f  ms/step %.2f  alg TF %.0f  clocks %s' % (d['value'], d['e2e']['value'], d['ms_per_step'], d['algorithmic_tflops'], d['clocks']))
for k,v in d['kernels'].items(): print('  %-13s %7.3f ms  %s TF/s  %s GB/s' % (k, v['ms_per_step'], None if v['tflops'] is None else round(v['tflops']), None if v['gbs'] is None else round(v['gbs'])))
PY
tail -3 gpurun_out/tb_bench.err
