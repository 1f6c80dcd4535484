#!/bin/bash
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
timeout 1500 python -m pytest -q -p no:cacheprovider -s tests/test_gpu_attn_fullbatch.py tests/test_gpu_parity.py tests/test_gpu_kernels.py tests/test_gpu_multidisc.py tests/test_gpu_fp32.py tests/test_gpu_edge.py > gpurun_out/split_tests.log 2>&1
echo "rc=$?" >> gpurun_out/split_tests.log
timeout 1200 python bench.py --steps 3 --warmup 2 --no-cpu-baseline > gpurun_out/split_bench.json 2> gpurun_out/split_bench.err
tail -3 gpurun_out/split_tests.log; grep "batch-1 work" gpurun_out/split_tests.log
python -c "
import json; d=json.loads(open('gpurun_out/split_bench.json').read().strip().splitlines()[-1]); print(d['value'], d['extras']['batch1_ip_latency_ms'], d['attention']['tflops'])"
bash tools/gpu/run_prof_r2.sh
