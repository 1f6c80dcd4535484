#!/bin/bash
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
timeout 1500 python -m pytest -q -p no:cacheprovider tests/test_gpu_parity.py tests/test_gpu_kernels.py tests/test_gpu_pic.py tests/test_gpu_multidisc.py tests/test_gpu_edge.py tests/test_gpu_attn_fullbatch.py > gpurun_out/splitk_tests.log 2>&1
echo "rc=$?" >> gpurun_out/splitk_tests.log; tail -3 gpurun_out/splitk_tests.log
timeout 1200 python bench.py --steps 3 --warmup 2 --no-cpu-baseline > gpurun_out/splitk_bench.json 2> gpurun_out/splitk_bench.err
python -c "
import json; d=json.loads(open('gpurun_out/splitk_bench.json').read().strip().splitlines()[-1]); print(d['value'], d['extras']['batch1_ip_latency_ms'], d['extras']['cfg1-ip']['requests_per_s'])"
timeout 120 ./tools/chain_rate
