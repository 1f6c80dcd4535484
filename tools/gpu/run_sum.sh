#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_dbg.so timeout 300 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/seq_tests.log 2>&1
echo "dbg tests exit $?"; grep -E "mbar|passed|failed" gpurun_out/seq_tests.log | head -5
if grep -q " passed" gpurun_out/seq_tests.log && ! grep -q "failed" gpurun_out/seq_tests.log; then
for v in sum nosum; do
  if [ $v = sum ]; then L=libbat.so; else L=libbat_nosum.so; fi
  BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/$L timeout 300 python bench.py --steps 6 --warmup 3 --no-cpu-baseline > gpurun_out/seq_$v.json 2>/dev/null
  python -c "import json;d=json.loads(open('gpurun_out/seq_$v.json').read().strip().splitlines()[-1]);print('$v attn', round(d['attention']['tflops'],1), 'req/s', round(d['value'],1), 'clk', d['clocks']['sm_mhz'])"
done
fi
