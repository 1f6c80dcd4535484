#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_dbg.so timeout 300 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_edge.py -q -x -p no:cacheprovider 2>&1 | tail -1
for v in new old new; do
  if [ $v = new ]; then L=libbat.so; else L=libbat_old.so; fi
  BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/$L timeout 300 python bench.py --steps 6 --warmup 3 --no-cpu-baseline > gpurun_out/pref_$v.json 2>/dev/null
  python -c "import json;d=json.loads(open('gpurun_out/pref_$v.json').read().strip().splitlines()[-1]);print('$v attn', round(d['attention']['tflops'],1), 'req/s', round(d['value'],1), 'clk', d['clocks']['sm_mhz'])"
done
