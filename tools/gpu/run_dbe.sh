#!/bin/bash
cd $GRAFT_REPO_ROOT
BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_dbedbg.so timeout 300 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py -q -x -p no:cacheprovider 2>&1 | tail -1
for v in normal dbe normal dbe; do
  if [ $v = normal ]; then L=libbat.so; else L=libbat_dbe.so; fi
  BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/$L timeout 300 python bench.py --steps 4 --warmup 3 --no-cpu-baseline > gpurun_out/dbe_$v.json 2>/dev/null
  python -c "import json;d=json.loads(open('gpurun_out/dbe_$v.json').read().strip().splitlines()[-1]);print('$v attn', round(d['attention']['tflops'],1), 'clk', d['clocks']['sm_mhz'])"
done
