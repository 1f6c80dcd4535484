#!/bin/bash
cd $GRAFT_REPO_ROOT
for v in 2 0 4 2; do
  if [ $v = 2 ]; then L=libbat.so; else L=libbat_pp$v.so; fi
  BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/$L timeout 300 python bench.py --steps 4 --warmup 3 --no-cpu-baseline > gpurun_out/poly3_$v.json 2>/dev/null
  python -c "import json;d=json.loads(open('gpurun_out/poly3_$v.json').read().strip().splitlines()[-1]);print('poly $v attn', round(d['attention']['tflops'],1), 'clk', d['clocks']['sm_mhz'])"
done
