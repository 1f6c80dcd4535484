#!/bin/bash
cd $GRAFT_REPO_ROOT
for v in 2 4 6; do
  BAT_ATTN=pair BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_pp$v.so timeout 300 python bench.py --steps 4 --warmup 3 --no-cpu-baseline > gpurun_out/poly2_$v.json 2>/dev/null
  python -c "import json;d=json.loads(open('gpurun_out/poly2_$v.json').read().strip().splitlines()[-1]);print('pair poly $v', round(d['attention']['tflops'],1), round(d['value'],1))"
done
