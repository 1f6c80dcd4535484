#!/bin/bash
# exp2 MUFU/FMA split sweep for both attention kernels (bench attention TFLOP/s)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for v in 0 2 8; do
  for k in pair tc; do
    if [ $k = tc ]; then E="BAT_ATTN=tc"; else E=""; fi
    env $E BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_pp$v.so timeout 300 python bench.py --steps 4 --warmup 3 --no-cpu-baseline > gpurun_out/poly_${k}_$v.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/poly_${k}_$v.json').read().strip().splitlines()[-1]);print('$k poly $v', round(d['attention']['tflops'],1), round(d['value'],1))"
  done
done
