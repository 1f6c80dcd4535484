#!/bin/bash
# DBE softmax: exp2 FMA-pipe share sweep (BAT_POLY_PAIRS 0 / 2 (default) / 4) + instrumented timeline
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
for v in base dbep0 dbep4 base dbep0 dbep4; do
  if [ $v = base ]; then L=""; else L="BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_$v.so"; fi
  env $L timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --workload cfg2 --corpus 16384 > gpurun_out/dbe3_${v}.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/dbe3_${v}.json').read().strip().splitlines()[-1]); print('$v cfg2', round(d['value'],1), round(d['attention']['tflops'],1), d['clocks']['sm_mhz'])"
done
env B=8 NU=8192 NI=20 ORDER=UP timeout 300 python tools/attn_timeline.py 2>&1 | sed -n 1,30p | cut -c1-240
