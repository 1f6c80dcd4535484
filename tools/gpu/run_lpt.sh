#!/bin/bash
cd $GRAFT_REPO_ROOT
for cfg in "3 8" "4 8" "4 4" "4 16"; do
  set -- $cfg
  BAT_LPT_SINGLE=$1 BAT_LPT_ITEM=$2 timeout 300 python bench.py --steps 6 --warmup 3 --no-cpu-baseline > gpurun_out/lpt_$1_$2.json 2>/dev/null
  python -c "import json;d=json.loads(open('gpurun_out/lpt_$1_$2.json').read().strip().splitlines()[-1]);print('single $1 item $2: attn', round(d['attention']['tflops'],1), 'attn ms', round(d['attention']['ms_per_step'],2), 'req/s', round(d['value'],1), 'clk', d['clocks']['sm_mhz'])"
done
