#!/bin/bash
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
for v in base sleep; do
  if [ $v = base ]; then L=""; else L="BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_$v.so"; fi
  echo "== $v"; env $L B=8 NU=8192 NI=20 ORDER=UP timeout 300 python tools/attn_timeline.py 2>&1 | sed -n 18,22p | cut -c1-240
  env $L timeout 900 python bench.py --steps 5 --warmup 2 --no-cpu-baseline --no-extras --workload cfg1-ip --corpus 8192 > gpurun_out/sl_$v.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/sl_$v.json').read().strip().splitlines()[-1]); print('$v', round(d['value'],1), round(d['attention']['tflops'],1), d['clocks']['sm_mhz'])"
done
