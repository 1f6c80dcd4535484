#!/bin/bash
# DBE softmax: the two teams' exp phases take turns (BAT_ATTN_SEQ=2, libbat_seqx.so) vs free overlap
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_seqx.so timeout 900 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_kernels.py tests/test_gpu_parity.py -k "attention or small or tiny" 2>&1 | tail -1
for v in base seqx base seqx; do
  if [ $v = base ]; then L=""; else L="BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_$v.so"; fi
  for wl in cfg1-ip cfg2; do
  env $L timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --workload $wl --corpus 16384 > gpurun_out/seqx_${v}_$wl.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/seqx_${v}_$wl.json').read().strip().splitlines()[-1]); print('$v $wl', round(d['value'],1), round(d['attention']['tflops'],1), d['clocks']['sm_mhz'])"
  done
done
BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_seqx.so B=8 NU=8192 NI=20 ORDER=UP timeout 300 python tools/attn_timeline.py 2>&1 | sed -n 1,24p | cut -c1-240
