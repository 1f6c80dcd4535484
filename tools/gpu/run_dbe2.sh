#!/bin/bash
# decide-before-exp softmax (new default) vs single pass + vote (libbat_opt.so): parity + in-step A/B;
# CUDA-graph replay of bat_prefill_plan (default) vs BAT_GRAPH=0 on the batch-1 latency
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
timeout 900 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_graph.py tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_fp32.py tests/test_gpu_attn_fullbatch.py tests/test_gpu_pic.py 2>&1 | tail -2
for v in base opt base opt; do
  if [ $v = base ]; then L=""; else L="BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_$v.so"; fi
  for wl in cfg1-ip cfg2; do
    env $L timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --workload $wl --corpus 16384 > gpurun_out/dbe2_${v}_$wl.json 2>/dev/null
    python -c "
import json; d=json.loads(open('gpurun_out/dbe2_${v}_$wl.json').read().strip().splitlines()[-1]); print('$v $wl', round(d['value'],1), round(d['attention']['tflops'],1), d['clocks']['sm_mhz'])"
  done
done
for g in 1 0; do
  BAT_GRAPH=$g timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --corpus 16384 > gpurun_out/graph_$g.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/graph_$g.json').read().strip().splitlines()[-1]); e=d['extras']; print('graph=$g', round(d['value'],1), 'cfg1-ip', round(e['cfg1-ip']['requests_per_s'],1), 'batch1', e['batch1_ip_latency_ms'])"
done
env B=8 NU=8192 NI=20 ORDER=UP timeout 300 python tools/attn_timeline.py 2>&1 | sed -n 1,24p | cut -c1-240
bash tools/gpu/run_race2.sh
