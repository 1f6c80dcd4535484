#!/bin/bash
# A/B: softmax (and loader) warps waiting on their mbarriers with a suspend hint vs re-polling;
# then bench.py --gpus 2 with two ranks sharing the GPU at a medium corpus
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
for v in base ssleep allsleep; do
  if [ $v = base ]; then L=""; else L="BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_$v.so"; fi
  echo "== $v"; env $L B=8 NU=8192 NI=20 ORDER=UP timeout 300 python tools/attn_timeline.py 2>&1 | sed -n 18,22p | cut -c1-240
  for wl in cfg1-ip cfg2; do
    env $L timeout 900 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --workload $wl --corpus 16384 > gpurun_out/ss_${v}_$wl.json 2>/dev/null
    python -c "
import json; d=json.loads(open('gpurun_out/ss_${v}_$wl.json').read().strip().splitlines()[-1]); print('$v $wl', round(d['value'],1), round(d['attention']['tflops'],1), d['clocks']['sm_mhz'])"
  done
done
BAT_BENCH_SHARED_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 4 --warmup 3 --corpus 32768 --batch 32 --no-extras --no-cpu-baseline > gpurun_out/r2f_bench2.json 2> gpurun_out/r2f_bench2.err; echo "bench2 rc=$?"
tail -2 gpurun_out/r2f_bench2.err; head -c 1500 gpurun_out/r2f_bench2.json
