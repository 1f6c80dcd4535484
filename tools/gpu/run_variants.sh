#!/bin/bash
# per-work-item attention records on the bench data for several library builds (VARIANTS="a b"),
# plus the CTA-0 timeline of the default build
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
P=paper_conf_asplos_0017wzlxszh0w26_b200
for v in default ${VARIANTS}; do
  if [ "$v" = default ]; then lib=$P/libbat.so; else lib=$P/libbat_$v.so; fi
  BAT_LIB=$PWD/$lib BAT_ATTN_ITEMS=gpurun_out/items_$v.txt BAT_ATTN_LAYER=5 timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu-baseline > gpurun_out/bench_$v.json 2> gpurun_out/bench_$v.err
  echo "== $v exit $? attention ms/step $(python -c "import json;d=json.load(open('gpurun_out/bench_$v.json'));print(round(d['kernels']['attention']['ms_per_step'],3), round(d['attention']['tflops']))")"
  python tools/attn_items.py gpurun_out/items_$v.txt | tail -2
done
ORDER=IP timeout 300 python tools/attn_timeline.py > gpurun_out/tl_IP.txt 2>&1
