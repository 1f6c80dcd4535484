#!/bin/bash
# SwiGLU GEMM: 1-CTA 128x256 tiles (default) vs the CTA-pair kernel (256x256 per pair) at several
# rasterisation groups (BAT_GEMM_GROUP_SWIGLU, in M-tiles of the kernel used); configs[2] bench
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/sw_$tag.json 2>gpurun_out/sw_$tag.err
  python - "$tag" <<'PY'
import json, sys
tag = sys.argv[1]
d = json.loads(open(f'gpurun_out/sw_{tag}.json').read().strip().splitlines()[-1])
k = d['kernels']
print(tag, 'req/s', round(d['value'], 1), 'gate_up TF', round(k['gemm_gate_up']['tflops'], 1), 'ms', round(k['gemm_gate_up']['ms_per_step'], 2),
      'down TF', round(k['gemm_down']['tflops'], 1), 'attn TF', round(d['attention']['tflops'], 1), 'MHz', d['clocks']['sm_mhz'], flush=True)
PY
}
for rep in 1 2; do
  run base$rep X=1
  run p1_$rep BAT_GEMM_SWIGLU_PAIR=1 BAT_GEMM_GROUP_SWIGLU=1
  run p4_$rep BAT_GEMM_SWIGLU_PAIR=1 BAT_GEMM_GROUP_SWIGLU=4
  run p16_$rep BAT_GEMM_SWIGLU_PAIR=1 BAT_GEMM_GROUP_SWIGLU=16
done
# per-work-item attention records of one layer of the configs[2] step
BAT_ATTN_ITEMS=gpurun_out/items_cfg2.txt BAT_ATTN_LAYER=5 timeout 300 python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-extras --corpus 16384 > /dev/null 2> gpurun_out/items_cfg2.err
python tools/attn_items.py gpurun_out/items_cfg2.txt
