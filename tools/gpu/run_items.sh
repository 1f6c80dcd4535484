#!/bin/bash
# per-work-item attention records on the real bench data (layer BAT_ATTN_LAYER) + softmax poly sweep
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
BAT_ATTN_ITEMS=gpurun_out/items_bench.txt BAT_ATTN_LAYER=${LAYER:-5} timeout 300 python bench.py --steps 2 --warmup 1 --no-cpu-baseline > /dev/null 2> gpurun_out/items_bench.err
echo "bench exit $?"; tail -2 gpurun_out/items_bench.err
python tools/attn_items.py gpurun_out/items_bench.txt
for pp in ${POLYS:-}; do echo "poly $pp"; timeout 60 ./tools/softmax_rate_p$pp | head -2; done
