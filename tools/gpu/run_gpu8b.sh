#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
for pp in 0 2 8; do
  (cd paper_conf_asplos_0017wzlxszh0w26_b200 && rm -f build/k_attn.o && make -j8 EXTRA_NVFLAGS=-DBAT_POLY_PAIRS=$pp > /dev/null 2>&1)
  echo "== poly pairs $pp"
  timeout 300 python tools/attn_timeline.py 2>&1 | grep -E "stage\+attention|^   [45] "
done
