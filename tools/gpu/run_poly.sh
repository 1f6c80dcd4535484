#!/bin/bash
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
for v in p0 p8 p32; do
  echo "== $v"; BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_$v.so B=8 NU=8192 NI=20 ORDER=UP timeout 300 python tools/attn_timeline.py 2>&1 | sed -n 18,23p | cut -c1-240
done
echo "== p16"; B=8 NU=8192 NI=20 ORDER=UP timeout 300 python tools/attn_timeline.py 2>&1 | sed -n 18,23p | cut -c1-240
