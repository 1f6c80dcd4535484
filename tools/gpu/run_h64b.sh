#!/bin/bash
# h64 diagnosis: LDTM / MUFU overlap microbenchmark, CTA-0 timelines (UP long items, configs[1] IP)
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
timeout 60 ./tools/ldtm_mufu
H64=1 B=8 NU=8192 NI=20 ORDER=UP timeout 300 python tools/attn_timeline.py 2>&1 | sed -n 1,60p | cut -c1-200
BAT_ATTN=v1 B=8 NU=8192 NI=20 ORDER=UP timeout 300 python tools/attn_timeline.py 2>&1 | sed -n 1,3p | cut -c1-200
