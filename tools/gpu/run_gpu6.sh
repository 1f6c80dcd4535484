#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
for pp in 0 1; do
  (cd paper_conf_asplos_0017wzlxszh0w26_b200 && rm -f build/k_attn.o && make -j8 EXTRA_NVFLAGS=-DBAT_POLY_PAIRS=$pp > /dev/null 2>&1)
  echo "== poly pairs $pp"
  PP=$pp timeout 300 python tools/diag_tiny.py 2>&1 | tail -5
done
python -c "
import numpy as np
for k in ['IP_True','IP_False','UP_True']:
    a=np.load(f'gpurun_out/hf_{k}_0.npy'); b=np.load(f'gpurun_out/hf_{k}_1.npy')
    print(k,'pp0 vs pp1 max diff',np.abs(a-b).max())
"
