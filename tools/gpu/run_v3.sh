#!/bin/bash
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
timeout 600 python -m pytest -q -x -p no:cacheprovider tests/test_gpu_kernels.py -k attention > gpurun_out/v5d_kernels.log 2>&1
echo "rc=$?" >> gpurun_out/v5d_kernels.log; tail -3 gpurun_out/v5d_kernels.log
B=8 NU=8192 NI=20 ORDER=UP timeout 300 python tools/attn_timeline.py > gpurun_out/tl10_up.txt 2>&1
ORDER=IP timeout 300 python tools/attn_timeline.py > gpurun_out/tl10_ip.txt 2>&1
for f in gpurun_out/tl10_up.txt gpurun_out/tl10_ip.txt; do echo $f; head -1 $f; sed -n 20,24p $f | cut -c1-200; tail -1 $f; done
