#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.used --format=csv > gpurun_out/smi.txt 2>&1
export PYTHONUNBUFFERED=1
for t in "test_gpu_kernels.py -k gemm" "test_gpu_kernels.py -k kv_append" "test_gpu_kernels.py -k attention" "test_gpu_parity.py"; do
  echo "=== $t" >> gpurun_out/gpu1.log
  timeout 420 python -m pytest tests/$t -q -x -p no:cacheprovider --timeout 150 --timeout-method=thread >> gpurun_out/gpu1.log 2>&1
  echo "exit $?" >> gpurun_out/gpu1.log
done
tail -c 20000 gpurun_out/gpu1.log
