#!/bin/bash
# round 2: the new GPU tests first, then everything
cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest -q -p no:cacheprovider -s tests/test_gpu_dist.py tests/test_gpu_score.py tests/test_gpu_plan_device.py tests/test_gpu_attn_fullbatch.py > gpurun_out/r2_new.log 2>&1
echo "new rc=$?" >> gpurun_out/r2_new.log
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r2_gputests.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_gputests.log
tail -3 gpurun_out/r2_new.log gpurun_out/r2_gputests.log
