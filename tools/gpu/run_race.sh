#!/bin/bash
# compute-sanitizer racecheck over the parity set, full report kept (round 2 final)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
S=/usr/local/cuda/bin/compute-sanitizer
timeout 2400 $S --tool racecheck --racecheck-report all --print-limit 400 python -m pytest -q -p no:cacheprovider \
  tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_fp32.py tests/test_gpu_pic.py tests/test_gpu_score.py \
  tests/test_gpu_multidisc.py tests/test_gpu_edge.py > gpurun_out/r2_racecheck_full.log 2>&1
echo "racecheck rc=$?"
grep -E "ERROR SUMMARY|RACECHECK SUMMARY|passed|failed" gpurun_out/r2_racecheck_full.log | tail -5
grep -A8 "Race reported" gpurun_out/r2_racecheck_full.log | head -80
