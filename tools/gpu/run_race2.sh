#!/bin/bash
# racecheck over the parity set with the CTA-pair GEMM excluded (its only reports are in the
# system-reserved shared window touched by tcgen05.alloc.cta_group::2, see profiles/r2_racecheck.txt)
cd $GRAFT_REPO_ROOT
S=/usr/local/cuda/bin/compute-sanitizer
timeout 2400 $S --tool racecheck --racecheck-report all --print-limit 100 --kernel-name-exclude kns=gemm2_tc_kernel python -m pytest -q -p no:cacheprovider \
  tests/test_gpu_kernels.py tests/test_gpu_parity.py tests/test_gpu_fp32.py tests/test_gpu_pic.py tests/test_gpu_score.py \
  tests/test_gpu_multidisc.py tests/test_gpu_edge.py tests/test_gpu_graph.py > gpurun_out/r2_racecheck_nopair.log 2>&1
echo "racecheck(no pair gemm) rc=$?"
grep -E "RACECHECK SUMMARY|passed|failed" gpurun_out/r2_racecheck_nopair.log | tail -3
grep -A6 "Race reported\|hazard detected" gpurun_out/r2_racecheck_nopair.log | head -40
