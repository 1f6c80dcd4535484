#!/bin/bash
# compute-sanitizer over the round-2 fused epilogues (a4 in the QKV epilogue, RMSNorm producer /
# consumer, SwiGLU on CTA pairs with 8 epilogue warps) and the kernel / parity tests
cd $GRAFT_REPO_ROOT
run() {  # name tool tests...
  local name=$1 tool=$2; shift 2
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 20 python -m pytest "$@" -q -x -p no:cacheprovider > gpurun_out/san2_${name}_$tool.log 2>&1
  echo "$name $tool exit $?: $(grep -E 'ERROR SUMMARY' gpurun_out/san2_${name}_$tool.log | tail -1) $(grep -E ' passed| failed' gpurun_out/san2_${name}_$tool.log | tail -1)"
}
run fused memcheck tests/test_gpu_fused_epilogues.py
run kernels memcheck tests/test_gpu_kernels.py tests/test_gpu_parity.py -k "not tiny_config0"
run fused synccheck tests/test_gpu_fused_epilogues.py -k "stage and small64"
