#!/bin/bash
# compute-sanitizer memcheck / synccheck over the parity cases (every kernel of the path, the
# three attention kernels, the fp32 mode); results summarised into gpurun_out/san_*.log
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
run() {  # name env tool tests...
  local name=$1 envs=$2 tool=$3; shift 3
  env $envs timeout 1500 compute-sanitizer --tool $tool --error-exitcode 99 --print-limit 20 python -m pytest "$@" -q -x -p no:cacheprovider > gpurun_out/san_${name}_$tool.log 2>&1
  echo "$name $tool exit $?: $(grep -E 'ERROR SUMMARY' gpurun_out/san_${name}_$tool.log | tail -1) $(grep -E ' passed| failed' gpurun_out/san_${name}_$tool.log | tail -1)"
}
run tc "BAT_ATTN=tc" memcheck tests/test_gpu_parity.py tests/test_gpu_kernels.py tests/test_gpu_multidisc.py tests/test_gpu_edge.py
run pair "BAT_ATTN=pair" memcheck tests/test_gpu_parity.py -k "small"
run db "BAT_ATTN=db" memcheck tests/test_gpu_parity.py -k "small"
run fp32 "X=1" memcheck tests/test_gpu_fp32.py -k "tiny or small64"
run tc "BAT_ATTN=tc" synccheck tests/test_gpu_parity.py -k "small"
run tc "BAT_ATTN=tc" racecheck tests/test_gpu_parity.py -k "tiny_config0"
