#!/bin/bash
# fused a4: parity (default 4-warp QKV epilogue and the 8-warp variant) + configs[2] A/B
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
P=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200
timeout 900 python -m pytest tests/test_gpu_fused_epilogues.py tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_multidisc.py tests/test_gpu_pic.py -q -x -p no:cacheprovider 2>&1 | tail -3
BAT_LIB=$P/libbat_q8.so timeout 300 python -m pytest tests/test_gpu_fused_epilogues.py -q -x -p no:cacheprovider -k stage 2>&1 | tail -2
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/st_$tag.json 2>gpurun_out/st_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/st_$tag.json
}
for rep in 1 2; do
  run fused_$rep X=1
  run fusedq8_$rep BAT_LIB=$P/libbat_q8.so
  run unfused_$rep BAT_FUSED_STAGE=0
done
