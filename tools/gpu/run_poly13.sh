#!/bin/bash
# exp2 FMA-pipe share around the default (2 of 16 column pairs): 1 and 3, configs[2], same box
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
P=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200
for v in p1 p3; do BAT_LIB=$P/libbat_$v.so timeout 300 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_attn_rescale.py -q -x -p no:cacheprovider -k attention 2>&1 | tail -1; done
run() {  # tag env...
  local tag=$1; shift
  env "$@" timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-extras --corpus 16384 > gpurun_out/pq_$tag.json 2>gpurun_out/pq_$tag.err
  python tools/bench_line.py "$tag" gpurun_out/pq_$tag.json
}
for rep in 1 2 3; do
  run base_$rep X=1
  run p1_$rep BAT_LIB=$P/libbat_p1.so
  run p3_$rep BAT_LIB=$P/libbat_p3.so
done
