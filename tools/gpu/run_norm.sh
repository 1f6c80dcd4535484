#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edge.py tests/test_gpu_kernels.py tests/test_gpu_multidisc.py -q -x -p no:cacheprovider 2>&1 | tail -1
for v in new old; do
  if [ $v = new ]; then L=libbat.so; else L=libbat_oldnorm.so; fi
  BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/$L timeout 300 python bench.py --steps 6 --warmup 3 --no-cpu-baseline > gpurun_out/norm_$v.json 2>/dev/null
  python -c "import json;d=json.loads(open('gpurun_out/norm_$v.json').read().strip().splitlines()[-1]);k=d['kernels'];print('$v stage ms', round(k['stage']['ms_per_step'],3), 'GB/s', round(k['stage']['gbs']), 'req/s', round(d['value'],1), 'clk', d['clocks']['sm_mhz'])"
done
