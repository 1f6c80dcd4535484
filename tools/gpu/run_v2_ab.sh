#!/bin/bash
# v2 attention kernel: microbench, layer-level parity, bench A/B against v1; fixed tests
cd $GRAFT_REPO_ROOT
timeout 120 ./tools/fa4_chain > gpurun_out/fa4_chain.txt 2>&1
timeout 900 python -m pytest -q -x -p no:cacheprovider -s tests/test_gpu_kernels.py -k attention > gpurun_out/v2_kernels.log 2>&1
echo "rc=$?" >> gpurun_out/v2_kernels.log
timeout 900 python -m pytest -q -p no:cacheprovider -s tests/test_gpu_attn_fullbatch.py tests/test_gpu_parity.py tests/test_gpu_dist.py tests/test_gpu_score.py > gpurun_out/v2_parity.log 2>&1
echo "rc=$?" >> gpurun_out/v2_parity.log
timeout 900 python bench.py --steps 5 --warmup 2 --no-cpu-baseline --no-extras --workload cfg1-ip --corpus 8192 > gpurun_out/v2_bench_cfg1.json 2> gpurun_out/v2_bench_cfg1.err
BAT_ATTN=v1 timeout 900 python bench.py --steps 5 --warmup 2 --no-cpu-baseline --no-extras --workload cfg1-ip --corpus 8192 > gpurun_out/v1_bench_cfg1.json 2> gpurun_out/v1_bench_cfg1.err
cat gpurun_out/fa4_chain.txt; tail -2 gpurun_out/v2_kernels.log gpurun_out/v2_parity.log
python - <<'PY'
import json
for f in ["gpurun_out/v2_bench_cfg1.json", "gpurun_out/v1_bench_cfg1.json"]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, round(d["value"], 1), "attn", round(d["attention"]["tflops"], 1), "clk", d["clocks"]["sm_mhz"])
    except Exception as e:
        print(f, "ERR", e)
PY
