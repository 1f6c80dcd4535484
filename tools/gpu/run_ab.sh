#!/bin/bash
# attention A/B: debug-build kernel tests (mbarrier timeouts trap instead of hanging), then the
# bench with the double-buffered kernel (default) and the single-buffered one (BAT_ATTN=tc)
TAG=${1:-ab}
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_dbg.so timeout 400 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/dbg_$TAG.log 2>&1
echo "dbg tests exit $?"; grep -E "mbar|passed|failed|Error|assert" gpurun_out/dbg_$TAG.log | head -20
timeout 600 python -m pytest tests/test_gpu_fp32.py -q -x -s -p no:cacheprovider > gpurun_out/fp32_$TAG.log 2>&1
echo "fp32 tests exit $?"; grep -E "worst|passed|failed|Error|assert" gpurun_out/fp32_$TAG.log | head -30
if grep -q "passed" gpurun_out/dbg_$TAG.log && ! grep -q "failed" gpurun_out/dbg_$TAG.log; then
  timeout 600 python bench.py --steps 6 --warmup 3 --no-cpu-baseline > gpurun_out/bench_db_$TAG.json 2> gpurun_out/bench_db_$TAG.err
  echo "bench db exit $?"
  BAT_ATTN=tc timeout 600 python bench.py --steps 6 --warmup 3 --no-cpu-baseline > gpurun_out/bench_tc_$TAG.json 2> gpurun_out/bench_tc_$TAG.err
  echo "bench tc exit $?"
  python - $TAG <<'PY'
import json,sys
for k in ("db","tc"):
    try:
        d=json.loads(open(f"gpurun_out/bench_{k}_{sys.argv[1]}.json").read().strip().splitlines()[-1])
    except Exception as e:
        print(k,"no json",e); continue
    print(k, "req/s %.1f"%d["value"], "attn", json.dumps(d.get("attention")), "ms/step %.2f"%d["ms_per_step"])
PY
fi
