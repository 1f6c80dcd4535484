#!/bin/bash
# CTA-pair attention: debug-build kernel/parity tests (mbarrier timeouts trap), then bench pair vs tc
TAG=${1:-pair}
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
BAT_ATTN=pair BAT_LIB=$PWD/paper_conf_asplos_0017wzlxszh0w26_b200/libbat_dbg.so timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -p no:cacheprovider -k attention > gpurun_out/dbg_$TAG.log 2>&1
echo "dbg kernel tests exit $?"; grep -E "mbar|passed|failed|Error|assert|excess" gpurun_out/dbg_$TAG.log | head -20
if grep -q " passed" gpurun_out/dbg_$TAG.log && ! grep -q "failed" gpurun_out/dbg_$TAG.log; then
  BAT_ATTN=pair timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -p no:cacheprovider > gpurun_out/par_$TAG.log 2>&1
  echo "parity exit $?"; tail -3 gpurun_out/par_$TAG.log
  BAT_ATTN=pair timeout 600 python bench.py --steps 6 --warmup 3 --no-cpu-baseline > gpurun_out/bench_pair_$TAG.json 2> gpurun_out/bench_pair_$TAG.err
  echo "bench pair exit $?"; tail -2 gpurun_out/bench_pair_$TAG.err
  BAT_ATTN=tc timeout 600 python bench.py --steps 6 --warmup 3 --no-cpu-baseline > gpurun_out/bench_tc_$TAG.json 2> gpurun_out/bench_tc_$TAG.err
  python - $TAG <<'PY'
import json,sys
for k in ("pair","tc"):
    try:
        d=json.loads(open(f"gpurun_out/bench_{k}_{sys.argv[1]}.json").read().strip().splitlines()[-1])
    except Exception as e:
        print(k,"no json",e); continue
    print(k, "req/s %.1f"%d["value"], "attn", json.dumps(d.get("attention")), "ms/step %.2f"%d["ms_per_step"])
PY
fi
