#!/bin/bash
cd $GRAFT_REPO_ROOT
for v in v5 v1; do
  BAT_ATTN=$v timeout 900 python bench.py --steps 5 --warmup 2 --no-cpu-baseline --no-extras --workload cfg1-ip --corpus 8192 > gpurun_out/ab2_$v.json 2> gpurun_out/ab2_$v.err
done
python - <<'PY'
import json
for v in ["v5", "v1"]:
    try:
        d = json.loads(open(f"gpurun_out/ab2_{v}.json").read().strip().splitlines()[-1])
        print(v, round(d["value"], 1), "attn", round(d["attention"]["tflops"], 1), "attn ms", round(d["attention"]["ms_per_step"],2), "clk", d["clocks"]["sm_mhz"])
    except Exception as e:
        print(v, "ERR", e, open(f"gpurun_out/ab2_{v}.err").read()[-500:])
PY
