#!/bin/bash
# SwiGLU GEMM rasterisation group sweep on the configs[2] bench (M ~ 104K rows per step)
cd $GRAFT_REPO_ROOT
for g in 32 64 128 16; do
  BAT_GEMM_GROUP_SWIGLU=$g timeout 900 python bench.py --steps 5 --warmup 2 --no-cpu-baseline --no-extras > gpurun_out/gs_$g.json 2> gpurun_out/gs_$g.err
done
python - <<'PY'
import json
for g in [32, 64, 128, 16]:
    try:
        d = json.loads(open(f"gpurun_out/gs_{g}.json").read().strip().splitlines()[-1])
        k = d["kernels"]["gemm_gate_up"]
        print(g, round(d["value"], 2), "gu ms", round(k["ms_per_step"], 2), "tf", round(k["tflops"], 1), "clk", d["clocks"]["sm_mhz"], "W", d["clocks"].get("power_w_median"))
    except Exception as e:
        print(g, "ERR", e)
PY
