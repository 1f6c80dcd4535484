"""One summary line of a bench.py JSON output (A/B sweeps): req/s, per-kernel ms / TFLOP/s, clock."""
import json
import sys

tag, path = sys.argv[1], sys.argv[2]
try:
    d = json.loads(open(path).read().strip().splitlines()[-1])
except Exception as e:  # noqa: BLE001 - a failed run prints its tag
    print(tag, "FAILED", e)
    sys.exit(0)
k = d["kernels"]
ms = lambda n: round(k.get(n, {}).get("ms_per_step", 0.0), 2)  # noqa: E731
tf = lambda n: round(k.get(n, {}).get("tflops") or 0.0, 1)  # noqa: E731
print(tag, "req/s", round(d["value"], 1), "step ms", round(d["ms_per_step"], 1),
      "| gate_up", ms("gemm_gate_up"), tf("gemm_gate_up"), "| down", ms("gemm_down"), tf("gemm_down"),
      "| o", ms("gemm_o"), "| qkv", ms("gemm_qkv"), "| norm", ms("rmsnorm"), "| stage", ms("stage"),
      "| embed", ms("embed"), "| attn", ms("attention"), tf("attention"), "| MHz", d["clocks"]["sm_mhz"], flush=True)
