"""Summarise ncu outputs into profiles/: the launch list (per-kernel totals and shares) and the
key metrics of a --set full capture, plus the per-launch DRAM traffic bench.py reports.

usage: python tools/ncu_summary.py TAG   (reads gpurun_out/launches_TAG.csv, gpurun_out/full_TAG.ncu-rep)
"""
import collections
import csv
import io
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = ["dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum", "launch__registers_per_thread",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "sm__cycles_elapsed.avg.per_second",
        "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "smsp__issue_active.avg.pct_of_peak_sustained_active"]
NAMES = {"gemm_tc_kernel<1>": "gemm_qkv", "gemm_tc_kernel<3>": "gemm_gate_up", "gemm2_tc_kernel<3>": "gemm_gate_up"}


def short(name):
    name = re.sub(r"^void\s+", "", name)
    name = re.sub(r"\(.*$", "", name)
    name = re.sub(r"^.*::", "", name)
    return name


def launches(tag):
    path = os.path.join(ROOT, "gpurun_out", f"launches_{tag}.csv")
    txt = open(path).read()
    start = txt.find('"ID"')
    rows = list(csv.DictReader(io.StringIO(txt[start:])))
    tot = collections.OrderedDict()
    unit = set()
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        k = short(r["Kernel Name"])
        v = float(r["Metric Value"].replace(",", ""))
        unit.add(r["Metric Unit"])
        scale = {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "nsecond": 1e-6, "ms": 1.0, "msecond": 1.0}.get(r["Metric Unit"], 1e-6)
        n, t = tot.get(k, (0, 0.0))
        tot[k] = (n + 1, t + v * scale)
    total = sum(t for _, t in tot.values())
    out = [f"# ncu launch list ({tag}): {os.environ.get('NCU_CMD', 'bench.py --steps 2 --warmup 1')}, timed region only",
           "# (--profile-from-start off; --metrics gpu__time_duration.sum --clock-control none).  Per-launch times",
           "# are cold-cache and serialised: compare SHARES with bench.py's live CUDA-event kernel table.",
           f"# raw unit {sorted(unit)}; workload: {os.environ.get('NCU_WORKLOAD', 'configs[2] batch 64 (bench.py default)')}",
           f"{'kernel':40s} {'launches':>9s} {'total_ms':>10s} {'share':>7s}"]
    for k, (n, t) in sorted(tot.items(), key=lambda kv: -kv[1][1]):
        out.append(f"{k:40s} {n:9d} {t:10.3f} {100 * t / total:6.1f}%")
    out.append(f"{'TOTAL':40s} {sum(n for n, _ in tot.values()):9d} {total:10.3f}")
    return "\n".join(out) + "\n"


def full(tag):
    rep = os.path.join(ROOT, "gpurun_out", f"full_{tag}.ncu-rep")
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    col = {h: i for i, h in enumerate(hdr)}
    out = [f"# ncu --set full --clock-control none ({tag}): first launches of bench.py's timed region",
           f"# ({os.environ.get('NCU_WORKLOAD', 'configs[1] IP, batch 64')}); kernels {os.environ.get('NCU_KERNELS', 'attn|gemm')}."]
    traffic = collections.OrderedDict()
    for r in data:
        name = r[col["Kernel Name"]]
        out.append(f"== {name}")
        for k in KEYS:
            if k in col:
                out.append(f"   {k:75s} {r[col[k]]:>16s} {units[col[k]]}")
        try:
            rd = float(r[col["dram__bytes_read.sum"]].replace(",", ""))
            wr = float(r[col["dram__bytes_write.sum"]].replace(",", ""))
            mul = lambda u: {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
            traffic.setdefault(short(name), rd * mul(units[col["dram__bytes_read.sum"]]) +
                               wr * mul(units[col["dram__bytes_write.sum"]]))
        except (KeyError, ValueError):
            pass
    return "\n".join(out) + "\n", traffic


if __name__ == "__main__":
    tag = sys.argv[1]
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    if os.path.exists(os.path.join(ROOT, "gpurun_out", f"launches_{tag}.csv")):
        s = launches(tag)
        open(os.path.join(ROOT, "profiles", f"{tag}_launches_summary.txt"), "w").write(s)
        print(s)
    if os.path.exists(os.path.join(ROOT, "gpurun_out", f"full_{tag}.ncu-rep")):
        s, tr = full(tag)
        open(os.path.join(ROOT, "profiles", f"{tag}_ncu_full_summary.txt"), "w").write(s)
        print(s)
        print(json.dumps(tr, indent=1))
