"""cuBLAS (torch.mm) throughput on the bench's GEMM shapes, for comparison with gemm_tc_kernel
(reference numbers only; nothing on the product path calls cuBLAS)."""
import torch
M = 64 * 520
shapes = {"qkv": (M, 2048, 1536), "o": (M, 1536, 1536), "gate_up": (M, 17920, 1536), "down": (M, 1536, 8960)}
for name, (m, n, k) in shapes.items():
    a = torch.randn(m, k, device="cuda", dtype=torch.bfloat16)
    b = torch.randn(n, k, device="cuda", dtype=torch.bfloat16)
    for _ in range(3):
        c = a @ b.t()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    it = 20
    e0.record()
    for _ in range(it):
        c = a @ b.t()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / it
    print(f"cuBLAS {name:8s} M={m} N={n} K={k}: {ms:.3f} ms  {2 * m * n * k / ms / 1e9:.0f} TFLOP/s")

# the same shapes through libbat's tcgen05 GEMM (bat_debug_gemm: tensor maps built per call)
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_0017wzlxszh0w26_b200 import bat
for name, (m, n, k), epi in (("qkv", shapes["qkv"], 1), ("o", shapes["o"], 2), ("gate_up", (M, 8960, 1536), 3),
                             ("down", shapes["down"], 2)):
    a = torch.randn(m, k, device="cuda", dtype=torch.bfloat16)
    rows = 2 * n if epi == 3 else n
    b = (torch.randn(rows, k, device="cuda") * 0.02).to(torch.bfloat16)
    out = torch.zeros(m, n, device="cuda", dtype=torch.float32 if epi == 2 else torch.bfloat16)
    bias = torch.zeros(n, device="cuda", dtype=torch.bfloat16)
    call = lambda: bat.bat_debug_gemm(epi, m, n, k, a, b, rows, out, n, bias if epi == 1 else None, n if epi == 3 else 0)
    for _ in range(3):
        call()
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    it = 20
    e0.record()
    for _ in range(it):
        call()
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / it
    fl = 2 * m * rows * k
    print(f"libbat {name:8s} M={m} N={rows} K={k} epi={epi}: {ms:.3f} ms  {fl / ms / 1e9:.0f} TFLOP/s")
