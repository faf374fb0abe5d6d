"""B2B GEMM timing vs two cuBLAS matmuls (development aid)."""
import sys, json
import numpy as np, torch
sys.path.insert(0, ".")
import ftgen
from paper_conf_sosp_liuqc0hs0y24_b200 import ft
def t(fn, reps=50):
    for _ in range(5): fn()
    torch.cuda.synchronize()
    s, e = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    s.record()
    for _ in range(reps): fn()
    e.record(); torch.cuda.synchronize()
    return s.elapsed_time(e) / reps
for M, N in [(16384, 4096), (65536, 4096), (16384, 16384), (131072, 2048)]:
    g = ftgen.b2b_inputs(M, N, 64, 64, 1, "bf16")
    A, B, C = (torch.from_numpy(g[k]).cuda().to(torch.bfloat16) for k in ("A", "B", "C"))
    ours = t(lambda: ft.b2b_gemm(A, B, C))
    cub = t(lambda: (A @ B) @ C)
    fl = 2.0 * M * N * 64 * 2
    print(json.dumps(dict(M=M, N=N, ours_ms=ours, cublas_ms=cub, ours_tflops=fl / ours / 1e9, speedup=cub / ours)))
