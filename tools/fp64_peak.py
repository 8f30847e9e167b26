"""Measure B200 FP64 roofline denominators once: hand DMMA/DFMA issue peaks and cuBLAS ZGEMM/DGEMM.

SURVEY.md §0 item 6 / §8(d): MEASURED_PEAKS.json has HBM and BF16 only, so the FP64 peak is measured here.
Writes one JSON line per measurement to stdout.
"""
import json, subprocess, sys, time
import torch

def cublas(dtype, m, n, k, reps=10):
    a = torch.randn(m, k, dtype=dtype, device="cuda")
    b = torch.randn(k, n, dtype=dtype, device="cuda")
    for _ in range(3):
        torch.matmul(a, b)
    torch.cuda.synchronize()
    best = 1e30
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True); e1 = torch.cuda.Event(enable_timing=True)
        e0.record(); torch.matmul(a, b); e1.record(); torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    f = (8.0 if dtype.is_complex else 2.0) * m * n * k
    return f / best / 1e9

if __name__ == "__main__":
    for dt in (torch.float64, torch.complex128):
        for (m, n, k) in ((8192, 8192, 8192), (4096, 4096, 4096), (64, 64, 352800), (352800, 64, 64)):
            print(json.dumps({"kind": "cublas", "dtype": str(dt), "m": m, "n": n, "k": k, "tflops": round(cublas(dt, m, n, k), 3)}), flush=True)
