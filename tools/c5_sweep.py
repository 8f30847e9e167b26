"""C5 (BASELINE.json configs[4]): the nonlocal-projector sweep.

Ngrid = 352,800 (the paper's 70x70x72 mesh); norb in {32..512} x nproj in {64..1024}.
For each shape one context runs `steps` LFD steps (NL half, local, NL half) and the per-launch device
time of GEMM-1 (k_gemm1: C = dV B^H Psi) and GEMM-2 (k_gemm2*: Psi <- (Psi + B C') n) is read from the
library's CUDA-event profiler. Flops are counted as 8 per complex multiply-add (the 3M kernels do 6
real flops per complex MAC on the tensor pipe; the rate reported is the effective one). cuBLAS ZGEMM
(torch.matmul on complex128) on the same two shapes is timed alongside as the library baseline.

  python tools/c5_sweep.py [--steps 3] [--quick] > profiles/rNN_c5_sweep.jsonl
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def cublas_ms(m, n, k, conj_a, reps=5):
    import torch
    if conj_a:  # C (m x n) = A^H (k x m)^H X (k x n)
        a = torch.randn(k, m, dtype=torch.complex128, device="cuda")
        x = torch.randn(k, n, dtype=torch.complex128, device="cuda")
        f = lambda: torch.matmul(a.mH, x)
    else:
        a = torch.randn(m, k, dtype=torch.complex128, device="cuda")
        x = torch.randn(k, n, dtype=torch.complex128, device="cuda")
        f = lambda: torch.matmul(a, x)
    for _ in range(2):
        f()
    torch.cuda.synchronize()
    best = 1e30
    for _ in range(reps):
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record()
        f()
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1))
    return best


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=3)
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--no-cublas", action="store_true")
    args = ap.parse_args()
    import torch
    from lfd_workloads.configs import C5_NORB, C5_NPROJ, workload
    from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd

    w = workload("C2")
    ng = w.ngrid
    norbs = (32, 128, 512) if args.quick else C5_NORB
    nprojs = (64, 256, 1024) if args.quick else C5_NPROJ
    peak = 37.167              # measured DMMA.8x8x4 issue peak (profiles/r01_fp64_peaks.jsonl)
    peak3m = peak * 4.0 / 3.0  # the 3M kernels issue 3 real DMMA per complex MAC (8 flops counted)
    for no in norbs:
        for npj in nprojs:
            g = torch.Generator(device="cuda").manual_seed(no * 7919 + npj)
            shape = (1, w.nx, w.ny, w.nz)
            psi = torch.randn(shape + (no,), dtype=torch.complex128, device="cuda", generator=g)
            psi *= (1.0 / (w.dV * ng)) ** 0.5
            proj = torch.randn(shape + (npj,), dtype=torch.complex128, device="cuda", generator=g)
            proj *= (1.0 / (w.dV * ng)) ** 0.5
            occ = [[2.0] * no]
            dnl = [[0.07] * npj]
            ctx = Context(psi, proj, dnl, occ, (w.hx, w.hy, w.hz), w.dt)
            ctx.step(1)
            lfd.lfd_profile_enable(ctx.ctx, True)
            ctx.step(args.steps)
            prof = lfd.lfd_profile_read(ctx.ctx)
            ctx.close()
            flops = 8.0 * ng * no * npj
            rec = {"config": "C5", "ngrid": ng, "norb": no, "nproj": npj, "gflop_per_gemm": flops / 1e9}
            for k, name in (("nl_proj", "gemm1"), ("nl_back", "gemm2")):
                ms = prof[k][0] / max(prof[k][1], 1)
                tf = flops / (ms * 1e-3) / 1e12
                rec[name] = {"ms": ms, "tflops_effective": tf, "frac_of_fp64_peak": tf / peak,
                             "frac_of_dmma_pipe": tf / peak3m}
            if not args.no_cublas:
                c1 = cublas_ms(npj, no, ng, True)
                c2 = cublas_ms(ng, no, npj, False)
                rec["cublas_zgemm"] = {"gemm1_ms": c1, "gemm1_tflops": flops / (c1 * 1e-3) / 1e12,
                                       "gemm2_ms": c2, "gemm2_tflops": flops / (c2 * 1e-3) / 1e12}
            rec["peak_tflops"] = peak
            print(json.dumps(rec), flush=True)
            del psi, proj
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
