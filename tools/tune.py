"""A/B timing of internal kernel variants (env knobs read at lfd_init) on the C2 workload.

  python tools/tune.py --knob LFD_GEMM2_VARIANT --values 0 1 [--steps 20]
Prints one JSON line per value with the per-kernel-class device time per launch (ms).
"""
import argparse

import numpy as np
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--knob", required=True)
    ap.add_argument("--values", nargs="+", required=True)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--config", default="C2")
    ap.add_argument("--sp", action="store_true", help="the SP variant (complex64 Psi / B)")
    args = ap.parse_args()
    import torch
    from lfd_workloads import make_inputs, workload
    from lfd_workloads.generate import midpoint_A
    from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
    w = workload(args.config)
    x = make_inputs(w, seed=1)
    dev = torch.device("cuda:0")
    if args.sp:
        x.psi0 = x.psi0.astype(np.complex64)
        x.proj = x.proj.astype(np.complex64) if w.nproj else None
    proj = torch.from_numpy(x.proj).to(dev) if w.nproj else None
    v = torch.from_numpy(x.vloc).to(dev)
    for val in args.values:
        os.environ[args.knob] = str(val)
        psi = torch.from_numpy(x.psi0.copy()).to(dev)
        ctx = Context(psi, proj, x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc)
        ctx.set_potential(v)
        for n in range(3):
            ctx.set_vector_potential(midpoint_A(w, n))
            ctx.step(1)
        lfd.lfd_profile_enable(ctx.ctx, True)
        rho = torch.empty((w.ndom, w.ngrid), dtype=torch.float64, device=dev)
        J = torch.empty((w.ndom, 3), dtype=torch.float64, device=dev)
        for n in range(args.steps):
            ctx.set_vector_potential(midpoint_A(w, n))
            ctx.step(1)
            lfd.lfd_density_current(ctx.ctx, rho, None, J)
        prof = lfd.lfd_profile_read(ctx.ctx)
        ctx.close()
        out = {"knob": args.knob, "value": val,
               "ms_per_launch": {k: round(t / n, 5) for k, (t, n) in prof.items() if n}}
        print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
