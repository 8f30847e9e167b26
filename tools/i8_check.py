"""Quick A/B of the int8-digit tensor-core GEMM-2 (LFD_NL_I8=1) against the DMMA path (LFD_NL_I8=0):
the same steps on the same inputs in two contexts; prints the relative difference and per-call times.
  python tools/i8_check.py [workload ...]"""
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from lfd_workloads import make_inputs, workload  # noqa: E402
from lfd_workloads.generate import midpoint_A  # noqa: E402
from paper_conf_ipps_razakhllknvn24_b200 import Context  # noqa: E402


def run(w, x, i8, steps):
    os.environ["LFD_NL_I8"] = "1" if i8 else "0"
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    ctx = Context(psi, torch.from_numpy(x.proj).to(dev), x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc)
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    for n in range(steps):
        ctx.set_vector_potential(midpoint_A(w, n))
        ctx.step(1)
    ctx.sync()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for n in range(10):
        ctx.set_vector_potential(midpoint_A(w, n))
        ctx.step(1)
    ctx.sync()
    dt = (time.perf_counter() - t0) / 10
    out = psi.cpu().numpy()
    ctx.close()
    return out, dt


for name in sys.argv[1:] or ["P0", "C1", "C2"]:
    w = workload(name)
    x = make_inputs(w, seed=1)
    steps = 2 if name.startswith("C2") else 20
    a, ta = run(w, x, False, steps)
    b, tb = run(w, x, True, steps)
    print(f"{name}: rel diff {np.linalg.norm(a - b) / np.linalg.norm(a):.3e}  dmma {ta*1e3:.3f} ms/step  "
          f"i8 {tb*1e3:.3f} ms/step", flush=True)
