"""(norb, nproj) = (512, 64) at the C2 grid: is one nonlocal factor deterministic, and where does it differ
from the torch complex128 reference (with a full device sync between the snapshot and the factor)?"""
import sys
import numpy as np
import torch
sys.path.insert(0, ".")
from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
from lfd_workloads.configs import workload

w = workload("C2")
nx, ny, nz, no, npj = 70, 70, 72, 512, 64
ng = nx * ny * nz
g = torch.Generator(device="cuda").manual_seed(no * 7919 + npj)
shape = (1, nx, ny, nz)
psi = torch.randn(shape + (no,), dtype=torch.complex128, device="cuda", generator=g) * (1.0 / (w.dV * ng)) ** 0.5
proj = torch.randn(shape + (npj,), dtype=torch.complex128, device="cuda", generator=g) * (1.0 / (w.dV * ng)) ** 0.5
torch.cuda.synchronize()
before = psi.clone()
torch.cuda.synchronize()
P = before.reshape(ng, no)
B = proj.reshape(ng, npj)
C = w.dV * (B.mH @ P)
R = P + B @ ((-0.5j * w.dt * 0.07) * C)
R = R * (torch.linalg.vector_norm(P, dim=0) / torch.linalg.vector_norm(R, dim=0))
outs = []
for rep in range(12):
    fl = lfd.LFD_FLAG_NO_PDL if rep >= 8 else 0
    psi.copy_(before)
    torch.cuda.synchronize()
    ctx = Context(psi, proj, np.full((1, npj), 0.07), np.full((1, no), 2.0), (w.hx, w.hy, w.hz), w.dt, flags=fl)
    torch.cuda.synchronize()
    lfd.lfd_step_prologue(ctx.ctx)
    ctx.sync()
    torch.cuda.synchronize()
    got = psi.reshape(ng, no).clone()
    ctx.close()
    E = (got - R).abs() / (R - P).abs().clamp_min(1e-300)
    bad = torch.nonzero(E > 1e-6)
    acc = float(torch.linalg.vector_norm(got - R) / torch.linalg.vector_norm(R - P))
    print(f"rep {rep} acc {acc:.2e} bad {bad.shape[0]}", bad[:6].tolist(), flush=True)
    outs.append(got)
for i in range(1, len(outs)):
    d = (outs[i] != outs[0]).any(dim=1)
    print("rep", i, "vs rep 0: rows differing", int(d.sum()), torch.nonzero(d)[:6].flatten().tolist(), flush=True)
