import sys, os; sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from lfd_workloads import make_inputs, workload
from lfd_workloads.generate import midpoint_A
from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
dev = torch.device("cuda:0")
for name, steps in [("P0", 20), ("P3", 3), ("C1", 10), ("C1", 10)]:
    w = workload(name)
    x = make_inputs(w, seed=22)
    basis = np.ascontiguousarray(np.concatenate([x.psi0, x.proj], axis=-1))
    nref = basis.shape[-1]
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    proj = torch.from_numpy(x.proj).to(dev)
    ctx = Context(psi, proj, x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc, nref_max=nref)
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    for n in range(steps):
        ctx.set_vector_potential(midpoint_A(w, n)); ctx.step(1)
    b = torch.from_numpy(basis).cuda()
    occ = ctx.remap_occ(b); ctx.sync()
    C = w.dV * torch.einsum("drk,drs->dks", b.reshape(w.ndom, -1, nref).conj(), psi.reshape(w.ndom, -1, w.norb))
    want = (torch.from_numpy(x.occ).to(dev)[:, None, :] * C.abs() ** 2).sum(-1)
    print(name, nref, float((occ - want).abs().max() / want.abs().max()), bool(torch.isnan(occ).any()), bool(torch.isnan(psi).any()))
    ctx.close()
