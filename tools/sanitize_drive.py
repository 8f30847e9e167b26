"""Small driver for compute-sanitizer runs (tests/test_gpu_sanitizer.py): a few LFD steps, density,
energy and remap_occ on tiny shapes covering every kernel variant (periodic / zero BC, nproj 0 / < 64 /
not a multiple of 4 / > 64, fused and unfused stencil paths)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

from lfd_workloads import make_inputs, workload  # noqa: E402
from lfd_workloads.generate import midpoint_A  # noqa: E402
from paper_conf_ipps_razakhllknvn24_b200 import Context  # noqa: E402

dev = torch.device("cuda:0")
shapes = [workload("P0"), workload("P2z"), workload("P3").with_(nx=6, ny=6, nz=8), workload("P1"),
          workload("P0").with_(nproj=0), workload("P0").with_(nz=90, nproj=7)]
for w in shapes:
    x = make_inputs(w, seed=5)
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    proj = torch.from_numpy(x.proj).to(dev) if w.nproj else None
    nref = w.norb + w.nproj
    ctx = Context(psi, proj, x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc, nref_max=nref)
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    for n in range(3):
        ctx.set_vector_potential(midpoint_A(w, n))
        ctx.step(1)
    if w.nproj:
        ctx.step_sequence(np.stack([midpoint_A(w, n) for n in range(3)]))
    ctx.density_current()
    ctx.energy()
    basis = np.concatenate([x.psi0, x.proj], axis=-1) if w.nproj else x.psi0
    ctx.remap_occ(torch.from_numpy(np.ascontiguousarray(basis)).to(dev))
    ctx.sync()
    assert not torch.isnan(psi).any(), w.name
    ctx.close()
print("sanitize drive ok")
