"""Small driver for compute-sanitizer runs (tests/test_gpu_sanitizer.py): a few LFD steps, the merged-factor
sequence, density, energy and remap_occ on tiny shapes covering every kernel variant (periodic / zero BC,
nproj 0 / < 64 / not a multiple of 4 / > 64, fused and unfused stencil paths).

  python tools/sanitize_drive.py [dmma | i8 | sp]
i8: the int8-digit tcgen05 GEMMs forced (LFD_FLAG_NL_I8: TMEM, mbarrier rings, bulk copies, the exponent
handshake with the K_y K_z pass); sp: the complex64 variant."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

from lfd_workloads import make_inputs, workload  # noqa: E402
from lfd_workloads.generate import midpoint_A  # noqa: E402
from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd  # noqa: E402

mode = sys.argv[1] if len(sys.argv) > 1 else "dmma"
dev = torch.device("cuda:0")
if mode == "i8":
    shapes = [workload("P0"), workload("P1"), workload("P0").with_(nx=8, ny=8, nz=70, norb=64, nocc=32, nproj=64)]
    flags = lfd.LFD_FLAG_NL_I8
else:
    shapes = [workload("P0"), workload("P2z"), workload("P3").with_(nx=6, ny=6, nz=8), workload("P1"),
              workload("P0").with_(nproj=0), workload("P0").with_(nz=90, nproj=7)]
    flags = 0
cdt = np.complex64 if mode == "sp" else np.complex128
for w in shapes:
    x = make_inputs(w, seed=5)
    psi = torch.from_numpy(x.psi0.astype(cdt)).to(dev)
    proj = torch.from_numpy(x.proj.astype(cdt)).to(dev) if w.nproj else None
    nref = w.norb + w.nproj
    ctx = Context(psi, proj, x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc, nref_max=nref, flags=flags)
    if mode == "i8":
        assert lfd.lfd_nl_path(ctx.ctx) == 1, w
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    for n in range(3):
        ctx.set_vector_potential(midpoint_A(w, n))
        ctx.step(1)
    if w.nproj:
        ctx.step_sequence(np.stack([midpoint_A(w, n) for n in range(3)]))
    ctx.density_current()
    ctx.energy()
    basis = np.concatenate([x.psi0, x.proj], axis=-1) if w.nproj else x.psi0
    ctx.remap_occ(torch.from_numpy(np.ascontiguousarray(basis.astype(cdt))).to(dev))
    ctx.sync()
    assert not torch.isnan(psi).any(), w.name
    ctx.close()
if mode == "dmma":  # dense Hermitian D (LFD_FLAG_DENSE_D): the B Q rotation at init, then the diagonal path
    w = workload("P0")
    x = make_inputs(w, seed=6)
    rng = np.random.default_rng(0)
    M = rng.standard_normal((1, w.nproj, w.nproj)) + 1j * rng.standard_normal((1, w.nproj, w.nproj))
    Dm = np.ascontiguousarray(0.05 * (M + np.conj(np.swapaxes(M, 1, 2))))
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    ctx = Context(psi, torch.from_numpy(x.proj).to(dev), Dm, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc,
                  flags=lfd.LFD_FLAG_DENSE_D)
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    ctx.step(2)
    ctx.energy()
    ctx.sync()
    assert not torch.isnan(psi).any()
    ctx.close()
print("sanitize drive ok")
