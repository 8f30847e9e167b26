"""GPU-vs-oracle parity of the NEXT-row functions: lfd_energy (calc_energy,
P:212 / Fig. 5) and lfd_remap_occ (remap_occ, P:58 / P:212), through the C ABI, on the same seeded
inputs after propagation. Tolerance: 1e-10 relative (FP64; differences are summation order only)."""
import numpy as np
import pytest

from lfd_workloads import make_inputs, workload
from lfd_workloads.generate import midpoint_A

pytestmark = pytest.mark.gpu


def _run(w, x, steps, nref_max=0):
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    proj = torch.from_numpy(x.proj).to(dev) if w.nproj else None
    ctx = Context(psi, proj, x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc, nref_max=nref_max)
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    A = np.zeros((w.ndom, 3))
    for n in range(steps):
        A = midpoint_A(w, n)
        ctx.set_vector_potential(A)
        ctx.step(1)
    return ctx, psi, A


def _ref_state(w, x, steps):
    from oracle import ref
    cfg = ref.RefConfig(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    p = x.psi0.copy()
    A = np.zeros((w.ndom, 3))
    for n in range(steps):
        A = midpoint_A(w, n)
        ref.step(cfg, p, x.proj if w.nproj else None, x.dnl if w.nproj else None, x.vloc, A, 1)
    return cfg, p, A


@pytest.mark.parametrize("name,steps", [("P0", 20), ("P2z", 10), ("P3", 3), ("C1", 10), ("P1", 5)])
def test_energy_parity(name, steps):
    from oracle import ref
    w = workload(name)
    x = make_inputs(w, seed=21)
    ctx, psi, A = _run(w, x, steps)
    E = ctx.energy()
    ctx.sync()
    E = E.cpu().numpy()
    ctx.close()
    cfg, p, Ar = _ref_state(w, x, steps)
    Er = np.concatenate([ref.energy(ref.RefConfig(1, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt),
                                    np.ascontiguousarray(p[d:d + 1]), x.occ[d:d + 1], np.ascontiguousarray(x.vloc[d:d + 1]),
                                    Ar[d], np.ascontiguousarray(x.proj[d:d + 1]) if w.nproj else None,
                                    x.dnl[d:d + 1] if w.nproj else None) for d in range(w.ndom)])
    scale = np.abs(Er[:, :3]).sum(axis=1).max()
    assert np.abs(E - Er).max() <= 1e-10 * scale, (E, Er)


@pytest.mark.parametrize("name,steps", [("P0", 20), ("P3", 3), ("C1", 10)])
def test_remap_occ_parity(name, steps):
    import torch
    from oracle import ref
    w = workload(name)
    x = make_inputs(w, seed=22)
    basis = np.ascontiguousarray(np.concatenate([x.psi0, x.proj], axis=-1))
    nref = basis.shape[-1]
    ctx, psi, A = _run(w, x, steps, nref_max=nref)
    occ = ctx.remap_occ(torch.from_numpy(basis).cuda())
    ctx.sync()
    occ = occ.cpu().numpy()
    ctx.close()
    cfg, p, _ = _ref_state(w, x, steps)
    occ_r = ref.remap_occ(cfg, p, x.occ, basis)
    assert np.abs(occ - occ_r).max() <= 1e-10 * np.abs(occ_r).max()
    # occupations move from the occupied block into the unoccupied one under light + scissor
    assert occ[:, w.norb:].sum() > 0
