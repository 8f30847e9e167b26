"""Dense Hermitian nonlocal coupling D (LFD_FLAG_DENSE_D, Eq. 5 v_nl = sum_uv
|b_u> D_uv <b_v|) against the oracle's dense-D factor (oracle/lfd_ref.c, pinned in
tests/test_oracle_pins_dense.py) on identical seeded inputs, at the FP64 bound of the parity contract: the
first-order and exactly unitary factors, the DMMA and int8-digit GEMM paths, the merged sequence, the nonlocal
energy, the SP variant (its derived bound), and the argument checks."""
from __future__ import annotations

import numpy as np
import pytest

from lfd_workloads import make_inputs, workload
from lfd_workloads.generate import midpoint_A

from .test_gpu_parity import TOL, assert_parity, laser, rel

pytestmark = pytest.mark.gpu

DENSE, EXACT, I8, DMMA, SP = 32, 2, 16, 8, 4


def dense_D(w, seed=0, scale=0.07):
    """Hermitian couplings per domain: the scissor Delta_sci I plus a random Hermitian part of the same size."""
    rng = np.random.default_rng(seed)
    M = rng.standard_normal((w.ndom, w.nproj, w.nproj)) + 1j * rng.standard_normal((w.ndom, w.nproj, w.nproj))
    H = 0.5 * (M + np.conj(np.swapaxes(M, 1, 2)))
    return np.ascontiguousarray(scale * (np.eye(w.nproj)[None] + 0.5 * H / np.sqrt(w.nproj)))


def run_gpu(w, x, steps, Dm, flags, seq=False, sp=False):
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    dev = torch.device("cuda:0")
    dt = np.complex64 if sp else np.complex128
    psi = torch.from_numpy(x.psi0.astype(dt)).to(dev)
    proj = torch.from_numpy(x.proj.astype(dt)).to(dev)
    ctx = Context(psi, proj, Dm, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc, flags=flags | DENSE)
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    if seq:
        ctx.step_sequence(np.stack([midpoint_A(w, n) for n in range(steps)]))
    else:
        for n in range(steps):
            ctx.set_vector_potential(midpoint_A(w, n))
            ctx.step(1)
    ctx.set_vector_potential(midpoint_A(w, steps - 1))
    rho, j, J = ctx.density_current()
    E = ctx.energy()
    ctx.sync()
    out = (psi.cpu().numpy().astype(np.complex128), rho.cpu().numpy().reshape(w.ndom, -1),
           j.cpu().numpy().reshape(w.ndom, 3, -1), J.cpu().numpy())
    E = E.cpu().numpy()
    ctx.close()
    return out, E


def run_ref(w, x, steps, Dm, exact=False, psi0=None, proj=None):
    from oracle import ref
    cfg = ref.RefConfig(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    p = (x.psi0 if psi0 is None else psi0).copy()
    B = x.proj if proj is None else proj
    A = np.zeros((w.ndom, 3))
    for n in range(steps):
        A = midpoint_A(w, n)
        ref.step_dense(cfg, p, B, Dm, x.vloc, A, 1, exact=exact)
    rho, j, J = ref.density_current(cfg, p, x.occ, A)
    Enl = ref.energy_nl_dense(cfg, p, x.occ, B, Dm)
    return (p, rho, j, J), Enl


@pytest.mark.parametrize("name,steps,flags", [("P0", 60, 0), ("P0", 60, I8), ("P1", 15, 0), ("P2z", 20, 0),
                                              ("P3", 4, 0), ("C1", 10, I8)])
def test_dense_first_order_parity(name, steps, flags):
    w = workload(name)
    x = make_inputs(w, seed=21)
    Dm = dense_D(w)
    got, E = run_gpu(w, x, steps, Dm, flags)
    want, Enl = run_ref(w, x, steps, Dm)
    assert_parity(w, got, want)
    assert np.abs(E[:, 2] - Enl).max() <= TOL * max(np.abs(Enl).max(), 1e-300)


@pytest.mark.parametrize("name,flags", [("P0", 0), ("P0", I8), ("C1", 0)])
def test_dense_exact_factor_parity(name, flags):
    """orthonormal projector columns (the workloads' B): exp(-i eps B D B^H dV) via D's eigenbasis"""
    w = workload(name)
    x = make_inputs(w, seed=22)
    Dm = dense_D(w, seed=1, scale=0.3)
    got, _ = run_gpu(w, x, 20, Dm, flags | EXACT)
    want, _ = run_ref(w, x, 20, Dm, exact=True)
    assert_parity(w, got, want)


@pytest.mark.parametrize("name", ["P0", "P3"])
def test_dense_sequence_parity(name):
    """lfd_step_sequence (merged adjacent factors) with dense D equals the oracle stepping one step at a time"""
    w = workload(name)
    x = make_inputs(w, seed=23)
    Dm = dense_D(w, seed=2)
    got, _ = run_gpu(w, x, 6, Dm, 0, seq=True)
    want, _ = run_ref(w, x, 6, Dm)
    assert_parity(w, got, want)


def test_dense_nonorthonormal_projectors():
    """B rescaled per column (G != I) and mixed into Psi: the rotated Gram matrix and the norm closed form"""
    w = workload("P0")
    x = make_inputs(w, seed=24)
    rng = np.random.default_rng(3)
    x.proj = np.ascontiguousarray(x.proj * (0.4 + rng.random(w.nproj)) + 0.3 * x.psi0[..., : w.nproj])
    Dm = dense_D(w, seed=4, scale=0.5)
    got, _ = run_gpu(w, x, 30, Dm, 0)
    want, _ = run_ref(w, x, 30, Dm)
    assert_parity(w, got, want)


def test_dense_sp_variant():
    """complex64 Psi / B with a dense D: within the SP bound n * 30 * 2^-24 of the FP64 oracle"""
    w = workload("P0")
    x = make_inputs(w, seed=25)
    x.psi0 = x.psi0.astype(np.complex64).astype(np.complex128)
    x.proj = x.proj.astype(np.complex64).astype(np.complex128)
    Dm = dense_D(w, seed=5)
    steps = 20
    got, _ = run_gpu(w, x, steps, Dm, 0, sp=True)
    want, _ = run_ref(w, x, steps, Dm)
    e = rel(got[0], want[0])
    assert 1e-9 < e < steps * 30 * 2.0 ** -24, e


def test_dense_rejects_non_hermitian():
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
    w = workload("P0")
    x = make_inputs(w, seed=26)
    Dm = dense_D(w)
    Dm[0, 0, 1] += 0.01
    dev = torch.device("cuda:0")
    with pytest.raises(lfd.LFDError) as e:
        Context(torch.from_numpy(x.psi0.copy()).to(dev), torch.from_numpy(x.proj).to(dev), Dm, x.occ,
                (w.hx, w.hy, w.hz), w.dt, flags=DENSE)
    assert e.value.status == -1
