"""GPU parity of the exactly unitary nonlocal factor (LFD_FLAG_EXACT_NL) against
the oracle's lfd_ref_step_exact, through the C ABI: per-step calls (projection carry on and off), the
merged-factor sequence, several domains, orthonormality conservation with a large scissor, and the
EINVAL for non-orthonormal projector columns. Tolerance: the north star's 1e-10 (FP64)."""
import numpy as np
import pytest

from lfd_workloads import make_inputs, workload
from lfd_workloads.generate import midpoint_A

from .test_gpu_parity import assert_parity, rel

pytestmark = pytest.mark.gpu


def _gpu(w, x, steps, flags, sequence=False, dnl=None):
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    d = x.dnl if dnl is None else dnl
    ctx = Context(psi, torch.from_numpy(x.proj).to(dev), d, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc,
                  flags=flags | lfd.LFD_FLAG_EXACT_NL)
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    if sequence:
        ctx.step_sequence(np.stack([midpoint_A(w, n) for n in range(steps)]))
    else:
        for n in range(steps):
            ctx.set_vector_potential(midpoint_A(w, n))
            ctx.step(1)
    ctx.set_vector_potential(midpoint_A(w, steps - 1))
    rho, j, J = ctx.density_current()
    ctx.sync()
    out = (psi.cpu().numpy(), rho.cpu().numpy().reshape(w.ndom, -1), j.cpu().numpy().reshape(w.ndom, 3, -1),
           J.cpu().numpy())
    ctx.close()
    return out


def _ref(w, x, steps, dnl=None):
    from oracle import ref
    cfg = ref.RefConfig(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    p = x.psi0.copy()
    d = x.dnl if dnl is None else dnl
    for n in range(steps):
        ref.step_exact(cfg, p, x.proj, d, x.vloc, midpoint_A(w, n), 1)
    rho, j, J = ref.density_current(cfg, p, x.occ, midpoint_A(w, steps - 1))
    return p, rho, j, J


@pytest.mark.parametrize("name,steps,seq", [("P0", 100, False), ("P0", 40, True), ("P2z", 20, False),
                                            ("P1", 10, False), ("C3", 10, True)])
def test_exact_nl_parity(name, steps, seq):
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    w = workload(name) if name != "C3" else workload("C3").with_(a_spread=0.1, vnoise=0.02)
    x = make_inputs(w, seed=51)
    want = _ref(w, x, steps)
    got = _gpu(w, x, steps, 0, sequence=seq)
    assert_parity(w, got, want)
    if not seq:
        got2 = _gpu(w, x, steps, lfd.LFD_FLAG_NO_CARRY)
        assert rel(got[0], got2[0]) < 1e-13


def test_exact_nl_keeps_orthonormality_with_large_scissor():
    w = workload("C1").with_(laser=True, e0=0.02, pol=(0.3, -0.4, 0.87))
    x = make_inputs(w, seed=52)
    big = np.ascontiguousarray(x.dnl * 30.0)
    psi, *_ = _gpu(w, x, 50, 0, dnl=big)
    P = psi.reshape(-1, w.norb)
    S = w.dV * P.conj().T @ P
    assert np.abs(S - np.eye(w.norb)).max() < 1e-12
    want = _ref(w, x, 50, dnl=big)
    assert rel(psi, want[0]) < 1e-10


def test_exact_nl_rejects_nonorthonormal_projectors():
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
    w = workload("P0")
    x = make_inputs(w, seed=53)
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    proj = torch.from_numpy(x.proj * 1.01).to(dev)
    with pytest.raises(lfd.LFDError) as e:
        Context(psi, proj, x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, flags=lfd.LFD_FLAG_EXACT_NL)
    assert e.value.status == -1
