"""lfd_step_graph (captured CUDA graphs of up to 32 steps + density) against the per-step calls it replaces
(bitwise: same kernels, same order) and against the oracle (1e-10), across chunk boundaries, carry states,
the SP variant, and occupation changes (which must invalidate the captured density tensor maps)."""
import numpy as np
import pytest

from lfd_workloads import make_inputs, workload
from lfd_workloads.generate import midpoint_A

pytestmark = pytest.mark.gpu


def _ctx(w, x, sp=False, flags=0):
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    dev = torch.device("cuda:0")
    dt = np.complex64 if sp else np.complex128
    psi = torch.from_numpy(x.psi0.astype(dt)).to(dev)
    proj = torch.from_numpy(x.proj.astype(dt)).to(dev) if w.nproj else None
    ctx = Context(psi, proj, x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc, flags=flags)
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    return ctx, psi


def _eager(w, x, A, sp=False, flags=0):
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    ctx, psi = _ctx(w, x, sp, flags)
    dev = psi.device
    rho = torch.empty((w.ndom, w.ngrid), dtype=torch.float64, device=dev)
    J = torch.empty((len(A), w.ndom, 3), dtype=torch.float64, device=dev)
    for n in range(len(A)):
        lfd.lfd_set_vector_potential(ctx.ctx, A[n])
        lfd.lfd_step(ctx.ctx, 1)
        lfd.lfd_density_current(ctx.ctx, rho, None, J[n])
    ctx.sync()
    out = psi.cpu().numpy(), rho.cpu().numpy(), J.cpu().numpy()
    ctx.close()
    return out


def _graph(w, x, A, chunks, sp=False, flags=0, occ_change=None):
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    ctx, psi = _ctx(w, x, sp, flags)
    dev = psi.device
    rho = torch.empty((w.ndom, w.ngrid), dtype=torch.float64, device=dev)
    J = torch.empty((len(A), w.ndom, 3), dtype=torch.float64, device=dev)
    n0 = 0
    for i, c in enumerate(chunks):
        if occ_change is not None and i == 1:
            ctx.set_occupations(occ_change)
        lfd.lfd_step_graph(ctx.ctx, A[n0:n0 + c], rho, J[n0:n0 + c])
        n0 += c
    assert n0 == len(A)
    ctx.sync()
    out = psi.cpu().numpy(), rho.cpu().numpy(), J.cpu().numpy()
    ctx.close()
    return out


@pytest.mark.parametrize("name,steps,chunks", [("P0", 70, (70,)), ("P0", 40, (5, 35)), ("P1", 33, (1, 32)),
                                               ("C3", 6, (3, 3))])
def test_graph_bitwise_equals_per_step(name, steps, chunks):
    w = workload(name)
    x = make_inputs(w, seed=91)
    A = np.stack([midpoint_A(w, n) for n in range(steps)])
    a, b = _eager(w, x, A), _graph(w, x, A, chunks)
    for u, v in zip(a, b):
        assert np.array_equal(u, v)


def test_graph_against_oracle_and_sp_and_no_carry():
    from oracle import ref
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    w = workload("P0")
    x = make_inputs(w, seed=92)
    A = np.stack([midpoint_A(w, n) for n in range(40)])
    psi, rho, J = _graph(w, x, A, (40,), flags=lfd.LFD_FLAG_NO_CARRY)
    cfg = ref.RefConfig(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    p = x.psi0.copy()
    for n in range(40):
        ref.step(cfg, p, x.proj, x.dnl, x.vloc, A[n], 1)
    rr, _, Jr = ref.density_current(cfg, p, x.occ, A[-1])
    assert np.linalg.norm(psi - p) / np.linalg.norm(p) < 1e-10
    assert np.linalg.norm(rho - rr) / np.linalg.norm(rr) < 1e-10
    a, b = _eager(w, x, A[:12], sp=True), _graph(w, x, A[:12], (12,), sp=True)
    for u, v in zip(a, b):
        assert np.array_equal(u, v)


def test_graph_after_occupation_change():
    """set_occupations re-encodes the density kernel's tensor maps; cached graphs must be re-captured."""
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    w = workload("P0")
    x = make_inputs(w, seed=93)
    A = np.stack([midpoint_A(w, n) for n in range(8)])
    occ2 = x.occ.copy()
    occ2[:, : w.nocc - 2] = 2.0
    occ2[:, w.nocc - 2:] = 0.0
    got = _graph(w, x, A, (4, 4), occ_change=occ2)
    ctx, psi = _ctx(w, x)
    rho = torch.empty((w.ndom, w.ngrid), dtype=torch.float64, device=psi.device)
    J = torch.empty((8, w.ndom, 3), dtype=torch.float64, device=psi.device)
    for n in range(8):
        if n == 4:
            ctx.set_occupations(occ2)
        lfd.lfd_set_vector_potential(ctx.ctx, A[n])
        lfd.lfd_step(ctx.ctx, 1)
        lfd.lfd_density_current(ctx.ctx, rho, None, J[n])
    ctx.sync()
    assert np.array_equal(got[1], rho.cpu().numpy()) and np.array_equal(got[2], J.cpu().numpy())
    ctx.close()


@pytest.mark.parametrize("name,steps,chunks", [("P0", 40, (5, 35)), ("C1", 12, (1, 11))])
def test_graph_bitwise_with_int8_gemms(name, steps, chunks):
    """the int8-digit tensor-core GEMMs (forced on these small grids) under capture: the orbital-exponent
    handshake (k_kin_yz -> k_gemm1_i8, cleared by its last CTA) and the completion counters replay exactly"""
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    w = workload(name)
    x = make_inputs(w, seed=44)
    A = np.stack([midpoint_A(w, n) for n in range(steps)])
    a = _eager(w, x, A, flags=lfd.LFD_FLAG_NL_I8)
    b = _graph(w, x, A, chunks, flags=lfd.LFD_FLAG_NL_I8)
    for u, v in zip(a, b):
        assert np.array_equal(u, v)
