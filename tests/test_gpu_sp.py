"""GPU parity of the SP variant (LFD_FLAG_SP: complex64 Psi / B, FP32 sweeps, int8-digit or 3xTF32 tensor-core projector
GEMMs, FP64 small kernels) against the FP64 oracle, through the C ABI.

Tolerance: every step rounds each orbital value O(30) times at the FP32 unit roundoff
u = 2^-24 (9 pair sweeps with 2 roundings each, two phase multiplies, two nonlocal updates, the 3xTF32
products at ~u), and the propagator is unitary, so errors add at most linearly:
    ||Psi_sp - Psi_ref|| / ||Psi_ref|| <= n_steps * 30 * 2^-24  (1.8e-4 after 100 steps),
the same bound for rho and j (quadratic in Psi: twice the relative error, within the factor 30 margin),
|J_sp - J_ref| <= the bound x mean|j_ref|. The inputs of both sides are the complex64 values (the oracle
reads them widened to complex128), so input rounding is not counted."""
import numpy as np
import pytest

from lfd_workloads import make_inputs, workload
from lfd_workloads.generate import midpoint_A

pytestmark = pytest.mark.gpu


def sp_tol(steps):
    return max(steps, 1) * 30 * 2.0 ** -24


def _inputs(w, seed):
    x = make_inputs(w, seed=seed)
    x.psi0 = x.psi0.astype(np.complex64)
    if x.proj is not None:
        x.proj = x.proj.astype(np.complex64)
    return x


def _gpu(w, x, steps, flags=0, sequence=False, energy=False):
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context
    dev = torch.device("cuda:0")
    psi = torch.from_numpy(x.psi0.copy()).to(dev)
    proj = torch.from_numpy(x.proj).to(dev) if w.nproj else None
    ctx = Context(psi, proj, x.dnl, x.occ, (w.hx, w.hy, w.hz), w.dt, bc=w.bc, flags=flags)
    ctx.set_potential(torch.from_numpy(x.vloc).to(dev))
    if sequence:
        ctx.step_sequence(np.stack([midpoint_A(w, n) for n in range(steps)]))
    else:
        for n in range(steps):
            ctx.set_vector_potential(midpoint_A(w, n))
            ctx.step(1)
    ctx.set_vector_potential(midpoint_A(w, steps - 1))
    rho, j, J = ctx.density_current()
    E = ctx.energy() if energy else None
    ctx.sync()
    out = (psi.cpu().numpy().astype(np.complex128), rho.cpu().numpy().reshape(w.ndom, -1),
           j.cpu().numpy().reshape(w.ndom, 3, -1), J.cpu().numpy(), None if E is None else E.cpu().numpy())
    ctx.close()
    return out


def _ref(w, x, steps, exact=False):
    from oracle import ref
    cfg = ref.RefConfig(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    p = x.psi0.astype(np.complex128)
    B = x.proj.astype(np.complex128) if w.nproj else None
    for n in range(steps):
        (ref.step_exact if exact else ref.step)(cfg, p, B, x.dnl if w.nproj else None, x.vloc, midpoint_A(w, n), 1)
    A = midpoint_A(w, steps - 1)
    rho, j, J = ref.density_current(cfg, p, x.occ, A)
    E = ref.energy(cfg, p, x.occ, x.vloc, A, B, x.dnl if w.nproj else None)
    return p, rho, j, J, E


def rel(a, b):
    return np.linalg.norm(a - b) / np.linalg.norm(b)


def assert_sp(w, got, want, steps):
    tol = sp_tol(steps)
    psi, rho, j, J, _ = got
    rpsi, rrho, rj, rJ, _ = want
    e = (rel(psi, rpsi), rel(rho, rrho), np.linalg.norm(j - rj) / max(np.linalg.norm(rj), 1e-3 * np.linalg.norm(rrho)),
         np.abs(J - rJ).max() / max(np.abs(rj).mean(), 1e-3 * np.abs(rrho).mean()))
    assert max(e) <= tol, (e, tol)
    assert e[0] > 1e-9  # it really ran in single precision
    return e


@pytest.mark.parametrize("name,steps", [("P0", 100), ("P1", 20), ("P2z", 20), ("P3", 5), ("C1", 10)])
def test_sp_parity(name, steps):
    w = workload(name)
    x = _inputs(w, 81)
    assert_sp(w, _gpu(w, x, steps), _ref(w, x, steps), steps)


def test_sp_sequence_and_energy():
    w = workload("P0")
    x = _inputs(w, 82)
    got = _gpu(w, x, 40, sequence=True, energy=True)
    want = _ref(w, x, 40)
    assert_sp(w, got, want, 40)
    assert np.abs(got[4] - want[4]).max() <= sp_tol(40) * np.abs(want[4]).max()


def test_sp_exact_nl_and_no_carry():
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    w = workload("P0")
    x = _inputs(w, 83)
    want = _ref(w, x, 30, exact=True)
    assert_sp(w, _gpu(w, x, 30, flags=lfd.LFD_FLAG_EXACT_NL), want, 30)
    assert_sp(w, _gpu(w, x, 30, flags=lfd.LFD_FLAG_EXACT_NL | lfd.LFD_FLAG_NO_CARRY), want, 30)


def test_sp_c2_full_size_two_steps():
    """The bench shape (70x70x72, 64 orbitals, 64 projectors) in SP: sampled orbitals against the oracle."""
    from oracle import ref
    w = workload("C2")
    x = _inputs(w, 84)
    got = _gpu(w, x, 2)
    cols = [0, 17, 63]
    cfg = ref.RefConfig(1, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, len(cols), w.nproj, w.dt)
    p = np.ascontiguousarray(x.psi0[..., cols].astype(np.complex128))
    for n in range(2):
        ref.step(cfg, p, x.proj.astype(np.complex128), x.dnl, x.vloc, midpoint_A(w, n), 1)
    assert rel(got[0][..., cols], p) <= sp_tol(2)


@pytest.mark.parametrize("name,steps", [("P0", 100), ("P1", 20), ("P2z", 20), ("C1", 10)])
def test_sp_parity_int8_digit_gemms(name, steps):
    """the SP projector GEMMs on the tcgen05 int8 tensor cores (4 digits per operand; forced on these small grids,
    the default at C2): same bound; the orbital exponents for GEMM-1 come from the SP z pass"""
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    w = workload(name)
    x = _inputs(w, 85)
    assert_sp(w, _gpu(w, x, steps, flags=lfd.LFD_FLAG_NL_I8), _ref(w, x, steps), steps)


def test_sp_int8_sequence_energy_exact():
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    w = workload("P0")
    x = _inputs(w, 86)
    got = _gpu(w, x, 40, flags=lfd.LFD_FLAG_NL_I8, sequence=True, energy=True)
    want = _ref(w, x, 40)
    assert_sp(w, got, want, 40)
    assert np.abs(got[4] - want[4]).max() <= sp_tol(40) * np.abs(want[4]).max()
    want_x = _ref(w, x, 30, exact=True)
    assert_sp(w, _gpu(w, x, 30, flags=lfd.LFD_FLAG_NL_I8 | lfd.LFD_FLAG_EXACT_NL), want_x, 30)


def test_sp_c2_default_path_is_int8_tensor_cores():
    import torch
    from paper_conf_ipps_razakhllknvn24_b200 import Context, lfd
    w = workload("C2")
    x = _inputs(w, 87)
    dev = torch.device("cuda:0")
    ctx = Context(torch.from_numpy(x.psi0).to(dev), torch.from_numpy(x.proj).to(dev), x.dnl, x.occ,
                  (w.hx, w.hy, w.hz), w.dt)
    assert lfd.lfd_nl_path(ctx.ctx) == 3
    ctx.close()


@pytest.mark.parametrize("case", ["periodic", "zero_bc_odd_nx"])
def test_sp_fused_first_factor(case):
    """The SP first factor's GEMM-2 fused with Phi . K_x (k_gemm2x_i8 on complex64 lines, 4 digits, the march in
    FP32): shapes that select it (even orbital count, ny nz even) with the int8-digit GEMMs forced -- periodic
    (segmented march) and zero BC with an odd nx (whole-line march) -- at the SP bound over 60 steps."""
    from paper_conf_ipps_razakhllknvn24_b200 import lfd
    if case == "periodic":
        w = workload("P0").with_(nx=20, norb=8, nocc=6)
    else:
        w = workload("P2z").with_(ny=6, nz=10, norb=4, nocc=4)
    x = _inputs(w, 88)
    steps = 60
    assert_sp(w, _gpu(w, x, steps, flags=lfd.LFD_FLAG_NL_I8), _ref(w, x, steps), steps)
