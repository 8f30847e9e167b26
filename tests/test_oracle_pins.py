"""Pins of the CPU oracle against what the mathematics fixes (no GPU; `-m "not gpu"`).

Each test names the passage / reading it pins (PAPER.md line "P:n", SURVEY.md §8(c) reading "Rn").
None of them re-types the oracle's formulas: the ground truths are dense library matrix
exponentials, textbook FD operators, closed forms (free-electron plane waves), invariants
(norm, orthonormality, time reversal, gauge covariance) and derived identities (Gram closed form).
"""
from __future__ import annotations

import numpy as np
import pytest
from scipy.linalg import expm

from oracle import ref
from tests import _dense as D

C = ref.C_LIGHT


def cfg_of(nx, ny, nz, h=(0.3, 0.35, 0.4), bc=ref.BC_PERIODIC, norb=3, nproj=0, dt=0.04, ndom=1):
    return ref.RefConfig(ndom, nx, ny, nz, h[0], h[1], h[2], bc, norb, nproj, dt)


def rand_psi(rng, shape):
    return (rng.standard_normal(shape) + 1j * rng.standard_normal(shape)).astype(np.complex128)


# --- R3/R4: the link sets are a splitting of the textbook FD Peierls operator -------------------

@pytest.mark.parametrize("n,bc", [(8, D.PERIODIC), (2, D.PERIODIC), (10, D.PERIODIC), (7, D.ZERO), (8, D.ZERO), (2, D.ZERO)])
def test_link_sets_sum_to_fd_operator(n, bc):
    h, a = 0.3, 0.7
    HE = D.link_set_hamiltonian(n, h, a, bc, 0)
    HO = D.link_set_hamiltonian(n, h, a, bc, 1)
    assert np.abs(HE + HO - D.fd_peierls_1d(n, h, a, bc)).max() < 1e-12
    assert np.abs(HE - HE.conj().T).max() == 0 and np.abs(HO - HO.conj().T).max() == 0


def test_fd_operator_plane_wave_dispersion():
    """R2: hopping to r+e_d carries e^{+i a h}: a plane wave e^{ikx} has (1-cos((k+a)h))/h^2."""
    n, h, a = 12, 0.3, 0.7
    T = D.fd_peierls_1d(n, h, a, D.PERIODIC)
    k = 2 * np.pi * 3 / (n * h)
    psi = np.exp(1j * k * h * np.arange(n))
    assert np.allclose(T @ psi, (1 - np.cos((k + a) * h)) / h**2 * psi, atol=1e-12)


# --- one E/O sweep == exact exponential of its link-set generator (Alg. 1-3; R4, R5, R8) ---

@pytest.mark.parametrize("bc,dims", [(ref.BC_PERIODIC, (8, 4, 6)), (ref.BC_ZERO, (7, 5, 4)), (ref.BC_ZERO, (4, 3, 2))])
@pytest.mark.parametrize("axis", [0, 1, 2])
@pytest.mark.parametrize("parity", [0, 1])
def test_link_sweep_matches_dense_expm(bc, dims, axis, parity):
    rng = np.random.default_rng(10 + axis + 3 * parity)
    h = (0.3, 0.35, 0.4)
    cfg = cfg_of(*dims, h=h, bc=bc, norb=3)
    psi = rand_psi(rng, dims + (3,))
    tau, a = 0.037, 0.9 - 0.6 * axis
    ref_out = psi.copy()
    ref.link_sweep(cfg, ref_out, axis, parity, tau, a)
    Hd = D.link_set_hamiltonian(dims[axis], h[axis], a, bc, parity)
    U = D.axis_op(expm(-1j * tau * Hd), axis, dims)
    want = (U @ psi.reshape(-1, 3)).reshape(psi.shape)
    assert np.abs(ref_out - want).max() < 1e-14 * np.abs(psi).max() * 10


# --- K_d on free-electron plane waves (closed form, R2/R4) -------------------------------------

@pytest.mark.parametrize("khpa", [0.0, np.pi])
def test_kinetic_plane_wave_exact_phase(khpa):
    """(k+a)h in {0, pi}: the plane wave is an eigenvector of every link, so 100 K_x steps give
    exactly exp(-i n dt (1-cos((k+a)h))/h^2)."""
    nx, h, dt, steps = 8, 0.3, 0.04, 100
    cfg = cfg_of(nx, 2, 2, h=(h, 0.5, 0.5), norb=1, dt=dt)
    m = 2
    k = 2 * np.pi * m / (nx * h)
    a = khpa / h - k
    psi = np.exp(1j * k * h * np.arange(nx))[:, None, None, None] * np.ones((nx, 2, 2, 1))
    psi = psi.astype(np.complex128)
    p = psi.copy()
    for _ in range(steps):
        ref.kinetic(cfg, p, 0, dt, a)
    E = (1 - np.cos((k + a) * h)) / h**2
    assert np.abs(p - psi * np.exp(-1j * steps * dt * E)).max() < 1e-13


def test_kinetic_second_order_in_dt():
    """Generic k: global error vs the exact FD evolution shrinks 4x per halving of dt."""
    nx, h, a, T = 10, 0.3, 0.31, 0.8
    k = 2 * np.pi * 1 / (nx * h)
    x = h * np.arange(nx)
    errs = []
    for dt in (0.08, 0.04, 0.02):
        cfg = cfg_of(nx, 2, 2, h=(h, 0.5, 0.5), norb=1, dt=dt)
        rng = np.random.default_rng(3)
        psi = rand_psi(rng, (nx, 1, 1, 1))
        psi = np.repeat(np.repeat(psi, 2, axis=1), 2, axis=2)
        p = psi.copy()
        for _ in range(int(round(T / dt))):
            ref.kinetic(cfg, p, 0, dt, a)
        Tfd = D.fd_peierls_1d(nx, h, a, D.PERIODIC)
        want = expm(-1j * T * Tfd) @ psi[:, 0, 0, 0]
        errs.append(np.abs(p[:, 0, 0, 0] - want).max())
    r1, r2 = errs[0] / errs[1], errs[1] / errs[2]
    assert 3.5 < r1 < 4.6 and 3.5 < r2 < 4.6, errs
    del k, x


# --- full local propagator == product of dense exponentials (Eq. 6 local factor; R6, R7) --------

def _dense_local(dims, h, a3, v, dt, bc):
    Phi = np.diag(np.exp(-0.5j * dt * v.reshape(-1)))
    U = Phi.copy()
    for d in range(3):
        U = D.axis_op(D.split_kinetic_dense(dims[d], h[d], a3[d], bc, dt), d, dims) @ U
    return Phi @ U


@pytest.mark.parametrize("bc,dims", [(ref.BC_PERIODIC, (4, 4, 6)), (ref.BC_ZERO, (3, 5, 4))])
def test_local_matches_dense_product(bc, dims):
    rng = np.random.default_rng(7)
    h = (0.3, 0.35, 0.4)
    A = np.array([0.2, -0.5, 0.9]) * C
    v = rng.standard_normal(dims)
    dt = 0.04
    cfg = cfg_of(*dims, h=h, bc=bc, norb=2, dt=dt)
    psi = rand_psi(rng, dims + (2,))
    out = psi.copy()
    ref.local(cfg, out, v, A)
    U = _dense_local(dims, h, A / C, v, dt, bc)
    want = (U @ psi.reshape(-1, 2)).reshape(psi.shape)
    assert np.abs(out - want).max() < 1e-13


def test_local_converges_second_order_to_exact():
    """Local step -> expm(-i dt (T + V)): global error ratio ~4 per dt halving (Eq. 4/6)."""
    dims, h = (4, 4, 6), (0.3, 0.35, 0.4)
    rng = np.random.default_rng(5)
    a3 = np.array([0.2, -0.5, 0.9])
    v = rng.standard_normal(dims)
    H = sum(D.axis_op(D.fd_peierls_1d(dims[d], h[d], a3[d], D.PERIODIC), d, dims) for d in range(3))
    H = H + np.diag(v.reshape(-1))
    psi0 = rand_psi(rng, dims + (1,))
    Ttot = 0.4
    want = expm(-1j * Ttot * H) @ psi0.reshape(-1)
    errs = []
    for dt in (0.04, 0.02, 0.01):
        cfg = cfg_of(*dims, h=h, norb=1, dt=dt)
        p = psi0.copy()
        for _ in range(int(round(Ttot / dt))):
            ref.local(cfg, p, v, a3 * C)
        errs.append(np.abs(p.reshape(-1) - want).max())
    assert 3.6 < errs[0] / errs[1] < 4.4 and 3.6 < errs[1] / errs[2] < 4.4, errs


def test_directions_commute():
    """R6: K_x, K_y, K_z act on different tensor factors, so any order agrees to roundoff."""
    rng = np.random.default_rng(1)
    dims = (6, 4, 8)
    cfg = cfg_of(*dims, norb=5)
    psi = rand_psi(rng, dims + (5,))
    p1, p2 = psi.copy(), psi.copy()
    for d in (0, 1, 2):
        ref.kinetic(cfg, p1, d, 0.05, 0.3 * d - 0.2)
    for d in (2, 0, 1):
        ref.kinetic(cfg, p2, d, 0.05, 0.3 * d - 0.2)
    assert np.abs(p1 - p2).max() < 1e-14


# --- invariants of the full step (Eq. 6) --------------------------------------------------

def test_time_reversal_real_symmetric_case():
    """A = 0, no NL, real v, real psi0: U is symmetric and unitary, so U^n conj(U^n psi0) = psi0."""
    rng = np.random.default_rng(2)
    dims = (6, 4, 8)
    cfg = cfg_of(*dims, norb=3, dt=0.04)
    v = rng.standard_normal(dims)
    psi0 = rng.standard_normal(dims + (3,)).astype(np.complex128)
    p = psi0.copy()
    ref.step(cfg, p, None, None, v, np.zeros(3), 50)
    p = np.ascontiguousarray(p.conj())
    ref.step(cfg, p, None, None, v, np.zeros(3), 50)
    assert np.abs(p - psi0).max() < 1e-13


def test_gauge_covariance():
    """a_d L_d in 2 pi Z: U(a) psi = G U(0) G^dagger psi, G = e^{-i a.r} (R2; no NL)."""
    rng = np.random.default_rng(4)
    dims, h = (6, 4, 8), (0.3, 0.35, 0.4)
    L = np.array(dims) * np.array(h)
    a3 = 2 * np.pi * np.array([1, -1, 2]) / L
    cfg = cfg_of(*dims, h=h, norb=2, dt=0.03)
    v = rng.standard_normal(dims)
    psi = rand_psi(rng, dims + (2,))
    X, Y, Z = np.meshgrid(*(h[i] * np.arange(dims[i]) for i in range(3)), indexing="ij")
    G = np.exp(-1j * (a3[0] * X + a3[1] * Y + a3[2] * Z))[..., None]
    pa = psi.copy()
    ref.step(cfg, pa, None, None, v, a3 * C, 3)
    p0 = np.ascontiguousarray(psi * G.conj())
    ref.step(cfg, p0, None, None, v, np.zeros(3), 3)
    assert np.abs(pa - G * p0).max() < 1e-13


# --- nonlocal factor (Eq. 6 denominator, Eq. 7, Eq. 9; R9-R12) ---------------------------------

def _orthonormal(rng, ng, k, dV):
    q, _ = np.linalg.qr(rand_psi(rng, (ng, k)))
    return q / np.sqrt(dV)


def test_nl_identity_when_orthogonal_to_projectors():
    rng = np.random.default_rng(8)
    dims = (4, 4, 4)
    cfg = cfg_of(*dims, norb=3, nproj=4)
    Q = _orthonormal(rng, 64, 7, cfg.dV)
    psi = np.ascontiguousarray(Q[:, :3].reshape(dims + (3,)))
    B = np.ascontiguousarray(Q[:, 3:].reshape(dims + (4,)))
    out = psi.copy()
    ref.nl_half(cfg, out, B, np.array([0.1, 0.2, 0.3, 0.4]))
    assert np.abs(out - psi).max() < 1e-14


def test_nl_on_projector_columns_closed_form():
    """psi_s = B_u (orthonormal B): (1 - i eps D_u P) B_u = (1 - i eps D_u) B_u, renormalised
    -> B_u (1 - i eps D_u)/|1 - i eps D_u|; distinct D_u catch index mix-ups, the phase sign catches
    a wrong sign of i, the modulus catches a missing dV or conj."""
    rng = np.random.default_rng(9)
    dims = (4, 6, 2)
    dt = 0.5
    cfg = cfg_of(*dims, norb=3, nproj=5, dt=dt)
    B = _orthonormal(rng, 48, 5, cfg.dV)
    Dn = np.array([0.3, -1.1, 0.7, 2.0, 0.05])
    cols = [3, 0, 2]
    psi = np.ascontiguousarray(B[:, cols].reshape(dims + (3,)))
    out = psi.copy()
    ref.nl_half(cfg, out, np.ascontiguousarray(B.reshape(dims + (5,))), Dn)
    eps = dt / 2
    fac = (1 - 1j * eps * Dn[cols]) / np.abs(1 - 1j * eps * Dn[cols])
    assert np.abs(out - psi * fac).max() < 1e-14


def test_nl_gram_closed_form_nonorthonormal():
    """Per-half Gram map S' = N (S + eps^2 (DC)^H G (DC)) N with C = dV B^H psi, G = dV B^H B,
    N = diag(n), n_s = sqrt(S_ss / (S + eps^2 (DC)^H G (DC))_ss), for NON-orthonormal B; norms kept."""
    rng = np.random.default_rng(11)
    dims = (4, 4, 6)
    dt = 0.3
    cfg = cfg_of(*dims, norb=4, nproj=3, dt=dt)
    psi = rand_psi(rng, dims + (4,)) * 0.2
    B = rand_psi(rng, dims + (3,)) * 0.3
    Dn = np.array([0.4, -0.9, 1.3])
    P, Bm = psi.reshape(-1, 4), B.reshape(-1, 3)
    dV, eps = cfg.dV, dt / 2
    S = dV * P.conj().T @ P
    Cm = dV * Bm.conj().T @ P
    G = dV * Bm.conj().T @ Bm
    DC = Dn[:, None] * Cm
    M = S + eps**2 * DC.conj().T @ G @ DC
    n = np.sqrt(np.diag(S).real / np.diag(M).real)
    want = n[:, None] * M * n[None, :]
    out = psi.copy()
    ref.nl_half(cfg, out, B, Dn)
    O = out.reshape(-1, 4)
    got = dV * O.conj().T @ O
    assert np.abs(got - want).max() < 1e-13 * np.abs(want).max()
    assert np.abs(np.diag(got) - np.diag(S)).max() < 1e-13


def test_step_conserves_norm_and_D0_orthonormality():
    """Norm conserved every step (NL on); with D = 0 the whole step is unitary so dV Psi^H Psi = I."""
    from lfd_workloads import make_inputs, workload
    from lfd_workloads.generate import midpoint_A
    w = workload("P0")
    x = make_inputs(w, seed=3)
    cfg = ref.RefConfig(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    for Dscale in (1.0, 0.0):
        p = x.psi0.copy()
        for n in range(100):
            ref.step(cfg, p, x.proj, x.dnl * Dscale, x.vloc, midpoint_A(w, n), 1)
        P = p.reshape(-1, w.norb)
        S = w.dV * P.conj().T @ P
        # 100 steps x (9 sweeps + 2 phases + 2 NL halves) ~ 1300 unitary maps, each adding O(1e-16)
        # rounding: a random-walk budget of 5e-13 (observed ~1e-13).
        assert np.abs(np.diag(S) - 1).max() < 5e-13
        if Dscale == 0.0:
            assert np.abs(S - np.eye(w.norb)).max() < 5e-13


def test_domains_independent():
    from lfd_workloads import make_inputs, workload
    w = workload("P1")
    x = make_inputs(w, seed=2)
    cfg = ref.RefConfig(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    A = np.array([[1.0, 2.0, -3.0], [0.5, -1.0, 4.0]])
    p = x.psi0.copy()
    ref.step(cfg, p, x.proj, x.dnl, x.vloc, A, 2)
    one = ref.RefConfig(1, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    for dm in range(2):
        q = x.psi0[dm:dm + 1].copy()
        ref.step(one, q, np.ascontiguousarray(x.proj[dm:dm + 1]), np.ascontiguousarray(x.dnl[dm:dm + 1]),
                 np.ascontiguousarray(x.vloc[dm:dm + 1]), A[dm], 2)
        assert np.array_equal(q, p[dm:dm + 1])


# --- density and current (R13, R14) -------------------------------------------------------

def test_plane_wave_density_current_energy_closed_forms():
    dims, h = (6, 4, 8), (0.3, 0.35, 0.4)
    L = np.array(dims) * np.array(h)
    V = L.prod()
    m = np.array([1, -1, 3])
    k = 2 * np.pi * m / L
    a3 = np.array([0.3, 0.7, -0.2])
    X, Y, Z = np.meshgrid(*(h[i] * np.arange(dims[i]) for i in range(3)), indexing="ij")
    psi = (np.exp(1j * (k[0] * X + k[1] * Y + k[2] * Z)) / np.sqrt(V))[..., None].astype(np.complex128)
    cfg = cfg_of(*dims, h=h, norb=1)
    f = np.array([[2.0]])
    rho, j, J = ref.density_current(cfg, psi, f, a3 * C)
    assert np.abs(rho - 2.0 / V).max() < 1e-14
    jw = 2.0 * np.sin((k + a3) * np.array(h)) / (np.array(h) * V)
    for d in range(3):
        assert np.abs(j[0, d] - jw[d]).max() < 1e-13
        assert abs(J[0, d] - jw[d]) < 1e-13
    Ew = 2.0 * np.sum((1 - np.cos((k + a3) * np.array(h))) / np.array(h) ** 2)
    assert abs(ref.kinetic_energy(cfg, psi, f[0], a3 * C) - Ew) < 1e-12


@pytest.mark.parametrize("bc,dims", [(ref.BC_PERIODIC, (6, 4, 8)), (ref.BC_ZERO, (5, 4, 3))])
def test_current_is_derivative_of_kinetic_energy(bc, dims):
    """R13: grid-mean link current J_d = (1/V) dE_kin/da_d (central difference); E_kin itself
    equals <psi|T|psi> with the textbook dense FD operator."""
    rng = np.random.default_rng(6)
    h = (0.3, 0.35, 0.4)
    cfg = cfg_of(*dims, h=h, bc=bc, norb=3)
    psi = rand_psi(rng, dims + (3,)) * 0.1
    f = np.array([2.0, 1.0, 0.5])
    a3 = np.array([0.31, -0.2, 0.45])
    T = sum(D.axis_op(D.fd_peierls_1d(dims[d], h[d], a3[d], bc), d, dims) for d in range(3))
    P = psi.reshape(-1, 3)
    Ed = cfg.dV * sum(f[s] * np.vdot(P[:, s], T @ P[:, s]).real for s in range(3))
    assert abs(ref.kinetic_energy(cfg, psi, f, a3 * C) - Ed) < 1e-12 * abs(Ed)
    V = cfg.dV * np.prod(dims)
    _, _, J = ref.density_current(cfg, psi, f[None, :], a3 * C)
    da = 1e-5
    for d in range(3):
        ap, am = a3.copy(), a3.copy()
        ap[d] += da
        am[d] -= da
        dE = (ref.kinetic_energy(cfg, psi, f, ap * C) - ref.kinetic_energy(cfg, psi, f, am * C)) / (2 * da)
        assert abs(J[0, d] - dE / V) < 1e-8 * max(1.0, abs(dE / V))


def test_density_sum_rule():
    rng = np.random.default_rng(12)
    dims = (4, 6, 4)
    cfg = cfg_of(*dims, norb=4)
    psi = rand_psi(rng, dims + (4,))
    f = np.array([[2.0, 2.0, 1.0, 0.0]])
    rho, _, _ = ref.density_current(cfg, psi, f, np.zeros(3))
    P = psi.reshape(-1, 4)
    want = sum(f[0, s] * np.vdot(P[:, s], P[:, s]).real for s in range(4)) * cfg.dV
    assert abs(rho.sum() * cfg.dV - want) < 1e-12 * want


def test_zero_current_real_orbitals_and_real_eigenvectors():
    """North star: j == 0 for real psi at A = 0; real eigenvectors of the (symmetric unitary) one-step
    operator keep j == 0 and rho constant for 100 steps."""
    rng = np.random.default_rng(13)
    dims = (4, 4, 4)
    cfg = cfg_of(*dims, norb=1, dt=0.04)
    v = rng.standard_normal(dims)
    psi = rng.standard_normal(dims + (1,)).astype(np.complex128)
    _, j, _ = ref.density_current(cfg, psi, np.array([[2.0]]), np.zeros(3))
    assert np.abs(j).max() == 0.0
    ng = 64
    U = np.zeros((ng, ng), dtype=np.complex128)
    for i in range(ng):
        e = np.zeros(dims + (1,), dtype=np.complex128)
        e.reshape(-1)[i] = 1
        ref.step(cfg, e, None, None, v, np.zeros(3), 1)
        U[:, i] = e.reshape(-1)
    assert np.abs(U - U.T).max() < 1e-15 and np.abs(U.conj().T @ U - np.eye(ng)).max() < 1e-14
    _, Vr = np.linalg.eigh(U.real + 0.6180339887 * U.imag)  # commuting real symmetric parts
    vec = Vr[:, 5].astype(np.complex128).reshape(dims + (1,))
    vec /= np.sqrt(cfg.dV)
    rho0, _, _ = ref.density_current(cfg, vec, np.array([[2.0]]), np.zeros(3))
    p = vec.copy()
    ref.step(cfg, p, None, None, v, np.zeros(3), 100)
    rho, j, _ = ref.density_current(cfg, p, np.array([[2.0]]), np.zeros(3))
    assert np.abs(j).max() < 1e-12 * np.abs(rho0).max()
    assert np.abs(rho - rho0).max() < 1e-12 * np.abs(rho0).max()


def test_oracle_rejects_bad_config():
    with pytest.raises(RuntimeError):
        ref.step(cfg_of(5, 4, 4), np.zeros((5, 4, 4, 3), np.complex128), None, None,
                 np.zeros((5, 4, 4)), np.zeros(3))
