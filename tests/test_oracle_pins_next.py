"""Pins of the oracle's NEXT-row functions: calc_energy and remap_occ
(P:212 names both; Fig. 5 P:302 times the energy kernel; P:58 motivates the occupation handshake)."""
import numpy as np
import pytest

from oracle import ref

C = ref.C_LIGHT


def cfg_of(nx, ny, nz, h=(0.3, 0.35, 0.4), bc=ref.BC_PERIODIC, norb=3, nproj=0, dt=0.04, ndom=1):
    return ref.RefConfig(ndom, nx, ny, nz, h[0], h[1], h[2], bc, norb, nproj, dt)


def plane_wave(dims, h, m):
    L = np.array(dims) * np.array(h)
    k = 2 * np.pi * np.array(m) / L
    X, Y, Z = np.meshgrid(*(h[i] * np.arange(dims[i]) for i in range(3)), indexing="ij")
    return (np.exp(1j * (k[0] * X + k[1] * Y + k[2] * Z)) / np.sqrt(L.prod()))[..., None], k


def test_energy_plane_wave_closed_forms():
    """Free plane wave in a potential v: E_kin = f sum_d (1-cos((k+a)h))/h^2, E_loc = f mean(v)."""
    dims, h = (6, 4, 8), (0.3, 0.35, 0.4)
    psi, k = plane_wave(dims, h, (1, 0, -2))
    psi = np.ascontiguousarray(psi)
    a3 = np.array([0.2, -0.1, 0.3])
    rng = np.random.default_rng(0)
    v = rng.standard_normal(dims)
    E = ref.energy(cfg_of(*dims, h=h, norb=1), psi, np.array([[2.0]]), v, a3 * C)
    ek = 2.0 * np.sum((1 - np.cos((k + a3) * np.array(h))) / np.array(h) ** 2)
    assert abs(E[0, 0] - ek) < 1e-12
    assert abs(E[0, 1] - 2.0 * v.mean()) < 1e-12
    assert E[0, 2] == 0.0 and abs(E[0, 3] - E[0, :3].sum()) < 1e-15


def test_energy_nonlocal_on_projector_columns():
    """psi_s = B_u (orthonormal B): <psi|sum D |B><B| |psi> = D_u; orthogonal psi gives 0."""
    rng = np.random.default_rng(1)
    dims = (4, 4, 4)
    cfg = cfg_of(*dims, norb=3, nproj=4)
    q, _ = np.linalg.qr(rng.standard_normal((64, 7)) + 1j * rng.standard_normal((64, 7)))
    q /= np.sqrt(cfg.dV)
    B = np.ascontiguousarray(q[:, :4].reshape(dims + (4,)))
    Dn = np.array([0.1, -0.7, 1.3, 0.4])
    f = np.array([2.0, 1.0, 0.5])
    psi = np.ascontiguousarray(q[:, [2, 0, 5]].reshape(dims + (3,)))  # B_2, B_0, and one orthogonal
    E = ref.energy(cfg, psi, f[None], np.zeros(dims), np.zeros(3), B, Dn[None])
    assert abs(E[0, 2] - (2.0 * Dn[2] + 1.0 * Dn[0])) < 1e-13


def test_energy_drift_second_order_at_A0_D0():
    """A = 0, D = 0: the split step conserves a shadow Hamiltonian, so <h> oscillates with an O(dt^2)
    amplitude: the max drift over a fixed time shrinks ~4x per halving of dt."""
    dims, h = (6, 6, 6), (0.35, 0.35, 0.35)
    rng = np.random.default_rng(2)
    v = 0.5 * rng.standard_normal(dims)
    psi0 = rng.standard_normal(dims + (2,)) + 1j * rng.standard_normal(dims + (2,))
    f = np.array([[2.0, 1.0]])
    T = 0.4
    drifts = []
    for dt in (0.04, 0.02):
        cfg = cfg_of(*dims, h=h, norb=2, dt=dt)
        p = psi0.copy()
        E0 = ref.energy(cfg, p, f, v, np.zeros(3))[0, 3]
        d = 0.0
        for _ in range(int(round(T / dt))):
            ref.step(cfg, p, None, None, v, np.zeros(3), 1)
            d = max(d, abs(ref.energy(cfg, p, f, v, np.zeros(3))[0, 3] - E0))
        drifts.append(d)
    assert 3.3 < drifts[0] / drifts[1] < 4.7, drifts


def test_remap_onto_grid_basis_is_density():
    """ref = the grid basis e_r / sqrt(dV): sum_s f_s |<e_r|psi_s>|^2 = rho_r dV."""
    rng = np.random.default_rng(3)
    dims = (4, 2, 4)
    cfg = cfg_of(*dims, norb=3)
    psi = rng.standard_normal(dims + (3,)) + 1j * rng.standard_normal(dims + (3,))
    f = np.array([[2.0, 0.5, 1.0]])
    grid = np.ascontiguousarray((np.eye(32) / np.sqrt(cfg.dV)).reshape(dims + (32,)).astype(np.complex128))
    occ = ref.remap_occ(cfg, psi, f, grid)
    rho, _, _ = ref.density_current(cfg, psi, f, np.zeros(3), want_j=False)
    assert np.abs(occ[0] - rho[0] * cfg.dV).max() < 1e-13 * np.abs(rho).max()


@pytest.mark.parametrize("seed", [4, 5])
def test_remap_on_initial_basis_returns_occupations(seed):
    """At t = 0 with ref = [Psi(0) | B] (orthonormal): the occupied columns get back f, B gets 0;
    after propagation the total over a complete orthonormal basis stays sum_s f_s."""
    from lfd_workloads import make_inputs, workload
    w = workload("P0").with_(nx=4, ny=4, nz=4, norb=3, nocc=3, nproj=61)
    x = make_inputs(w, seed=seed)
    cfg = ref.RefConfig(1, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    basis = np.ascontiguousarray(np.concatenate([x.psi0, x.proj], axis=-1))
    occ = ref.remap_occ(cfg, x.psi0, x.occ, basis)
    assert np.abs(occ[0, :3] - x.occ[0]).max() < 1e-12 and np.abs(occ[0, 3:]).max() < 1e-12
    p = x.psi0.copy()
    ref.step(cfg, p, x.proj, x.dnl, x.vloc, np.array([[0.0, 0.0, 5.0]]), 5)
    occ = ref.remap_occ(cfg, p, x.occ, basis)
    assert abs(occ.sum() - x.occ.sum()) < 1e-11
    assert occ[0, 3:].sum() > 0  # light and scissor excite into the unoccupied block


# --- exactly unitary nonlocal factor -------------------------------------

def _onb(rng, ng, k, dV):
    z = rng.standard_normal((ng, k)) + 1j * rng.standard_normal((ng, k))
    q, _ = np.linalg.qr(z)
    return q / np.sqrt(dV)


def test_exact_nl_equals_dense_matrix_exponential():
    """N_exact = expm(-i (dt/2) B diag(D) B^H dV) (scipy dense matrix exponential on a tiny grid),
    for dV-orthonormal B and distinct D_u of both signs; any psi (not only span(B))."""
    from scipy.linalg import expm
    rng = np.random.default_rng(31)
    dims = (4, 4, 2)
    ng = 32
    cfg = ref.RefConfig(1, *dims, 0.4, 0.5, 0.6, 0, 3, 4, 0.37)
    dV = cfg.dV
    B = _onb(rng, ng, 4, dV)
    Dn = np.array([0.9, -1.7, 0.35, 2.2])
    psi = rng.standard_normal((ng, 3)) + 1j * rng.standard_normal((ng, 3))
    H = (B * Dn) @ B.conj().T * dV
    want = expm(-1j * 0.5 * cfg.dt * H) @ psi
    out = np.ascontiguousarray(psi.reshape(dims + (3,)))
    ref.nl_half_exact(cfg, out, np.ascontiguousarray(B.reshape(dims + (4,))), Dn)
    assert np.abs(out.reshape(ng, 3) - want).max() < 1e-13 * np.abs(want).max()


def test_exact_nl_projector_columns_and_complement():
    """psi = B_u gets exactly e^{-i (dt/2) D_u} B_u; the part orthogonal to span(B) is unchanged."""
    rng = np.random.default_rng(32)
    dims = (4, 2, 4)
    ng = 32
    cfg = ref.RefConfig(1, *dims, 0.3, 0.3, 0.3, 0, 3, 3, 0.8)
    Q = _onb(rng, ng, 6, cfg.dV)
    B = Q[:, :3]
    Dn = np.array([0.5, -2.0, 1.25])
    cols = [2, 0, 1]
    psi = np.ascontiguousarray(B[:, cols].reshape(dims + (3,)))
    out = psi.copy()
    ref.nl_half_exact(cfg, out, np.ascontiguousarray(B.reshape(dims + (3,))), Dn)
    assert np.abs(out - psi * np.exp(-0.5j * cfg.dt * Dn[cols])).max() < 1e-14
    perp = np.ascontiguousarray(Q[:, 3:].reshape(dims + (3,)))
    out = perp.copy()
    ref.nl_half_exact(cfg, out, np.ascontiguousarray(B.reshape(dims + (3,))), Dn)
    assert np.abs(out - perp).max() < 1e-14


def test_exact_step_conserves_orthonormality_with_scissor():
    """With the exact factor the whole step is unitary, so dV Psi^H Psi = I is kept for D != 0
    (the first-order factor of Eq. 6 drifts at O(eps^2) there)."""
    from lfd_workloads import make_inputs, workload
    from lfd_workloads.generate import midpoint_A
    w = workload("P0")
    x = make_inputs(w, seed=33)
    cfg = ref.RefConfig(w.ndom, w.nx, w.ny, w.nz, w.hx, w.hy, w.hz, w.bc, w.norb, w.nproj, w.dt)
    p = x.psi0.copy()
    q = x.psi0.copy()
    for n in range(60):
        A = midpoint_A(w, n)
        ref.step_exact(cfg, p, x.proj, x.dnl * 20.0, x.vloc, A, 1)
        ref.step(cfg, q, x.proj, x.dnl * 20.0, x.vloc, A, 1)
    P = p.reshape(-1, w.norb)
    Q = q.reshape(-1, w.norb)
    S_exact = w.dV * P.conj().T @ P
    S_first = w.dV * Q.conj().T @ Q
    assert np.abs(S_exact - np.eye(w.norb)).max() < 1e-12
    # the two factors agree to O(eps^2) per step, and the first-order one loses orthonormality
    assert np.abs(S_first - np.eye(w.norb)).max() > 1e-8
    assert np.linalg.norm(p - q) / np.linalg.norm(p) < 1e-2
