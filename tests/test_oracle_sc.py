"""Pins of the oracle's self-consistent step (oracle/sc.py; readings R23-R28).

Each pin is fixed by something other than the oracle itself: Fourier-mode closed forms of the periodic
Poisson equation, the uniform-gas exchange formula and its functional derivative, the plasma oscillation
of a uniform electron gas against scipy's ODE solver, exact reduction to the plain step, second-order
total-energy conservation, and exact time reversal of the converged step."""
import dataclasses

import numpy as np
import pytest

from lfd_workloads import domain_tiling
from lfd_workloads.generate import _mgs
from oracle import ref, sc

C = ref.C_LIGHT


def grid_coords(dims, h):
    return np.meshgrid(*(h[i] * np.arange(dims[i]) for i in range(3)), indexing="ij")


@pytest.mark.parametrize("m", [(1, 0, 0), (0, -2, 1), (2, 3, -4), (3, 0, 5), (-1, 4, 0)])
def test_hartree_fourier_mode(m):
    """rho = 1 + a cos(G.r + phi) -> v_H = (4 pi a / |G|^2) cos(G.r + phi) exactly (R23); anisotropic
    grid and spacings so a transposed axis or a wrong h fails; (3, 0, 5) is the Nyquist mode of x and z
    (on the grid cos(G.r + phi) = (-1)^(i+k) cos(phi), still of this form)."""
    dims, h = (6, 8, 10), (0.3, 0.25, 0.4)
    L = np.array(dims) * np.array(h)
    G = 2 * np.pi * np.array(m) / L
    X, Y, Z = grid_coords(dims, h)
    ph = G[0] * X + G[1] * Y + G[2] * Z + 0.3
    rho = 1.0 + 0.7 * np.cos(ph)
    v = sc.hartree(rho, h)
    expect = 4 * np.pi * 0.7 / (G @ G) * np.cos(ph)
    assert np.max(np.abs(v - expect)) < 1e-12 * max(1.0, np.abs(expect).max())


def test_hartree_superposition_zero_mean_and_energy_derivative():
    dims, h = (6, 8, 10), (0.3, 0.25, 0.4)
    rng = np.random.default_rng(0)
    r1, r2 = rng.random(dims), rng.random(dims)
    v1, v2 = sc.hartree(r1, h), sc.hartree(r2, h)
    assert np.max(np.abs(sc.hartree(2 * r1 - 3 * r2, h) - (2 * v1 - 3 * v2))) < 1e-12
    assert abs(v1.mean()) < 1e-14 and abs(sc.hartree(r1 + 5.0, h) - v1).max() < 1e-12
    # E_H = (1/2) dV sum rho v_H is positive and v_H is its functional derivative (quadratic: exact)
    dV = np.prod(h)
    E = lambda r: 0.5 * dV * np.sum(r * sc.hartree(r, h))  # noqa: E731
    assert E(r1) > 0
    idx = (2, 5, 7)
    e = np.zeros(dims)
    e[idx] = 1e-3
    dE = (E(r1 + e) - E(r1 - e)) / (2e-3 * dV)
    assert abs(dE - v1[idx]) < 1e-9


def test_exchange_closed_form_and_derivative():
    """Uniform gas: v_x = -(3 rho / pi)^{1/3}; v_x = dE_x/drho (central difference) at every point."""
    for r0 in (1e-3, 0.05, 2.0):
        assert abs(sc.vx_lda(np.array([r0]))[0] + (3 * r0 / np.pi) ** (1 / 3)) < 1e-15
    rng = np.random.default_rng(1)
    rho = 0.01 + rng.random((4, 4, 4))
    dV = 0.02
    for idx in [(0, 0, 0), (1, 2, 3), (3, 3, 1)]:
        e = np.zeros_like(rho)
        e[idx] = 1e-6
        dE = (sc.ex_lda(rho + e, dV) - sc.ex_lda(rho - e, dV)) / (2e-6 * dV)
        assert abs(dE - sc.vx_lda(rho)[idx]) < 1e-7
    assert sc.vx_lda(np.array([-1e-17]))[0] == 0.0


def _plasma(dt, T, adot0=(50.0, -30.0, 20.0)):
    dims, h = (6, 8, 10), (0.3, 0.25, 0.4)
    V = np.prod(dims) * np.prod(h)
    cfg = ref.RefConfig(1, *dims, *h, 0, 1, 0, dt)
    psi = np.full((1, *dims, 1), 1 / np.sqrt(V), complex)
    p = sc.SCProblem(cfg, None, None, np.array([[2.0]]), np.zeros((1, np.prod(dims))),
                     np.zeros((1, 3), int), dims, n_corr=1)
    st = sc.sc_init(p, psi, np.zeros(3), Adot0=adot0)
    n = int(round(T / dt))
    sc.sc_step(p, st, np.zeros((2 * n + 1, 3)), n)
    return st, h, V


def test_maxwell_uniform_gas_plasma_oscillation():
    """k = 0 state of a uniform gas (f = 2): it stays uniform (v_H = 0, v_x constant; exactly for H_E + H_O,
    up to the O(dt^2) splitting error for the E/O sweeps when theta != 0) and its link current
    is J_d = f sin(A_d h_d / c)/(h_d V) exactly, so R25 makes A_ind a pendulum
    A'' = -4 pi c f sin(A h / c)/(h V); small amplitude: omega_p^2 = 4 pi rho. The Verlet result matches
    scipy's high-accuracy ODE solution with O(dt^2) error (R26)."""
    from scipy.integrate import solve_ivp

    T = 2.0
    res = []
    for dt in (0.04, 0.02):
        st, h, V = _plasma(dt, T)
        h = np.array(h)

        def rhs(t, y):
            return np.concatenate([y[3:], -4 * np.pi * C * 2.0 * np.sin(y[:3] * h / C) / (h * V)])

        sol = solve_ivp(rhs, (0, T), [0, 0, 0, 50.0, -30.0, 20.0], rtol=1e-12, atol=1e-12)
        res.append(np.abs(st.A_ind - sol.y[:3, -1]).max())
        assert np.abs(st.Adot - sol.y[3:, -1]).max() < 0.3 * dt**2 * 100
        rho = np.abs(st.psi[0, ..., 0]) ** 2 * 2.0
        assert np.abs(rho - 2.0 / V).max() < 1e-3 * (2.0 / V)  # uniform up to the O(dt^2) splitting error
    assert 3.6 < res[0] / res[1] < 4.4 and res[1] < 1e-3
    # small amplitude: period 2 pi / omega_p with omega_p^2 = 4 pi (f / V)
    st, h, V = _plasma(0.005, 0.0, adot0=(1e-3, 0, 0))
    wp = np.sqrt(4 * np.pi * 2.0 / V)
    quarter = np.pi / (2 * wp)
    st, _, _ = _plasma(quarter / 200, quarter, adot0=(1e-3, 0, 0))
    assert abs(st.Adot[0]) < 1e-3 * 1e-3 and abs(st.A_ind[0] - 1e-3 / wp) < 1e-7


def _small_problem(dt, nproj=0, exact=False, ncorr=1, flags=sc.SC_HARTREE | sc.SC_XC | sc.SC_MAXWELL):
    dims, h, norb = (6, 6, 8), (0.35, 0.3, 0.4), 3
    dV = np.prod(h)
    rng = np.random.default_rng(3)
    X = rng.standard_normal((np.prod(dims), norb + 2)) + 1j * rng.standard_normal((np.prod(dims), norb + 2))
    Q = _mgs(X, dV)
    psi0 = np.ascontiguousarray(Q[:, :norb].reshape(1, *dims, norb))
    B = np.ascontiguousarray(Q[:, norb:].reshape(1, *dims, 2)) if nproj else None
    vion = -0.5 * rng.random((1, np.prod(dims)))
    cfg = ref.RefConfig(1, *dims, *h, 0, norb, nproj, dt)
    p = sc.SCProblem(cfg, B, np.array([[0.3, 0.5]]) if nproj else None, np.array([[2.0, 2.0, 1.0]]), vion,
                     np.zeros((1, 3), int), dims, flags=flags, n_corr=ncorr, exact_nl=exact)
    return p, psi0


def test_sc_without_couplings_is_the_plain_step():
    """flags = 0: v_loc = v_ion and A = A_ext at the midpoints, so sc_step equals ref.step exactly."""
    p, psi0 = _small_problem(0.04, nproj=2, flags=0, ncorr=2)
    n = 4
    Aext = np.outer(np.sin(0.3 + np.arange(2 * n + 1) * 0.02), [30.0, -10.0, 5.0])
    st = sc.sc_init(p, psi0, Aext[0])
    sc.sc_step(p, st, Aext, n)
    psi = psi0.copy()
    v = p.vion.reshape(1, 6, 6, 8).copy()
    for k in range(n):
        ref.step(p.cfg, psi, p.proj, p.dnl, v, Aext[2 * k + 1][None, :], 1)
    assert np.array_equal(psi, st.psi)


def test_sc_energy_conservation_second_order():
    """A_ext = 0, D = 0: E_kin + E_ion + E_H + E_x + E_field is conserved up to O(dt^2) (ratio 4 per
    halving). A sign error in the Hartree or Maxwell coupling, or a wrong exchange prefactor, leaves an
    O(1) drift (checked when this pin was written)."""
    drift = []
    for dt in (0.04, 0.02, 0.01):
        p, psi0 = _small_problem(dt)
        st = sc.sc_init(p, psi0, np.zeros(3), Adot0=(3.0, -2.0, 1.0))
        E0 = sc.total_energy(p, st, np.zeros(3))
        n = int(round(0.8 / dt))
        sc.sc_step(p, st, np.zeros((2 * n + 1, 3)), n)
        E1 = sc.total_energy(p, st, np.zeros(3))
        drift.append(E1["total"] - E0["total"])
        assert abs(E1["field"] - E0["field"]) > 5 * abs(drift[-1])  # energy really flows
    r1, r2 = drift[0] / drift[1], drift[1] / drift[2]
    assert 3.5 < r1 < 4.5 and 3.5 < r2 < 4.5, drift


def test_sc_time_reversal_at_convergence():
    """Converged corrector (implicit midpoint in v, R27) + velocity Verlet (R26) + exactly unitary
    nonlocal factor: running the same steps with -dt and the reversed A_ext returns Psi(0), A_ind(0),
    dA_ind/dt(0) to roundoff; one corrector sweep does not (first-order reversibility defect)."""
    errs = {}
    for ncorr in (1, 8):
        p, psi0 = _small_problem(0.04, nproj=2, exact=True, ncorr=ncorr)
        st = sc.sc_init(p, psi0, np.zeros(3), Adot0=(3.0, -2.0, 1.0))
        n = 5
        Aext = np.outer(np.sin(np.arange(2 * n + 1) * 0.02), [20.0, 0.0, 10.0])
        sc.sc_step(p, st, Aext, n)
        pb = dataclasses.replace(p, cfg=dataclasses.replace(p.cfg, dt=-0.04))
        sc.sc_step(pb, st, Aext[::-1].copy(), n)
        errs[ncorr] = (np.abs(st.psi - psi0).max(), np.abs(st.A_ind).max(),
                       np.abs(st.Adot - [3.0, -2.0, 1.0]).max())
    assert max(errs[8]) < 1e-12, errs
    assert errs[1][0] > 1e-8


def test_domain_tiling_and_assembly():
    offs, gd = domain_tiling(8, (4, 6, 8))
    assert gd == (8, 12, 16)
    cfg = ref.RefConfig(8, 4, 6, 8, 0.3, 0.3, 0.3, 0, 1, 0, 0.04)
    sc.check_tiling(cfg, offs, gd)
    f = np.random.default_rng(0).random((8, 4 * 6 * 8))
    g = sc.assemble(cfg, f, offs, gd)
    assert np.array_equal(sc.restrict(cfg, g, offs), f)
    assert g[4, 6, 8] == f[7, 0] and g[3, 0, 0] == f[0, 3 * 48]
    bad = offs.copy()
    bad[1] = bad[0]
    with pytest.raises(ValueError):
        sc.check_tiling(cfg, bad, gd)
    for nd, expect in ((1, (4, 6, 8)), (2, (8, 6, 8)), (4, (8, 12, 8))):
        assert domain_tiling(nd, (4, 6, 8))[1] == expect
