"""Pins of the oracle's WHOLE Eq.-6 step with the nonlocal factor ON (no GPU; `-m "not gpu"`).

`lfd_ref_step` composes N o Local o N (Eq. 6: the renormalised first-order nonlocal factor of
Eq. 7 / Eq. 9, P:68 / P:210, on both sides of the space-splitting local propagator, P:68 / P:80). The
per-factor pins live in test_oracle_pins.py; these check the COMPOSITION against things the mathematics
fixes, so that dropping or doubling a nonlocal half, giving it eps = Delta instead of Delta/2, or
moving the renormalisation, fails here:

* closed form in an exact invariant subspace: lattice plane waves with (k + a) h in {0, pi} on every
  axis are eigenvectors of every pair-link sweep (P:80 pair blocks, reading R4) and of a constant v_loc
  phase; taking them as the dV-orthonormal projector columns B_u with DISTINCT D_u, one step maps
  psi = B_u to lambda_u ((1 - i eps D_u)/|1 - i eps D_u|)^2 B_u, and a two-column mix to a 2x2 closed
  form that also fixes where each renormalisation happens;
* convergence to the exact propagator: with dV-orthonormal B the step converges (order 1: the
  renormalisation of the first-order factor leaves an O(eps^2) error per factor, R11) to
  expm(-i T (H_FD + V + B diag(D) B^H dV)) with a dense library matrix exponential, while a
  composition with half / double the nonlocal weight converges to a different operator;
* the exactly unitary variant (`step_exact`) converges at second order (Strang) to the same operator.
"""
from __future__ import annotations

import numpy as np
import pytest
from scipy.linalg import expm

from oracle import ref
from tests import _dense as D

C = ref.C_LIGHT


def _grid(dims, h):
    return np.meshgrid(*(h[i] * np.arange(dims[i]) for i in range(3)), indexing="ij")


def _lattice_eigen_waves(dims, h, a3):
    """The 8 plane waves e^{i k.r}/sqrt(V) with (k_d + a_d) h_d in {0, pi} and k on the lattice
    (requires a_d L_d in 2 pi Z), together with the free-FD kinetic eigenvalue sum_d (1 - cos)/h_d^2."""
    L = np.array(dims) * np.array(h)
    X = _grid(dims, h)
    V = L.prod()
    waves, ekin = [], []
    for bits in range(8):
        kh = np.array([np.pi * ((bits >> d) & 1) for d in range(3)])
        k = kh / np.array(h) - a3
        ph = sum(k[d] * X[d] for d in range(3))
        waves.append(np.exp(1j * ph) / np.sqrt(V))
        ekin.append(np.sum((1 - np.cos(kh)) / np.array(h) ** 2))
    return np.stack(waves, axis=-1), np.array(ekin)


def _step_factor(eps, Du):
    g = 1 - 1j * eps * Du
    return g / np.abs(g)


@pytest.mark.parametrize("gauge", [(0, 0, 0), (1, -1, 2)])
def test_step_closed_form_on_projector_plane_waves(gauge):
    """psi_s = B_u: N gives (1 - i eps D_u)/|.| B_u, Local gives lambda_u B_u with lambda_u =
    e^{-i Delta v0} e^{-i Delta E_u} (E_u the FD eigenvalue: each K_d acts exactly on these waves),
    N again: psi = lambda_u f_u^2 B_u. Distinct D_u catch index mix-ups; f_u vs f_u^2 vs f_u^3
    catches a dropped or doubled half; eps = Delta/2 is fixed by the phase atan(eps D_u)."""
    dims, h = (4, 6, 4), (0.31, 0.27, 0.36)
    dt, v0 = 0.07, -0.43
    L = np.array(dims) * np.array(h)
    a3 = 2 * np.pi * np.array(gauge) / L
    W, ek = _lattice_eigen_waves(dims, h, a3)
    Dn = np.array([0.9, -2.3, 4.1, 1.7, -0.6, 3.3, 2.6, -1.4])
    cfg = ref.RefConfig(1, *dims, *h, ref.BC_PERIODIC, 8, 8, dt)
    B = np.ascontiguousarray(W)
    psi = np.ascontiguousarray(W[..., [5, 0, 3, 7, 1, 6, 2, 4]])
    u = np.array([5, 0, 3, 7, 1, 6, 2, 4])
    out = psi.copy()
    ref.step(cfg, out, B, Dn, np.full(dims, v0), a3 * C, 1)
    lam = np.exp(-1j * dt * v0) * np.exp(-1j * dt * ek[u])
    want = psi * (lam * _step_factor(0.5 * dt, Dn[u]) ** 2)
    assert np.abs(out - want).max() < 1e-13 * np.abs(psi).max()
    # three steps: the factors compose (no hidden state between calls)
    out3 = psi.copy()
    ref.step(cfg, out3, B, Dn, np.full(dims, v0), a3 * C, 3)
    want3 = psi * (lam * _step_factor(0.5 * dt, Dn[u]) ** 2) ** 3
    assert np.abs(out3 - want3).max() < 1e-13 * np.abs(psi).max()


def test_step_closed_form_two_column_mix():
    """psi = (c1 B_u + c2 B_w) with D_u != D_w: the 2-D span is invariant, each half rescales the pair
    (1 - i eps D) componentwise and renormalises the orbital; the local factor multiplies by lambda.
    Closed form written per factor in the paper's order (N first, then Local, then N). The relative
    weight of the two components after one step is g_u^2 lambda_u / (g_w^2 lambda_w), g = 1 - i eps D:
    with eps D ~ 0.3 a single half (g^1), a doubled half (g^3) or eps = Delta (g -> 1 - 2 i eps D)
    are all visibly different."""
    dims, h = (4, 4, 6), (0.3, 0.35, 0.28)
    dt, v0 = 0.2, 0.37
    W, ek = _lattice_eigen_waves(dims, h, np.zeros(3))
    u, w = 3, 6
    Dn = np.zeros(8)
    Dn[u], Dn[w] = 3.0, -1.2
    c = np.array([0.8, 0.6 * np.exp(0.7j)])
    cfg = ref.RefConfig(1, *dims, *h, ref.BC_PERIODIC, 1, 8, dt)
    psi = np.ascontiguousarray((c[0] * W[..., u] + c[1] * W[..., w])[..., None])
    out = psi.copy()
    ref.step(cfg, out, np.ascontiguousarray(W), Dn, np.full(dims, v0), np.zeros(3), 1)
    lam = np.exp(-1j * dt * (v0 + ek[[u, w]]))

    def closed(eps, nhalf):
        g = 1 - 1j * eps * Dn[[u, w]]
        x = c.copy()
        for k in range(nhalf):
            if k == 1:
                x = x * lam
            x = x * g
            x = x * np.linalg.norm(c) / np.linalg.norm(x)
        if nhalf < 2:
            x = x * lam
        return x[0] * W[..., u] + x[1] * W[..., w]

    want = closed(0.5 * dt, 2)
    assert np.abs(out[..., 0] - want).max() < 1e-13 * np.abs(want).max()
    for alt in (closed(0.5 * dt, 1), closed(0.5 * dt, 3), closed(dt, 2)):
        assert np.abs(alt - want).max() > 1e-3 * np.abs(want).max()


def _conv_problem():
    dims, h = (4, 4, 6), (0.3, 0.35, 0.4)
    rng = np.random.default_rng(5)
    a3 = np.array([0.2, -0.5, 0.9])
    v = rng.standard_normal(dims)
    ng = int(np.prod(dims))
    dV = float(np.prod(h))
    q, _ = np.linalg.qr(rng.standard_normal((ng, 7)) + 1j * rng.standard_normal((ng, 7)))
    B = q[:, :4] / np.sqrt(dV)
    Dn = np.array([1.5, -2.0, 0.7, 3.1])
    psi0 = q[:, 4:6] / np.sqrt(dV) + 0.3 * (rng.standard_normal((ng, 2)) + 1j * rng.standard_normal((ng, 2)))
    psi0 = psi0 / np.sqrt(dV * (np.abs(psi0) ** 2).sum(axis=0))
    H = sum(D.axis_op(D.fd_peierls_1d(dims[d], h[d], a3[d], D.PERIODIC), d, dims) for d in range(3))
    H = H + np.diag(v.reshape(-1))
    Vnl = (B * Dn) @ B.conj().T * dV
    return dims, h, a3, v, B, Dn, psi0, H, Vnl


def _run(step, dims, h, a3, v, B, Dn, psi0, dt, T):
    cfg = ref.RefConfig(1, *dims, *h, ref.BC_PERIODIC, 2, 4, dt)
    p = psi0.reshape(dims + (2,)).copy()
    Bg = np.ascontiguousarray(B.reshape(dims + (4,)))
    for _ in range(int(round(T / dt))):
        step(cfg, p, Bg, Dn, v, a3 * C, 1)
    return p.reshape(-1, 2)


def test_step_converges_to_exact_propagator_with_nonlocal():
    """Eq. 6 -> expm(-i T (H_FD + V + v_nl)), v_nl = B diag(D) B^H dV (Eq. 7/9). Order 1 (ratio -> 2 per
    dt halving: the renormalised first-order factor, R11); a composition with half or twice the
    nonlocal weight (one half dropped / doubled, or eps = Delta) stays O(1) away from this operator."""
    dims, h, a3, v, B, Dn, psi0, H, Vnl = _conv_problem()
    T = 0.4
    want = expm(-1j * T * (H + Vnl)) @ psi0
    errs = [np.abs(_run(ref.step, dims, h, a3, v, B, Dn, psi0, dt, T) - want).max()
            for dt in (0.04, 0.02, 0.01, 0.005)]
    ratios = [errs[i] / errs[i + 1] for i in range(3)]
    assert all(1.8 < r < 2.8 for r in ratios), (errs, ratios)
    assert errs[-1] < 1e-3
    # the wrong operators: the correct step is much closer to H + Vnl than to H + Vnl/2 or H + 2 Vnl
    for s in (0.5, 2.0):
        wrong = expm(-1j * T * (H + s * Vnl)) @ psi0
        assert np.abs(_run(ref.step, dims, h, a3, v, B, Dn, psi0, 0.005, T) - wrong).max() > 50 * errs[-1]


def test_step_exact_converges_second_order():
    """The exactly unitary factor exp(-i eps v_nl) around the local propagator is a Strang product:
    global error ratio ~4 per dt halving to the same exact propagator."""
    dims, h, a3, v, B, Dn, psi0, H, Vnl = _conv_problem()
    T = 0.4
    want = expm(-1j * T * (H + Vnl)) @ psi0
    errs = [np.abs(_run(ref.step_exact, dims, h, a3, v, B, Dn, psi0, dt, T) - want).max()
            for dt in (0.04, 0.02, 0.01)]
    assert 3.5 < errs[0] / errs[1] < 4.5 and 3.5 < errs[1] / errs[2] < 4.5, errs


def test_step_first_order_vs_exact_error_constant():
    """The two steps differ only by the renormalised vs exact factor: per step the difference is
    O(eps^2 D^2) (order-2 local error), so over a fixed time T it shrinks ~2x per dt halving."""
    dims, h, a3, v, B, Dn, psi0, H, Vnl = _conv_problem()
    T = 0.4
    d = [np.abs(_run(ref.step, dims, h, a3, v, B, Dn, psi0, dt, T)
                - _run(ref.step_exact, dims, h, a3, v, B, Dn, psi0, dt, T)).max() for dt in (0.02, 0.01)]
    assert 1.7 < d[0] / d[1] < 2.5, d
