"""Pins of the oracle's dense-Hermitian-D nonlocal factor (no GPU).

Eq. 5 puts the nonlocal ionic pseudopotential in v_nl; in Kleinman-Bylander form
v_nl = sum_uv |b_u> D_uv <b_v| with a Hermitian D (Eq. 7's scissor, is D = Delta_sci I). The oracle's
`lfd_ref_*_dense` functions take D as a full matrix. Ground truths here: the independently pinned diagonal
factor (special cases D diagonal, and D = Q diag(d) Q^H with rotated projectors B Q), dense scipy matrix
exponentials of the full Hamiltonian, and the quadratic form <psi|B D B^H dV|psi> with dense matrices.
"""
from __future__ import annotations

import numpy as np
import pytest
from scipy.linalg import expm

from oracle import ref
from tests import _dense as Dd

C = ref.C_LIGHT


def _rand(rng, shape):
    return rng.standard_normal(shape) + 1j * rng.standard_normal(shape)


def _herm(rng, n, scale=1.0):
    M = _rand(rng, (n, n))
    return scale * 0.5 * (M + M.conj().T)


def _setup(seed=3, dims=(4, 4, 6), h=(0.3, 0.35, 0.4), norb=3, nproj=4, orthonormal=True):
    rng = np.random.default_rng(seed)
    ng = int(np.prod(dims))
    dV = float(np.prod(h))
    q, _ = np.linalg.qr(_rand(rng, (ng, norb + nproj)))
    B = q[:, norb:] / np.sqrt(dV) if orthonormal else _rand(rng, (ng, nproj)) * 0.3
    psi = q[:, :norb] / np.sqrt(dV) + 0.4 * _rand(rng, (ng, norb))
    psi = psi / np.sqrt(dV * (np.abs(psi) ** 2).sum(axis=0))
    return rng, dims, h, dV, B, psi


def test_dense_diagonal_equals_diagonal_factor():
    """D = diag(d): the dense factor is the pinned diagonal one (same arithmetic up to rounding order)."""
    rng, dims, h, dV, B, psi = _setup(orthonormal=False)
    d = np.array([0.7, -1.3, 2.1, 0.4])
    cfg = ref.RefConfig(1, *dims, *h, ref.BC_PERIODIC, 3, 4, 0.3)
    a = psi.reshape(dims + (3,)).copy()
    b = a.copy()
    Bg = np.ascontiguousarray(B.reshape(dims + (4,)))
    ref.nl_half(cfg, a, Bg, d)
    ref.nl_half_dense(cfg, b, Bg, np.diag(d).astype(np.complex128))
    assert np.abs(a - b).max() < 1e-14 * np.abs(a).max()


def test_dense_rotation_equals_diagonal_on_rotated_projectors():
    """v_nl = B (Q diag(d) Q^H) B^H dV = (B Q) diag(d) (B Q)^H dV for unitary Q: the dense factor on B equals the
    pinned diagonal factor on B Q (non-orthonormal B, so the renormalisation sees a general Gram matrix)."""
    rng, dims, h, dV, B, psi = _setup(seed=5, orthonormal=False)
    Q, _ = np.linalg.qr(_rand(rng, (4, 4)))
    d = np.array([0.9, -0.4, 1.7, -2.2])
    Dm = Q @ np.diag(d) @ Q.conj().T
    cfg = ref.RefConfig(1, *dims, *h, ref.BC_PERIODIC, 3, 4, 0.5)
    a = psi.reshape(dims + (3,)).copy()
    b = a.copy()
    ref.nl_half_dense(cfg, a, np.ascontiguousarray(B.reshape(dims + (4,))), Dm)
    ref.nl_half(cfg, b, np.ascontiguousarray((B @ Q).reshape(dims + (4,))), d)
    assert np.abs(a - b).max() < 1e-13 * np.abs(a).max()


def test_exact_dense_factor_is_matrix_exponential():
    """exp(-i (Delta/2) B D B^H dV) (dense scipy expm of the ng x ng operator) for orthonormal B, non-diagonal D."""
    rng, dims, h, dV, B, psi = _setup(seed=7)
    Dm = _herm(rng, 4, 1.5)
    dt = 0.6
    cfg = ref.RefConfig(1, *dims, *h, ref.BC_PERIODIC, 3, 4, dt)
    got = psi.reshape(dims + (3,)).copy()
    ref.nl_half_exact_dense(cfg, got, np.ascontiguousarray(B.reshape(dims + (4,))), Dm)
    V = B @ Dm @ B.conj().T * dV
    want = expm(-0.5j * dt * V) @ psi
    assert np.abs(got.reshape(-1, 3) - want).max() < 1e-13 * np.abs(want).max()


def test_dense_norm_kept_and_gram_closed_form():
    """Each orbital keeps its norm; the unrenormalised norm is ||psi||^2 + eps^2 (DC)^H G (DC) (the cross term
    vanishes because C^H D C is real for Hermitian D): checked through the renormalisation factor."""
    rng, dims, h, dV, B, psi = _setup(seed=9, orthonormal=False)
    Dm = _herm(rng, 4, 1.0)
    dt = 0.4
    eps = dt / 2
    cfg = ref.RefConfig(1, *dims, *h, ref.BC_PERIODIC, 3, 4, dt)
    out = psi.reshape(dims + (3,)).copy()
    ref.nl_half_dense(cfg, out, np.ascontiguousarray(B.reshape(dims + (4,))), Dm)
    O = out.reshape(-1, 3)
    assert np.abs(dV * (np.abs(O) ** 2).sum(axis=0) - 1).max() < 1e-13
    Cm = dV * B.conj().T @ psi
    G = dV * B.conj().T @ B
    X = Dm @ Cm
    raw = psi - 1j * eps * B @ X
    n = np.sqrt(1.0 / (1.0 + eps**2 * np.einsum("us,uv,vs->s", X.conj(), G, X).real))
    assert np.abs(O - raw * n).max() < 1e-13 * np.abs(O).max()


def _conv(exact, dts):
    rng, dims, h, dV, B, psi = _setup(seed=11, norb=2, nproj=4)
    Dm = _herm(rng, 4, 2.0)
    v = rng.standard_normal(dims)
    a3 = np.array([0.2, -0.5, 0.9])
    H = sum(Dd.axis_op(Dd.fd_peierls_1d(dims[d], h[d], a3[d], Dd.PERIODIC), d, dims) for d in range(3))
    H = H + np.diag(v.reshape(-1)) + B @ Dm @ B.conj().T * dV
    T = 0.4
    want = expm(-1j * T * H) @ psi
    errs = []
    for dt in dts:
        cfg = ref.RefConfig(1, *dims, *h, ref.BC_PERIODIC, 2, 4, dt)
        p = psi.reshape(dims + (2,)).copy()
        Bg = np.ascontiguousarray(B.reshape(dims + (4,)))
        for _ in range(int(round(T / dt))):
            ref.step_dense(cfg, p, Bg, Dm[None], v, (a3 * C)[None], 1, exact=exact)
        errs.append(np.abs(p.reshape(-1, 2) - want).max())
    return errs


def test_dense_step_converges_first_order():
    errs = _conv(False, (0.04, 0.02, 0.01, 0.005))
    r = [errs[i] / errs[i + 1] for i in range(3)]
    assert all(1.7 < x < 2.8 for x in r) and errs[-1] < 2e-3, (errs, r)


def test_dense_exact_step_converges_second_order():
    errs = _conv(True, (0.04, 0.02, 0.01))
    assert 3.5 < errs[0] / errs[1] < 4.5 and 3.5 < errs[1] / errs[2] < 4.5, errs


def test_dense_nonlocal_energy_quadratic_form():
    rng, dims, h, dV, B, psi = _setup(seed=13, orthonormal=False)
    Dm = _herm(rng, 4, 1.3)
    f = np.array([2.0, 1.0, 0.5])
    cfg = ref.RefConfig(1, *dims, *h, ref.BC_PERIODIC, 3, 4, 0.1)
    got = ref.energy_nl_dense(cfg, psi.reshape(dims + (3,)).copy(), f[None],
                              np.ascontiguousarray(B.reshape(dims + (4,))), Dm[None])
    V = B @ Dm @ B.conj().T * dV
    want = sum(f[s] * dV * np.vdot(psi[:, s], V @ psi[:, s]).real for s in range(3))
    assert abs(got[0] - want) < 1e-13 * abs(want)
