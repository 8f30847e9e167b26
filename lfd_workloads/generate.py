"""Seeded synthetic inputs (recipe restated in DESIGN.md §5).

NumPy ``PCG64(seed)``; everything is generated on the host once, so the oracle and the GPU path see
identical bytes. Nothing here is the method's arithmetic: it builds v_loc, orthonormal initial KS
orbitals Psi(0), the unoccupied-orbital projector block B, occupations f, couplings D and the laser
vector potential A(t).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from .configs import DELTA_SCI, Workload

C_LIGHT = 137.035999084
OMEGA = 0.057  # 800 nm [a.u.]

# PbTiO3 sites in fractional coordinates of the tetragonal cell, with the Gaussian depth Z [Ha]
# (SURVEY §8(d)).
SITES = (
    ((0.0, 0.0, 0.0), 3.0),   # Pb
    ((0.5, 0.5, 0.54), 4.0),  # Ti
    ((0.5, 0.5, 0.11), 2.0),  # O
    ((0.5, 0.0, 0.62), 2.0),  # O
    ((0.0, 0.5, 0.62), 2.0),  # O
)
SIGMA = 0.6  # bohr


@dataclass
class Inputs:
    psi0: np.ndarray            # [ndom, nx, ny, nz, norb] complex128
    proj: np.ndarray | None     # [ndom, nx, ny, nz, nproj] complex128 (None iff nproj == 0)
    dnl: np.ndarray             # [ndom, nproj] float64
    occ: np.ndarray             # [ndom, norb] float64
    vloc: np.ndarray            # [ndom, nx, ny, nz] float64


def _vloc_domain(w: Workload) -> np.ndarray:
    """Sum of periodic Gaussian wells at the PbTiO3 sites of every cell the domain spans."""
    L = np.array([w.nx * w.hx, w.ny * w.hy, w.nz * w.hz])
    cell = L / np.array(w.cells)
    x = np.arange(w.nx) * w.hx
    y = np.arange(w.ny) * w.hy
    z = np.arange(w.nz) * w.hz
    X, Y, Z = np.meshgrid(x, y, z, indexing="ij")
    v = np.zeros((w.nx, w.ny, w.nz))
    for cx in range(w.cells[0]):
        for cy in range(w.cells[1]):
            for cz in range(w.cells[2]):
                for frac, zval in SITES:
                    R = (np.array([cx, cy, cz]) + np.array(frac)) * cell
                    d2 = np.zeros_like(X)
                    for comp, G, Lc in ((0, X, L[0]), (1, Y, L[1]), (2, Z, L[2])):
                        dd = G - R[comp]
                        dd -= Lc * np.round(dd / Lc)  # minimum image (sigma << L)
                        d2 += dd * dd
                    v -= zval * np.exp(-d2 / (2 * SIGMA**2))
    return v


def _mgs(X: np.ndarray, dV: float) -> np.ndarray:
    """Modified Gram-Schmidt, twice, in the dV-weighted inner product <a|b> = dV sum conj(a) b."""
    X = X.copy()
    for _ in range(2):
        for k in range(X.shape[1]):
            for q in range(k):
                X[:, k] -= (dV * np.vdot(X[:, q], X[:, k])) * X[:, q]
            X[:, k] /= np.sqrt(dV * np.vdot(X[:, k], X[:, k]).real)
    return X


def _haar(rng: np.random.Generator, n: int) -> np.ndarray:
    z = (rng.standard_normal((n, n)) + 1j * rng.standard_normal((n, n))) / np.sqrt(2)
    q, r = np.linalg.qr(z)
    d = np.diagonal(r)
    return q * (d / np.abs(d))


def _planewaves(w: Workload, count: int) -> np.ndarray:
    """count distinct lattice plane waves e^{i k.r}/sqrt(V), lowest |k| first; [ngrid, count]."""
    L = np.array([w.nx * w.hx, w.ny * w.hy, w.nz * w.hz])
    V = L.prod()
    m = 1
    while (2 * m + 1) ** 3 < count:
        m += 1
    ns = [(a, b, c) for a in range(-m, m + 1) for b in range(-m, m + 1) for c in range(-m, m + 1)]
    ks = sorted(ns, key=lambda n: (sum(((2 * np.pi * n[i] / L[i]) ** 2) for i in range(3)), n))[:count]
    out = np.empty((w.ngrid, count), dtype=np.complex128)
    x = np.arange(w.nx) * w.hx
    y = np.arange(w.ny) * w.hy
    z = np.arange(w.nz) * w.hz
    for j, n in enumerate(ks):
        k = 2 * np.pi * np.array(n) / L
        ex, ey, ez = np.exp(1j * k[0] * x), np.exp(1j * k[1] * y), np.exp(1j * k[2] * z)
        out[:, j] = (ex[:, None, None] * ey[None, :, None] * ez[None, None, :]).reshape(-1) / np.sqrt(V)
    return out


def make_inputs(w: Workload, seed: int = 1) -> Inputs:
    rng = np.random.Generator(np.random.PCG64(seed))
    ng, no, npj = w.ngrid, w.norb, w.nproj
    psi0 = np.empty((w.ndom, w.nx, w.ny, w.nz, no), dtype=np.complex128)
    proj = np.empty((w.ndom, w.nx, w.ny, w.nz, npj), dtype=np.complex128) if npj > 0 else None
    vbase = _vloc_domain(w)
    vloc = np.empty((w.ndom, w.nx, w.ny, w.nz))
    for dm in range(w.ndom):
        if w.basis == "gauss":
            X = rng.standard_normal((ng, no + npj)) + 1j * rng.standard_normal((ng, no + npj))
            Q = _mgs(X, w.dV)
            W1, W2 = Q[:, :no], Q[:, no:]
        else:
            W = _planewaves(w, no + npj)
            W1 = W[:, :no] @ _haar(rng, no)
            W2 = W[:, no:] @ _haar(rng, npj) if npj > 0 else None
        psi0[dm] = W1.reshape(w.nx, w.ny, w.nz, no)
        if npj > 0:
            proj[dm] = W2.reshape(w.nx, w.ny, w.nz, npj)
        v = vbase.copy()
        if w.vnoise:
            v += w.vnoise * (rng.random(v.shape) - 0.5)
        vloc[dm] = v + 0.01 * dm
    occ = np.zeros((w.ndom, no))
    occ[:, : w.nocc] = 2.0
    dnl = np.full((w.ndom, npj), DELTA_SCI)
    return Inputs(psi0=psi0, proj=proj, dnl=dnl, occ=occ, vloc=vloc)


def laser_A(w: Workload, t: float) -> np.ndarray:
    """A(t) [ndom, 3] in a.u.: A0 sin(omega t + pi/3) along w.pol, A0 = c E0 / omega.

    Callers evaluate it at the step midpoint t_n + Delta/2 (Eq. 4). Zero when w.laser is off.
    """
    A = np.zeros((w.ndom, 3))
    if not w.laser:
        return A
    a0 = C_LIGHT * w.e0 / OMEGA
    amp = a0 * np.sin(OMEGA * t + np.pi / 3)
    pol = np.asarray(w.pol, dtype=np.float64)
    pol = pol / np.linalg.norm(pol)
    for dm in range(w.ndom):
        A[dm] = amp * pol * (1.0 + w.a_spread * dm)
    return A


def midpoint_A(w: Workload, n: int) -> np.ndarray:
    """A at the midpoint of step n: t = (n + 1/2) Delta."""
    return laser_A(w, (n + 0.5) * w.dt)
