"""Dense-matrix helpers for the oracle pins (tests only; independent of oracle/ and the CUDA path).

They build the textbook objects the paper's method must reproduce:
  * the 3-point finite-difference Peierls operator of (1/2)(-i d/dx + a)^2 (Eq. 2/5),
  * the Hermitian generator of each link set (reading R4/R5), as an explicit matrix,
and then use scipy.linalg.expm (a library matrix exponential) as the ground truth.
"""
from __future__ import annotations

import numpy as np
from scipy.linalg import expm

PERIODIC, ZERO = 0, 1


def fd_peierls_1d(n: int, h: float, a: float, bc: int) -> np.ndarray:
    """T = (1/h^2) I - (1/(2h^2)) (e^{i a h} S + e^{-i a h} S^dagger), (S psi)_i = psi_{i+1}.

    Zero BC drops the wrap hopping but keeps the 1/h^2 diagonal (Dirichlet FD)."""
    T = np.eye(n, dtype=np.complex128) / h**2
    for i in range(n):
        j = i + 1
        if j == n:
            if bc == ZERO:
                continue
            j = 0
        T[i, j] += -np.exp(1j * a * h) / (2 * h**2)
        T[j, i] += -np.exp(-1j * a * h) / (2 * h**2)
    return T


def link_set_hamiltonian(n: int, h: float, a: float, bc: int, parity: int) -> np.ndarray:
    """Generator of one link set: E (parity 0) = links (2m, 2m+1); O (parity 1) = (2m+1, 2m+2) plus
    the periodic wrap (n-1, 0). Each link carries t[[1, -e^{i a h}], [-e^{-i a h}, 1]], t = 1/(2h^2);
    a point left without a link in this set carries t on the diagonal."""
    t = 1.0 / (2 * h * h)
    H = np.zeros((n, n), dtype=np.complex128)
    covered = np.zeros(n, dtype=bool)
    links = []
    start = 0 if parity == 0 else 1
    for i in range(start, n - 1, 2):
        links.append((i, i + 1))
    if parity == 1 and bc == PERIODIC:
        links.append((n - 1, 0))
    for i, j in links:
        H[i, i] += t
        H[j, j] += t
        H[i, j] += -t * np.exp(1j * a * h)
        H[j, i] += -t * np.exp(-1j * a * h)
        covered[i] = covered[j] = True
    for i in range(n):
        if not covered[i]:
            H[i, i] += t
    return H


def axis_op(M: np.ndarray, axis: int, dims: tuple) -> np.ndarray:
    """Embed a 1-D operator along `axis` of a (nx, ny, nz) grid flattened as ((ix*ny)+iy)*nz+iz."""
    mats = [np.eye(d, dtype=np.complex128) for d in dims]
    mats[axis] = M
    return np.kron(np.kron(mats[0], mats[1]), mats[2])


def split_kinetic_dense(n, h, a, bc, tau):
    """Dense K_d(tau) = e^{-i tau/2 H_E} e^{-i tau H_O} e^{-i tau/2 H_E} (E acts first)."""
    HE = link_set_hamiltonian(n, h, a, bc, 0)
    HO = link_set_hamiltonian(n, h, a, bc, 1)
    eE = expm(-0.5j * tau * HE)
    return eE @ expm(-1j * tau * HO) @ eE
