"""Host logic of the dense-D path (no GPU): the library's Hermitian eigensolver (csrc/herm_eig.h, used once
at lfd_init to rotate the projectors, D = Q diag(w) Q^H) compiled with g++ and checked against LAPACK
(numpy.linalg.eigh): eigenvalues, A Q = Q diag(w), Q unitary -- real, complex, degenerate and 1x1 cases."""
import os
import subprocess
import tempfile

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HDR = os.path.join(ROOT, "paper_conf_ipps_razakhllknvn24_b200", "csrc")

SRC = r'''
#include "herm_eig.h"
#include <cstdio>
int main() {
  int n;
  if (scanf("%d", &n) != 1) return 1;
  std::vector<std::complex<double>> A((size_t)n * n), Q((size_t)n * n);
  std::vector<double> w(n);
  for (auto& a : A) { double re, im; if (scanf("%lf %lf", &re, &im) != 2) return 1; a = {re, im}; }
  int sw = lfd::herm_eig(n, A.data(), w.data(), Q.data());
  printf("%d\n", sw);
  for (int i = 0; i < n; ++i) printf("%.17g\n", w[i]);
  for (auto& q : Q) printf("%.17g %.17g\n", q.real(), q.imag());
  return 0;
}
'''


@pytest.fixture(scope="module")
def exe():
    d = tempfile.mkdtemp()
    src = os.path.join(d, "eig.cpp")
    out = os.path.join(d, "eig")
    open(src, "w").write(SRC)
    subprocess.run(["g++", "-O2", "-std=c++17", "-I", HDR, "-o", out, src], check=True)
    return out


def _run(exe, A):
    n = A.shape[0]
    inp = f"{n}\n" + "\n".join(f"{float(z.real)!r} {float(z.imag)!r}" for z in A.reshape(-1)) + "\n"
    r = subprocess.run([exe], input=inp, capture_output=True, text=True, check=True)
    v = r.stdout.split()
    sw = int(v[0])
    w = np.array([float(x) for x in v[1:1 + n]])
    q = np.array([float(x) for x in v[1 + n:]]).reshape(-1, 2)
    return sw, w, (q[:, 0] + 1j * q[:, 1]).reshape(n, n)


@pytest.mark.parametrize("kind,n", [("complex", 6), ("complex", 33), ("real", 17), ("degenerate", 12), ("one", 1),
                                    ("diag", 5)])
def test_herm_eig_against_lapack(exe, kind, n):
    rng = np.random.default_rng(n)
    if kind == "real":
        M = rng.standard_normal((n, n))
        A = (M + M.T).astype(np.complex128)
    elif kind == "degenerate":  # repeated eigenvalues (a scissor-like D plus a rank-2 perturbation)
        Q0, _ = np.linalg.qr(rng.standard_normal((n, n)) + 1j * rng.standard_normal((n, n)))
        d = np.full(n, 0.07)
        d[:2] = (0.5, -0.3)
        A = Q0 @ np.diag(d) @ Q0.conj().T
    elif kind == "diag":
        A = np.diag(rng.standard_normal(n)).astype(np.complex128)
    else:
        M = rng.standard_normal((n, n)) + 1j * rng.standard_normal((n, n))
        A = M + M.conj().T
    sw, w, Q = _run(exe, A)
    assert sw >= 0
    wl = np.linalg.eigvalsh(A)
    scale = max(1.0, np.abs(wl).max())
    assert np.abs(np.sort(w) - wl).max() < 1e-13 * scale
    assert np.abs(A @ Q - Q * w[None, :]).max() < 1e-12 * scale
    assert np.abs(Q.conj().T @ Q - np.eye(n)).max() < 1e-13
