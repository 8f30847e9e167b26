// herm_eig.h -- host-side eigendecomposition of a small complex Hermitian matrix (cyclic Jacobi with unitary
// 2x2 rotations), used once at lfd_init for a dense nonlocal coupling D (LFD_FLAG_DENSE_D): D = Q diag(w) Q^H,
// so B D B^H = (B Q) diag(w) (B Q)^H and the step runs the diagonal-D kernels on the rotated projectors B Q.
// Header-only, no CUDA: tests/test_host_eig.py compiles it with g++ and checks it against numpy.linalg.eigh.
#ifndef LFD_HERM_EIG_H_
#define LFD_HERM_EIG_H_

#include <cmath>
#include <complex>
#include <vector>

namespace lfd {

// A: n x n row-major Hermitian (only its Hermitian part is used); w[n] eigenvalues, Q[n x n] row-major with the
// eigenvectors as columns (A Q = Q diag(w), Q unitary). Returns the number of sweeps (< 0: no convergence).
inline int herm_eig(int n, const std::complex<double>* A_in, double* w, std::complex<double>* Q) {
  using cd = std::complex<double>;
  std::vector<cd> A((size_t)n * n);
  for (int i = 0; i < n; ++i)
    for (int j = 0; j < n; ++j) A[(size_t)i * n + j] = 0.5 * (A_in[(size_t)i * n + j] + std::conj(A_in[(size_t)j * n + i]));
  for (int i = 0; i < n; ++i)
    for (int j = 0; j < n; ++j) Q[(size_t)i * n + j] = (i == j) ? 1.0 : 0.0;
  double tot = 0.0;
  for (size_t k = 0; k < (size_t)n * n; ++k) tot += std::norm(A[k]);
  int sweep = 0;
  for (; sweep < 100; ++sweep) {
    double off = 0.0;
    for (int p = 0; p < n; ++p)
      for (int q = p + 1; q < n; ++q) off += std::norm(A[(size_t)p * n + q]);
    if (off <= 1e-32 * tot || off == 0.0) break;
    for (int p = 0; p < n; ++p)
      for (int q = p + 1; q < n; ++q) {
        const cd apq = A[(size_t)p * n + q];
        const double r = std::abs(apq);
        if (r == 0.0) continue;
        const cd ph = apq / r;  // e^{i phi}
        const double app = A[(size_t)p * n + p].real(), aqq = A[(size_t)q * n + q].real();
        // real Jacobi rotation of [[app, r], [r, aqq]] (the phase moved into column / row q)
        const double th = (aqq - app) / (2.0 * r);
        const double t = (th >= 0 ? 1.0 : -1.0) / (std::fabs(th) + std::sqrt(th * th + 1.0));
        const double c = 1.0 / std::sqrt(t * t + 1.0), s = t * c;
        const cd e = std::conj(ph);  // e^{-i phi}
        // U on (p, q): U_pp = c, U_pq = s, U_qp = -s e^{-i phi}, U_qq = c e^{-i phi};  A <- U^H A U, Q <- Q U
        for (int k = 0; k < n; ++k) {  // columns
          const cd xp = A[(size_t)k * n + p], xq = A[(size_t)k * n + q];
          A[(size_t)k * n + p] = c * xp - s * e * xq;
          A[(size_t)k * n + q] = s * xp + c * e * xq;
          const cd vp = Q[(size_t)k * n + p], vq = Q[(size_t)k * n + q];
          Q[(size_t)k * n + p] = c * vp - s * e * vq;
          Q[(size_t)k * n + q] = s * vp + c * e * vq;
        }
        for (int k = 0; k < n; ++k) {  // rows
          const cd yp = A[(size_t)p * n + k], yq = A[(size_t)q * n + k];
          A[(size_t)p * n + k] = c * yp - s * ph * yq;
          A[(size_t)q * n + k] = s * yp + c * ph * yq;
        }
        A[(size_t)p * n + q] = 0.0;
        A[(size_t)q * n + p] = 0.0;
        A[(size_t)p * n + p] = A[(size_t)p * n + p].real();
        A[(size_t)q * n + q] = A[(size_t)q * n + q].real();
      }
  }
  for (int i = 0; i < n; ++i) w[i] = A[(size_t)i * n + i].real();
  return sweep < 100 ? sweep : -1;
}

}  // namespace lfd

#endif  // LFD_HERM_EIG_H_
