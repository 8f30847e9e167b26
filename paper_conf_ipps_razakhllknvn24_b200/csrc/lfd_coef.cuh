// lfd_coef.cuh -- per-domain stencil / current coefficients from the vector potential (step a1).
// Shared by k_coef (kin.cu, A captured by value) and the self-consistent step (sc.cu, A on the device).
#pragma once
#include "lfd_complex.cuh"
#include "lfd_internal.h"

namespace lfd {

// For axis d and tau in {Delta/2 (q=0), Delta (q=1)}: t_d = 1/(2 h_d^2), theta_d = (A_d/c) h_d,
// alpha = e^{-i tau t} cos(tau t), sigma = i e^{-i tau t} sin(tau t), up/dn = sigma e^{+-i theta}.
__device__ inline DomCoef make_coef(const double A[3], double hx, double hy, double hz, double dt) {
  const double h[3] = {hx, hy, hz};
  DomCoef c;
  for (int d = 0; d < 3; ++d) {
    double t = 1.0 / (2.0 * h[d] * h[d]);
    double theta = (A[d] / kCLight) * h[d];
    double st, ct;
    sincos(theta, &st, &ct);
    c.eth[d] = make_double2(ct, st);
    c.inv_h[d] = 1.0 / h[d];
    for (int q = 0; q < 2; ++q) {
      double tau = (q == 0) ? 0.5 * dt : dt;
      double sp, cp;
      sincos(tau * t, &sp, &cp);
      double2 ph = make_double2(cp, -sp);                  // e^{-i tau t}
      double2 sigma = make_double2(sp * sp, sp * cp);      // i e^{-i tau t} sin(tau t)
      c.alpha[d][q] = make_double2(cp * cp, -sp * cp);     // e^{-i tau t} cos(tau t)
      c.up[d][q] = cmul(sigma, make_double2(ct, st));      // sigma e^{+i theta}
      c.dn[d][q] = cmul(sigma, make_double2(ct, -st));     // sigma e^{-i theta}
      c.onsite[d][q] = ph;
      const double tn = sp / cp;                           // scaled form: w = i tan(tau t) e^{+-i theta}
      c.wu[d][q] = make_double2(-tn * st, tn * ct);
      c.wd[d][q] = make_double2(tn * st, tn * ct);
      c.rc[d][q] = 1.0 / cp;                               // zero-BC singleton, relative to c
    }
  }
  c.pad_ = 0.0;
  return c;
}

}  // namespace lfd
