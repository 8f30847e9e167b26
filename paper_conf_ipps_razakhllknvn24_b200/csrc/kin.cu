// kin.cu -- local propagator kernels for sm_100a.
//
// Paper: Eq. 6 local factor exp(-i Delta h_loc) by the O(N) space-splitting stencil (P:68,
// P:76-80). Alg. 3-5 stream each line along the stencil axis with one thread team per
// (other two coordinates, orbital block) and carry the pre-update neighbour (psi_old) so the update is
// in place. Here: one thread per (domain, other two coordinates, orbital) column; it streams its line
// in pair-aligned steps, keeping the pre-update values it still needs in registers (the psi_old carry
// of Alg. 3 l.6), so each pass reads and writes Psi exactly once. Consecutive threads own
// consecutive orbitals (the paper's orbital-innermost SoA), so every load/store of a warp is a
// contiguous 512-byte segment.
//
// K_d = E_d(Delta/2) O_d(Delta) E_d(Delta/2) (readings R4/R5): E links (2m,2m+1), O links (2m+1,2m+2)
// plus the periodic wrap (n-1,0); zero BC turns missing links into the on-site factor e^{-i tau t_d}.
#include "lfd_complex.cuh"
#include "lfd_internal.h"

namespace lfd {

__global__ void k_coef(CoefParams p, int dom0, int count, double hx, double hy, double hz, double dt,
                       DomCoef* __restrict__ coef) {
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= count) return;
  const double h[3] = {hx, hy, hz};
  DomCoef c;
  for (int d = 0; d < 3; ++d) {
    double t = 1.0 / (2.0 * h[d] * h[d]);
    double theta = (p.A[i][d] / kCLight) * h[d];
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
    }
  }
  c.pad_ = 0.0;
  coef[dom0 + i] = c;
}

cudaError_t launch_coef(const Geometry& g, const CoefParams& p, int dom0, int count, DomCoef* coef,
                        cudaStream_t st) {
  k_coef<<<(count + 127) / 128, 128, 0, st>>>(p, dom0, count, g.hx, g.hy, g.hz, g.dt, coef);
  return cudaGetLastError();
}

// Phi(r) = e^{-i (Delta/2) v_loc(r)}  (Strang placement of the potential, reading R7).
// The kernel also keeps a copy of v_loc for lfd_energy (vcopy may alias v: then it is not written).
__global__ void k_phase(const double* __restrict__ v, double2* __restrict__ phi, double* vcopy, long long n,
                        double half_dt) {
  long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const double vi = v[i];
  double s, c;
  sincos(half_dt * vi, &s, &c);
  phi[i] = make_double2(c, -s);
  if (vcopy != v) vcopy[i] = vi;
}

cudaError_t launch_phase(const Geometry& g, const double* v, double2* phi, double* vcopy, cudaStream_t st) {
  long long n = g.ng * g.ndom;
  k_phase<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(v, phi, vcopy, n, 0.5 * g.dt);
  return cudaGetLastError();
}

// One K_axis pass. Column c of domain blockIdx.y: outer = c / inner_len, inner = c % inner_len,
// element offset = outer*outer_stride + inner; successive points of the line are pt_stride apart.
template <bool kPeriodic, int kPhase>
__global__ void __launch_bounds__(256, 3) k_kin(double2* __restrict__ psi, const DomCoef* __restrict__ coef,
                                             const double2* __restrict__ phi, int axis, int n, int pt_stride,
                                             int inner_len, int outer_stride, int ncols, int norb,
                                             long long dom_stride, long long ng) {
  int c = blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= ncols) return;
  const int dom = blockIdx.y;
  const int outer = c / inner_len;
  const int inner = c - outer * inner_len;
  const int off = outer * outer_stride + inner;
  double2* line = psi + dom * dom_stride + off;
  const double2* ph = phi + dom * ng + off / norb;
  const int ph_stride = pt_stride / norb;

  const DomCoef* cf = coef + dom;
  const double2 a1 = cf->alpha[axis][0], u1 = cf->up[axis][0], d1 = cf->dn[axis][0], s1 = cf->onsite[axis][0];
  const double2 a2 = cf->alpha[axis][1], u2 = cf->up[axis][1], d2 = cf->dn[axis][1], s2 = cf->onsite[axis][1];

  auto ld = [&](int i) -> double2 {
    double2 v = line[(long long)i * pt_stride];
    if (kPhase == 1) v = cmul(ph[(long long)i * ph_stride], v);
    return v;
  };
  auto st = [&](int i, double2 v) {
    if (kPhase == 2) v = cmul(ph[(long long)i * ph_stride], v);
    line[(long long)i * pt_stride] = v;
  };

  const int P = (n + 1) >> 1;
  double2 E10 = cz(), O1 = cz(), prev_e1 = cz(), prev_oR = cz();
  // two pairs in flight ahead of the one being combined (memory-level parallelism for the HBM stream)
  double2 na = ld(0), nb = (n > 1) ? ld(1) : cz();
  double2 nc = cz(), nd = cz();
  if (P > 1) {
    nc = ld(2);
    nd = (3 < n) ? ld(3) : cz();
  }
  for (int p = 0; p < P; ++p) {
    const double2 a = na, b = nb;
    const bool pair = (2 * p + 1 < n);
    na = nc;
    nb = nd;
    if (p + 2 < P) {
      nc = ld(2 * p + 4);
      nd = (2 * p + 5 < n) ? ld(2 * p + 5) : cz();
    }
    double2 e0, e1 = cz();
    if (pair) {
      e0 = crow(a1, a, u1, b);  // first E(Delta/2) on link (2p, 2p+1)
      e1 = crow(d1, a, a1, b);
    } else {
      e0 = cmul(s1, a);  // zero-BC singleton (odd n)
    }
    if (p == 0) {
      E10 = e0;
    } else {
      const double2 oL = crow(a2, prev_e1, u2, e0);  // O(Delta) on link (2p-1, 2p)
      const double2 oR = crow(d2, prev_e1, a2, e0);
      if (p == 1) {
        O1 = oL;
      } else {  // second E(Delta/2) on link (2p-2, 2p-1): both O outputs are now known
        st(2 * p - 2, crow(a1, prev_oR, u1, oL));
        st(2 * p - 1, crow(d1, prev_oR, a1, oL));
      }
      prev_oR = oR;
    }
    prev_e1 = e1;
  }
  if ((n & 1) == 0) {
    double2 Olast, O0;
    if (kPeriodic) {  // wrap link (n-1, 0)
      Olast = crow(a2, prev_e1, u2, E10);
      O0 = crow(d2, prev_e1, a2, E10);
    } else {
      Olast = cmul(s2, prev_e1);
      O0 = cmul(s2, E10);
    }
    if (n == 2) {
      st(0, crow(a1, O0, u1, Olast));
      st(1, crow(d1, O0, a1, Olast));
    } else {
      st(n - 2, crow(a1, prev_oR, u1, Olast));
      st(n - 1, crow(d1, prev_oR, a1, Olast));
      st(0, crow(a1, O0, u1, O1));
      st(1, crow(d1, O0, a1, O1));
    }
  } else {  // odd n (zero BC): last point is an E singleton; point 0 an O singleton
    st(n - 1, cmul(s1, prev_oR));
    const double2 O0 = cmul(s2, E10);
    st(0, crow(a1, O0, u1, O1));
    st(1, crow(d1, O0, a1, O1));
  }
}

cudaError_t launch_kin(const Geometry& g, double2* psi, const DomCoef* coef, const double2* phi, int axis,
                       int phase_mode, cudaStream_t st) {
  const int nd[3] = {g.nx, g.ny, g.nz};
  const int norb = g.norb;
  int pt_stride, inner_len, outer_stride;
  if (axis == 0) {
    pt_stride = g.ny * g.nz * norb;
    inner_len = g.ny * g.nz * norb;
    outer_stride = 0;
  } else if (axis == 1) {
    pt_stride = g.nz * norb;
    inner_len = g.nz * norb;
    outer_stride = g.ny * g.nz * norb;
  } else {
    pt_stride = norb;
    inner_len = norb;
    outer_stride = g.nz * norb;
  }
  const int n = nd[axis];
  const int ncols = (int)(g.ng / n) * norb;
  dim3 grid((ncols + 255) / 256, g.ndom);
  const long long dom_stride = g.ng * norb;
  const bool per = (g.bc == 0);
#define LFD_KIN(P, M)                                                                                    \
  k_kin<P, M><<<grid, 256, 0, st>>>(psi, coef, phi, axis, n, pt_stride, inner_len, outer_stride, ncols, \
                                    norb, dom_stride, g.ng)
  if (per) {
    if (phase_mode == 1) LFD_KIN(true, 1); else if (phase_mode == 2) LFD_KIN(true, 2); else LFD_KIN(true, 0);
  } else {
    if (phase_mode == 1) LFD_KIN(false, 1); else if (phase_mode == 2) LFD_KIN(false, 2); else LFD_KIN(false, 0);
  }
#undef LFD_KIN
  return cudaGetLastError();
}

}  // namespace lfd
