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
#include "lfd_tma.cuh"

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

// ------------------------------------------------------------------------------------------------
// Fused K_y K_z pass with the post-phase:  Psi <- Phi . K_y K_z Psi  (one HBM read + write of Psi).
// K_y and K_z act on different axes of the tensor grid and commute exactly (reading R6), so the pass
// applies K_z to each (x, y) z-line as it arrives and streams the K_z-transformed lines through the
// pair-aligned y-march of K_y (the psi_old carry of Alg. 3, in registers).
// CTA = (x plane, chunk of kYZW = 8 orbitals, domain); thread (m, o) owns the z pair (2m, 2m+1) of
// orbital o0 + o. Each (x, y) plane segment [nz][8 orbitals] (nz rows of 128 contiguous bytes) arrives
// by TMA bulk copies into an S-deep shared-memory ring; K_z's O(Delta) links cross threads and go
// through a small exchange buffer (double-buffered by pair parity: one __syncthreads per y pair).
// ------------------------------------------------------------------------------------------------
constexpr int kYZW = 8;

struct PairCoef {
  double2 a1, u1, d1, s1, a2, u2, d2, s2;
};

__device__ __forceinline__ PairCoef pair_coef(const DomCoef* cf, int axis) {
  PairCoef c;
  c.a1 = cf->alpha[axis][0]; c.u1 = cf->up[axis][0]; c.d1 = cf->dn[axis][0]; c.s1 = cf->onsite[axis][0];
  c.a2 = cf->alpha[axis][1]; c.u2 = cf->up[axis][1]; c.d2 = cf->dn[axis][1]; c.s2 = cf->onsite[axis][1];
  return c;
}

// Streaming K_d along one line, fed one pair (2p, 2p+1) at a time (same algebra as k_kin's loop).
struct LineMarch {
  double2 E10, O1, prev_e1, prev_oR;
  template <class St>
  __device__ __forceinline__ void push(const PairCoef& c, int p, double2 a, double2 b, bool pair, St&& st) {
    double2 e0, e1 = cz();
    if (pair) {
      e0 = crow(c.a1, a, c.u1, b);
      e1 = crow(c.d1, a, c.a1, b);
    } else {
      e0 = cmul(c.s1, a);
    }
    if (p == 0) {
      E10 = e0;
    } else {
      const double2 oL = crow(c.a2, prev_e1, c.u2, e0);
      const double2 oR = crow(c.d2, prev_e1, c.a2, e0);
      if (p == 1) {
        O1 = oL;
      } else {
        st(2 * p - 2, crow(c.a1, prev_oR, c.u1, oL));
        st(2 * p - 1, crow(c.d1, prev_oR, c.a1, oL));
      }
      prev_oR = oR;
    }
    prev_e1 = e1;
  }
  template <bool kPer, class St>
  __device__ __forceinline__ void finish(const PairCoef& c, int n, St&& st) {
    if ((n & 1) == 0) {
      double2 Olast, O0;
      if (kPer) {
        Olast = crow(c.a2, prev_e1, c.u2, E10);
        O0 = crow(c.d2, prev_e1, c.a2, E10);
      } else {
        Olast = cmul(c.s2, prev_e1);
        O0 = cmul(c.s2, E10);
      }
      if (n == 2) {
        st(0, crow(c.a1, O0, c.u1, Olast));
        st(1, crow(c.d1, O0, c.a1, Olast));
      } else {
        st(n - 2, crow(c.a1, prev_oR, c.u1, Olast));
        st(n - 1, crow(c.d1, prev_oR, c.a1, Olast));
        st(0, crow(c.a1, O0, c.u1, O1));
        st(1, crow(c.d1, O0, c.a1, O1));
      }
    } else {
      st(n - 1, cmul(c.s1, prev_oR));
      const double2 O0 = cmul(c.s2, E10);
      st(0, crow(c.a1, O0, c.u1, O1));
      st(1, crow(c.d1, O0, c.a1, O1));
    }
  }
};

template <bool kPer>
__global__ void __launch_bounds__(512) k_kin_yz(double2* __restrict__ psi, const DomCoef* __restrict__ coef,
                                                 const double2* __restrict__ phi, int nx, int ny, int nz, int norb,
                                                 int nchunks, long long ng, int S) {
  extern __shared__ __align__(128) unsigned char smem[];
  const int seg = nz * kYZW;  // complex elements per plane segment
  double2* ring = reinterpret_cast<double2*>(smem);
  double2* xch = ring + (long long)S * seg;               // [2 pair parities][2 planes][nz][8]
  uint64_t* full = reinterpret_cast<uint64_t*>(xch + 4 * seg);
  const int dom = blockIdx.y;
  const int x = blockIdx.x / nchunks, oc = blockIdx.x - (blockIdx.x / nchunks) * nchunks;
  const int o0 = oc * kYZW, wv = min(kYZW, norb - o0);
  const int tid = threadIdx.x, o = tid % kYZW, m = tid / kYZW;
  const int z0 = 2 * m, z1 = 2 * m + 1;
  const bool has1 = z1 < nz;
  const bool act = o < wv;
  const long long yst = (long long)nz * norb;  // element stride between y planes
  double2* base = psi + (long long)dom * ng * norb + (long long)x * ny * yst + o0;
  const double2* phb = phi + (long long)dom * ng + (long long)x * ny * nz;
  const DomCoef* cf = coef + dom;
  const PairCoef cz_ = pair_coef(cf, 2), cy = pair_coef(cf, 1);

  if (tid == 0) {
    for (int s = 0; s < S; ++s) mbar_init(&full[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  auto issue = [&](int y) {  // warp 0: plane y -> slot y % S
    const int s = y % S;
    const int lane = tid & 31;
    if (lane == 0) mbar_expect_tx(&full[s], (uint32_t)(nz * wv * 16));
    __syncwarp();
    double2* dst = ring + (long long)s * seg;
    const double2* src = base + (long long)y * yst;
    for (int z = lane; z < nz; z += 32) tma_row(dst + z * kYZW, src + (long long)z * norb, (uint32_t)(wv * 16), &full[s]);
  };
  if (tid < 32)
    for (int y = 0; y < S && y < ny; ++y) issue(y);

  // first E_z(Delta/2) on (z0, z1) of plane y (from the ring) -> (e0, e1), also into the exchange buffer
  auto stage_in = [&](int y, double2* xb, double2& e0, double2& e1) {
    const int s = y % S;
    mbar_wait(&full[s], (uint32_t)((y / S) & 1));
    const double2* r = ring + (long long)s * seg;
    const double2 v0 = r[z0 * kYZW + o];
    if (has1) {
      const double2 v1 = r[z1 * kYZW + o];
      e0 = crow(cz_.a1, v0, cz_.u1, v1);
      e1 = crow(cz_.d1, v0, cz_.a1, v1);
      xb[z1 * kYZW + o] = e1;
    } else {  // zero BC, odd nz: singleton
      e0 = cmul(cz_.s1, v0);
      e1 = cz();
    }
    xb[z0 * kYZW + o] = e0;
  };
  // O_z(Delta) with the neighbours' E outputs, then the second E_z(Delta/2)
  auto stage_out = [&](const double2* xb, double2 e0, double2 e1, double2& w0, double2& w1) {
    double2 q0, q1 = cz();
    if (m > 0) q0 = crow(cz_.d2, xb[(z0 - 1) * kYZW + o], cz_.a2, e0);
    else if (kPer) q0 = crow(cz_.d2, xb[(nz - 1) * kYZW + o], cz_.a2, e0);
    else q0 = cmul(cz_.s2, e0);
    if (has1) {
      if (z1 + 1 < nz) q1 = crow(cz_.a2, e1, cz_.u2, xb[(z1 + 1) * kYZW + o]);
      else if (kPer) q1 = crow(cz_.a2, e1, cz_.u2, xb[o]);
      else q1 = cmul(cz_.s2, e1);
      w0 = crow(cz_.a1, q0, cz_.u1, q1);
      w1 = crow(cz_.d1, q0, cz_.a1, q1);
    } else {
      w0 = cmul(cz_.s1, q0);
      w1 = cz();
    }
  };
  auto st0 = [&](int y, double2 v) {
    if (act) base[(long long)y * yst + (long long)z0 * norb + o] = cmul(phb[(long long)y * nz + z0], v);
  };
  auto st1 = [&](int y, double2 v) {
    if (act && has1) base[(long long)y * yst + (long long)z1 * norb + o] = cmul(phb[(long long)y * nz + z1], v);
  };

  LineMarch L0, L1;
  L0.E10 = L0.O1 = L0.prev_e1 = L0.prev_oR = cz();
  L1 = L0;
  const int npairs = (ny + 1) >> 1;
  for (int p = 0; p < npairs; ++p) {
    const int ya = 2 * p, yb = 2 * p + 1;
    const bool hb = yb < ny;
    double2* xa = xch + (long long)((p & 1) * 2) * seg;
    double2* xb = xa + seg;
    double2 ea0, ea1, eb0 = cz(), eb1 = cz();
    stage_in(ya, xa, ea0, ea1);
    if (hb) stage_in(yb, xb, eb0, eb1);
    __syncthreads();  // exchange buffers written; ring slots of ya, yb consumed
    if (tid < 32) {
      if (ya + S < ny) issue(ya + S);
      if (hb && yb + S < ny) issue(yb + S);
    }
    double2 wa0, wa1, wb0 = cz(), wb1 = cz();
    stage_out(xa, ea0, ea1, wa0, wa1);
    if (hb) stage_out(xb, eb0, eb1, wb0, wb1);
    L0.push(cy, p, wa0, wb0, hb, st0);
    L1.push(cy, p, wa1, wb1, hb, st1);
  }
  L0.finish<kPer>(cy, ny, st0);
  L1.finish<kPer>(cy, ny, st1);
}

static int yz_stages(int nz) {
  const int seg_bytes = nz * kYZW * 16;
  int S = (200 * 1024 - 4 * seg_bytes) / seg_bytes;
  return S > 6 ? 6 : S;
}

bool kin_yz_supported(const Geometry& g) { return g.nz <= 128 && yz_stages(g.nz) >= 2; }

static size_t yz_smem(int nz, int S) { return (size_t)(S + 4) * nz * kYZW * 16 + (size_t)S * 8; }

cudaError_t kin_yz_set_attributes() {
  cudaError_t e = cudaFuncSetAttribute(k_kin_yz<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(k_kin_yz<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
}

cudaError_t launch_kin_yz(const Geometry& g, double2* psi, const DomCoef* coef, const double2* phi,
                          cudaStream_t st) {
  const int nchunks = (g.norb + kYZW - 1) / kYZW;
  const int S = yz_stages(g.nz);
  const int threads = ((g.nz + 1) / 2) * kYZW;
  dim3 grid(g.nx * nchunks, g.ndom);
  const size_t sm = yz_smem(g.nz, S);
  if (g.bc == 0)
    k_kin_yz<true><<<grid, threads, sm, st>>>(psi, coef, phi, g.nx, g.ny, g.nz, g.norb, nchunks, g.ng, S);
  else
    k_kin_yz<false><<<grid, threads, sm, st>>>(psi, coef, phi, g.nx, g.ny, g.nz, g.norb, nchunks, g.ng, S);
  return cudaGetLastError();
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
