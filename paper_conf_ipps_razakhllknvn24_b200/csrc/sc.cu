// sc.cu -- kernels of the self-consistent LFD step (include/lfd.h lfd_sc_*).
//
// Paper: the Hamiltonian of Eq. 5 carries the Hartree and local xc potentials of the density
// being propagated and the vector potential of Maxwell's equation, and each QD step is made
// "self-consistent, time-reversible". The readings R23-R28 fix what is computed:
//   R23  v_H = sum_{G != 0} 4 pi / |G|^2 rho_G e^{iG.r} on the periodic global grid (cuFFT D2Z / Z2D,
//        the 1/|G|^2 filter in k_sc_poisson),
//   R24  v_x = -(3 rho / pi)^{1/3} (k_sc_vhxc),
//   R25/R26  A_ind'' = -4 pi c Jbar by velocity Verlet (k_sc_maxwell_begin / _end),
//   R27  v_mid = 3/2 v(t_n) - 1/2 v(t_n-1), then (v(t_n) + v[rho(Psi^(k))]) / 2 (k_sc_vmid).
// These are O(grid) kernels next to the O(grid x orbitals) step; they run between the step's kernels on
// the context stream. The api.cu side orders them, the cuFFT plans and the NCCL all-reduce.
#include <cufft.h>

#include "lfd_coef.cuh"
#include "lfd_internal.h"

namespace lfd {

namespace {
constexpr double kPi = 3.141592653589793238462643383279502884;
}

// Maxwell state (doubles): [0] A_ind, [3] dA_ind/dt, [6] Jbar, [9] dA/dt at the half step, [12] A_ind(t_n+1),
// [15] A_mid, [18] A_end.  Single CTA: thread 0 advances the state, every thread then builds the coefficient
// tables of its domains for A_mid (stencil) and A_end (density of the step's result).
__global__ void k_sc_maxwell_begin(double* __restrict__ st, double3 a_mid, double3 a_end, double dt, int maxwell,
                                   int ndom, double hx, double hy, double hz, DomCoef* __restrict__ coef_mid,
                                   DomCoef* __restrict__ coef_end) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  __shared__ double Am[3], Ae[3];
  if (threadIdx.x == 0) {
    const double am[3] = {a_mid.x, a_mid.y, a_mid.z}, ae[3] = {a_end.x, a_end.y, a_end.z};
    for (int d = 0; d < 3; ++d) {
      if (maxwell) {
        const double vh = st[3 + d] - 2.0 * kPi * kCLight * dt * st[6 + d];  // half kick with J(t_n)
        const double an = st[d] + dt * vh;                                    // drift to t_n+1
        st[9 + d] = vh;
        st[12 + d] = an;
        Am[d] = am[d] + 0.5 * (st[d] + an);
        Ae[d] = ae[d] + an;
      } else {
        st[9 + d] = st[3 + d];
        st[12 + d] = st[d];
        Am[d] = am[d];
        Ae[d] = ae[d];
      }
      st[15 + d] = Am[d];
      st[18 + d] = Ae[d];
    }
  }
  __syncthreads();
  for (int d = threadIdx.x; d < ndom; d += blockDim.x) {
    if (coef_mid) coef_mid[d] = make_coef(Am, hx, hy, hz, dt);
    coef_end[d] = make_coef(Ae, hx, hy, hz, dt);
  }
}

// End of a step: Jbar(t_n+1) from the (all-reduced) density buffer; A_ind <- A_ind(t_n+1) and the second
// half kick dA/dt <- dA/dt(n+1/2) - 2 pi c dt Jbar(t_n+1).
__global__ void k_sc_maxwell_end(double* __restrict__ st, const double* __restrict__ jbar, double dt, int maxwell) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  const int d = threadIdx.x;
  if (d >= 3) return;
  const double J = jbar[d];
  st[6 + d] = J;
  if (maxwell) {
    st[d] = st[12 + d];
    st[3 + d] = st[9 + d] - 2.0 * kPi * kCLight * dt * J;
  }
}

// Jbar = sum_dom J_dom * (ng / GN): this rank's share of the global-grid mean current (fixed order).
__global__ void k_sc_jbar(const double* __restrict__ Jmac, int ndom, double w, double* __restrict__ out) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  const int d = threadIdx.x;
  if (d >= 3) return;
  double s = 0.0;
  for (int i = 0; i < ndom; ++i) s += Jmac[3 * i + d];
  out[d] = s * w;
}

// v_loc[dom][x][y][z] = v_ion[dom][..] + wa * va[g] + wb * vb[g], g = the point's global index.
__global__ void k_sc_vmid(const double* __restrict__ vion, const double* __restrict__ va,
                          const double* __restrict__ vb, double wa, double wb, const int* __restrict__ off,
                          int nx, int ny, int nz, int GY, int GZ, long long total, double* __restrict__ vout) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= total) return;
  const long long ng = (long long)nx * ny * nz;
  const int dom = (int)(i / ng);
  const long long r = i - (long long)dom * ng;
  const int z = (int)(r % nz);
  const int y = (int)((r / nz) % ny);
  const int x = (int)(r / ((long long)ny * nz));
  const long long gi = ((long long)(off[3 * dom] + x) * GY + (off[3 * dom + 1] + y)) * GZ + (off[3 * dom + 2] + z);
  double v = vion ? vion[i] : 0.0;
  v += wa * va[gi];
  if (wb != 0.0) v += wb * vb[gi];
  vout[i] = v;
}

// rho_G -> 4 pi / |G|^2 rho_G / GN (G = 0 dropped: neutralising background), on the D2Z half spectrum
// [GX][GY][GZ/2+1]; |m_d| = min(k, N_d - k) (the Nyquist term of an even N_d is its own mirror).
__global__ void k_sc_poisson(double2* __restrict__ spec, int GX, int GY, int GZ, double hx, double hy, double hz) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  const int GZh = GZ / 2 + 1;
  const long long n = (long long)GX * GY * GZh;
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const int kz = (int)(i % GZh);
  const int ky = (int)((i / GZh) % GY);
  const int kx = (int)(i / ((long long)GZh * GY));
  const int mx = min(kx, GX - kx), my = min(ky, GY - ky), mz = kz;
  const double gx = 2.0 * kPi * mx / (GX * hx), gy = 2.0 * kPi * my / (GY * hy), gz = 2.0 * kPi * mz / (GZ * hz);
  const double g2 = gx * gx + gy * gy + gz * gz;
  const double f = (i == 0) ? 0.0 : 4.0 * kPi / (g2 * ((double)GX * GY * GZ));
  double2 v = spec[i];
  spec[i] = make_double2(v.x * f, v.y * f);
}

// v_Hxc[g] = (hartree ? v_H[g] : 0) + (xc ? -(3 rho / pi)^{1/3} : 0), in place on v (v_H from the Z2D).
__global__ void k_sc_vhxc(const double* __restrict__ rho, double* __restrict__ v, long long n, int hartree, int xc) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  double r = hartree ? v[i] : 0.0;
  if (xc) r -= cbrt(3.0 * fmax(rho[i], 0.0) / kPi);
  v[i] = r;
}

// ---- launchers ------------------------------------------------------------------------------------
cudaError_t launch_sc_maxwell_begin(double* st, const double* a_mid, const double* a_end, double dt, bool maxwell,
                                    const Geometry& g, DomCoef* coef_mid, DomCoef* coef_end, cudaStream_t s) {
  launch_k(k_sc_maxwell_begin, 1, 256, 0, s, st, make_double3(a_mid[0], a_mid[1], a_mid[2]),
                                       make_double3(a_end[0], a_end[1], a_end[2]), dt, maxwell ? 1 : 0, g.ndom,
                                       g.hx, g.hy, g.hz, coef_mid, coef_end);
  return cudaGetLastError();
}

cudaError_t launch_sc_maxwell_end(double* st, const double* jbar, double dt, bool maxwell, cudaStream_t s) {
  launch_k(k_sc_maxwell_end, 1, 32, 0, s, st, jbar, dt, maxwell ? 1 : 0);
  return cudaGetLastError();
}

cudaError_t launch_sc_jbar(const double* Jmac, int ndom, double w, double* out, cudaStream_t s) {
  launch_k(k_sc_jbar, 1, 32, 0, s, Jmac, ndom, w, out);
  return cudaGetLastError();
}

cudaError_t launch_sc_vmid(const Geometry& g, const double* vion, const double* va, const double* vb, double wa,
                           double wb, const int* off, int GY, int GZ, double* vout, cudaStream_t s) {
  const long long total = (long long)g.ndom * g.ng;
  launch_k(k_sc_vmid, (unsigned)((total + 255) / 256), 256, 0, s, vion, va, vb, wa, wb, off, g.nx, g.ny, g.nz, GY, GZ,
                                                            total, vout);
  return cudaGetLastError();
}

cudaError_t launch_sc_poisson(double2* spec, const int* gd, const Geometry& g, cudaStream_t s) {
  const long long n = (long long)gd[0] * gd[1] * (gd[2] / 2 + 1);
  launch_k(k_sc_poisson, (unsigned)((n + 255) / 256), 256, 0, s, spec, gd[0], gd[1], gd[2], g.hx, g.hy, g.hz);
  return cudaGetLastError();
}

cudaError_t launch_sc_vhxc(const double* rho, double* v, long long n, bool hartree, bool xc, cudaStream_t s) {
  launch_k(k_sc_vhxc, (unsigned)((n + 255) / 256), 256, 0, s, rho, v, n, hartree ? 1 : 0, xc ? 1 : 0);
  return cudaGetLastError();
}

}  // namespace lfd
