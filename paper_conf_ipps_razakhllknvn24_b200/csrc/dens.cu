// dens.cu -- density and current (north star subsystem (4)) for sm_100a.
//
//   rho_r   = sum_s f_s |psi_rs|^2
//   j_d,r   = (1/h_d) Im( e^{i theta_d} sum_s f_s conj(psi_rs) psi_{r+e_d,s} )   (reading R13)
//   J_d     = (1/Ngrid) sum_r j_d,r
// One warp per (domain, x, y) line walks z; lanes span orbitals (orbital-innermost layout), so
// each row load is one contiguous segment; the 7 per-point sums are warp-shuffle reductions over
// orbitals with the occupation weights. Per-line sums of j are reduced in a fixed order by k_jreduce
// (deterministic, no atomics).
#include "lfd_complex.cuh"
#include "lfd_internal.h"

namespace lfd {

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

__global__ void __launch_bounds__(256) k_density(Geometry g, DensArgs a) {
  const int warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const int lines = g.nx * g.ny;
  if (warp >= lines * g.ndom) return;
  const int dom = warp / lines;
  const int line = warp - dom * lines;
  const int x = line / g.ny, y = line - (line / g.ny) * g.ny;
  const int norb = g.norb;
  const bool per = (g.bc == 0);
  const bool has_x = per || (x + 1 < g.nx);
  const bool has_y = per || (y + 1 < g.ny);
  const int xp = (x + 1 == g.nx) ? 0 : x + 1;
  const int yp = (y + 1 == g.ny) ? 0 : y + 1;
  const double2* P = a.psi + (long long)dom * g.ng * norb;
  const double* f = a.occ + (long long)dom * norb;
  const DomCoef* cf = a.coef + dom;
  const double2 ex = cf->eth[0], ey = cf->eth[1], ez = cf->eth[2];
  const double ihx = cf->inv_h[0], ihy = cf->inv_h[1], ihz = cf->inv_h[2];
  const long long rbase = ((long long)x * g.ny + y) * g.nz;
  const long long rxbase = ((long long)xp * g.ny + y) * g.nz;
  const long long rybase = ((long long)x * g.ny + yp) * g.nz;
  const long long xy = (long long)x * a.sx + (long long)y * a.sy;
  const long long obase = a.base[dom] + xy;
  const long long jobase = a.jbase[dom] + xy;
  double jsx = 0.0, jsy = 0.0, jsz = 0.0;
  for (int z = 0; z < g.nz; ++z) {
    const bool has_z = per || (z + 1 < g.nz);
    const int zp = (z + 1 == g.nz) ? 0 : z + 1;
    double rho = 0.0, pxr = 0.0, pxi = 0.0, pyr = 0.0, pyi = 0.0, pzr = 0.0, pzi = 0.0;
    for (int s = lane; s < norb; s += 32) {
      const double fs = __ldg(f + s);
      const double2 v = P[(rbase + z) * norb + s];
      rho = fma(fs, fma(v.x, v.x, v.y * v.y), rho);
      if (has_x) {
        const double2 w = cconjmul(v, P[(rxbase + z) * norb + s]);
        pxr = fma(fs, w.x, pxr);
        pxi = fma(fs, w.y, pxi);
      }
      if (has_y) {
        const double2 w = cconjmul(v, P[(rybase + z) * norb + s]);
        pyr = fma(fs, w.x, pyr);
        pyi = fma(fs, w.y, pyi);
      }
      if (has_z) {
        const double2 w = cconjmul(v, P[(rbase + zp) * norb + s]);
        pzr = fma(fs, w.x, pzr);
        pzi = fma(fs, w.y, pzi);
      }
    }
    rho = warp_sum(rho);
    pxr = warp_sum(pxr); pxi = warp_sum(pxi);
    pyr = warp_sum(pyr); pyi = warp_sum(pyi);
    pzr = warp_sum(pzr); pzi = warp_sum(pzi);
    // Im(e^{i theta} P) = cos(theta) Im P + sin(theta) Re P
    const double jx = has_x ? (ex.x * pxi + ex.y * pxr) * ihx : 0.0;
    const double jy = has_y ? (ey.x * pyi + ey.y * pyr) * ihy : 0.0;
    const double jz = has_z ? (ez.x * pzi + ez.y * pzr) * ihz : 0.0;
    jsx += jx; jsy += jy; jsz += jz;
    if (lane == 0) {
      a.rho[obase + z] = rho;
      if (a.j) {
        const long long o = jobase + z;
        a.j[o] = jx;
        a.j[o + a.jstride] = jy;
        a.j[o + 2 * a.jstride] = jz;
      }
    }
  }
  if (lane == 0) {
    double* jl = a.jline + ((long long)dom * lines + line) * 3;
    jl[0] = jsx; jl[1] = jsy; jl[2] = jsz;
  }
}

cudaError_t launch_density(const Geometry& g, const DensArgs& a, cudaStream_t st) {
  const long long warps = (long long)g.ndom * g.nx * g.ny;
  const unsigned blocks = (unsigned)((warps * 32 + 255) / 256);
  k_density<<<blocks, 256, 0, st>>>(g, a);
  return cudaGetLastError();
}

// J_d = (1/Ngrid) sum_lines jline (one block per domain, fixed-order tree over a fixed partition).
__global__ void __launch_bounds__(256) k_jreduce(const double* __restrict__ jline, int lines, double inv_ng,
                                                 double* __restrict__ Jmac) {
  __shared__ double sh[3][256];
  const int dom = blockIdx.x;
  double s[3] = {0.0, 0.0, 0.0};
  for (int l = threadIdx.x; l < lines; l += blockDim.x)
    for (int d = 0; d < 3; ++d) s[d] += jline[((long long)dom * lines + l) * 3 + d];
  for (int d = 0; d < 3; ++d) sh[d][threadIdx.x] = s[d];
  __syncthreads();
  for (int w = 128; w > 0; w >>= 1) {
    if (threadIdx.x < w)
      for (int d = 0; d < 3; ++d) sh[d][threadIdx.x] += sh[d][threadIdx.x + w];
    __syncthreads();
  }
  if (threadIdx.x < 3) Jmac[dom * 3 + threadIdx.x] = sh[threadIdx.x][0] * inv_ng;
}

cudaError_t launch_jreduce(const Geometry& g, const double* jline, double* Jmac, cudaStream_t st) {
  k_jreduce<<<g.ndom, 256, 0, st>>>(jline, g.nx * g.ny, 1.0 / (double)g.ng, Jmac);
  return cudaGetLastError();
}

}  // namespace lfd
