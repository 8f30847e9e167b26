// dens.cu -- density and current (north star subsystem (4)) for sm_100a.
//
//   rho_r   = sum_s f_s |psi_rs|^2
//   j_d,r   = (1/h_d) Im( e^{i theta_d} sum_s f_s conj(psi_rs) psi_{r+e_d,s} )   (reading R13)
//   J_d     = (1/Ngrid) sum_r j_d,r
// Lanes span orbitals (orbital-innermost layout) and the 7 per-point sums are shuffle
// reductions over orbitals with the occupation weights; per-CTA sums of j are reduced in a fixed
// order by k_jreduce (deterministic, no atomics).
#include "lfd_complex.cuh"
#include "lfd_internal.h"

namespace lfd {

// Tiling: a CTA owns a (kTY x kTZ) tile of (y, z) points and a chunk of kXC x-planes, which it walks in
// x order; each point is served by kSub consecutive lanes that split its orbitals (s = q, q+kSub, ...),
// so a warp load covers kSub*16 contiguous bytes per point. The x+1 / y+1 / z+1 neighbour rows are
// re-read through L1 (the x+1 row is the next iteration's own row; y+1 / z+1 rows mostly belong to the
// same tile), so HBM sees each row about once. Per-point sums are 3-level shuffle reductions over the
// kSub lanes; per-CTA partial J sums are reduced in a fixed order by k_jreduce.
constexpr int kSub = 8, kTY = 2, kTZ = 8, kXC = 10;
constexpr int kDensThreads = kSub * kTY * kTZ;  // 128

__global__ void __launch_bounds__(kDensThreads) k_density(Geometry g, DensArgs a, int ntz, int nty, int nxc) {
  __shared__ double jsh[3][kDensThreads / kSub];
  const int dom = blockIdx.y;
  int b = blockIdx.x;
  const int tz = b % ntz; b /= ntz;
  const int ty = b % nty; b /= nty;
  const int xc = b;
  const int q = threadIdx.x % kSub, pt = threadIdx.x / kSub;
  const int y = ty * kTY + pt / kTZ, z = tz * kTZ + pt % kTZ;
  const bool valid = (y < g.ny) && (z < g.nz);
  const int norb = g.norb;
  const bool per = (g.bc == 0);
  const bool has_y = valid && (per || y + 1 < g.ny);
  const bool has_z = valid && (per || z + 1 < g.nz);
  const int yp = (y + 1 >= g.ny) ? 0 : y + 1;
  const int zp = (z + 1 >= g.nz) ? 0 : z + 1;
  const double2* P = a.psi + (long long)dom * g.ng * norb;
  const double* f = a.occ + (long long)dom * norb;
  const DomCoef* cf = a.coef + dom;
  const double2 ex = cf->eth[0], ey = cf->eth[1], ez = cf->eth[2];
  const double ihx = cf->inv_h[0], ihy = cf->inv_h[1], ihz = cf->inv_h[2];
  const int x0 = xc * nxc, x1 = min(g.nx, x0 + nxc);
  double jsx = 0.0, jsy = 0.0, jsz = 0.0;
  for (int x = x0; x < x1; ++x) {
    const bool has_x = valid && (per || x + 1 < g.nx);
    const int xp = (x + 1 == g.nx) ? 0 : x + 1;
    const long long r = ((long long)x * g.ny + y) * g.nz + z;
    const long long rx = ((long long)xp * g.ny + y) * g.nz + z;
    const long long ry = ((long long)x * g.ny + yp) * g.nz + z;
    const long long rz = ((long long)x * g.ny + y) * g.nz + zp;
    double rho = 0.0, pxr = 0.0, pxi = 0.0, pyr = 0.0, pyi = 0.0, pzr = 0.0, pzi = 0.0;
    if (valid) {
#pragma unroll 4
      for (int s = q; s < norb; s += kSub) {
        const double fs = __ldg(f + s);
        const double2 v = __ldg(P + r * norb + s);
        rho = fma(fs, fma(v.x, v.x, v.y * v.y), rho);
        if (has_x) {
          const double2 w = cconjmul(v, __ldg(P + rx * norb + s));
          pxr = fma(fs, w.x, pxr);
          pxi = fma(fs, w.y, pxi);
        }
        if (has_y) {
          const double2 w = cconjmul(v, __ldg(P + ry * norb + s));
          pyr = fma(fs, w.x, pyr);
          pyi = fma(fs, w.y, pyi);
        }
        if (has_z) {
          const double2 w = cconjmul(v, __ldg(P + rz * norb + s));
          pzr = fma(fs, w.x, pzr);
          pzi = fma(fs, w.y, pzi);
        }
      }
    }
#pragma unroll
    for (int o = kSub / 2; o > 0; o >>= 1) {
      rho += __shfl_xor_sync(0xffffffffu, rho, o);
      pxr += __shfl_xor_sync(0xffffffffu, pxr, o);
      pxi += __shfl_xor_sync(0xffffffffu, pxi, o);
      pyr += __shfl_xor_sync(0xffffffffu, pyr, o);
      pyi += __shfl_xor_sync(0xffffffffu, pyi, o);
      pzr += __shfl_xor_sync(0xffffffffu, pzr, o);
      pzi += __shfl_xor_sync(0xffffffffu, pzi, o);
    }
    // Im(e^{i theta} P) = cos(theta) Im P + sin(theta) Re P
    const double jx = has_x ? (ex.x * pxi + ex.y * pxr) * ihx : 0.0;
    const double jy = has_y ? (ey.x * pyi + ey.y * pyr) * ihy : 0.0;
    const double jz = has_z ? (ez.x * pzi + ez.y * pzr) * ihz : 0.0;
    jsx += jx; jsy += jy; jsz += jz;
    if (q == 0 && valid) {
      const long long o = (long long)x * a.sx + (long long)y * a.sy + z;
      a.rho[a.base[dom] + o] = rho;
      if (a.j) {
        const long long oj = a.jbase[dom] + o;
        a.j[oj] = jx;
        a.j[oj + a.jstride] = jy;
        a.j[oj + 2 * a.jstride] = jz;
      }
    }
  }
  if (q == 0) {
    jsh[0][pt] = jsx; jsh[1][pt] = jsy; jsh[2][pt] = jsz;
  }
  __syncthreads();
  if (threadIdx.x < 3) {
    double t = 0.0;
    for (int i = 0; i < kDensThreads / kSub; ++i) t += jsh[threadIdx.x][i];
    a.jline[((long long)dom * gridDim.x + blockIdx.x) * 3 + threadIdx.x] = t;
  }
}

int density_blocks(const Geometry& g) {
  const int ntz = (g.nz + kTZ - 1) / kTZ, nty = (g.ny + kTY - 1) / kTY, nxc = (g.nx + kXC - 1) / kXC;
  return ntz * nty * nxc;
}

cudaError_t launch_density(const Geometry& g, const DensArgs& a, cudaStream_t st) {
  const int ntz = (g.nz + kTZ - 1) / kTZ, nty = (g.ny + kTY - 1) / kTY;
  dim3 grid(density_blocks(g), g.ndom);
  k_density<<<grid, kDensThreads, 0, st>>>(g, a, ntz, nty, kXC);
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
  k_jreduce<<<g.ndom, 256, 0, st>>>(jline, density_blocks(g), 1.0 / (double)g.ng, Jmac);
  return cudaGetLastError();
}

}  // namespace lfd
