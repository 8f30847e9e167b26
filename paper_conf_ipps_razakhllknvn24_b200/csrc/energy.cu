// energy.cu -- the two other "BLASified" LFD functions of P:212 on sm_100a:
//  * calc_energy: E = sum_s f_s <psi_s| T(A) + v_loc + v_nl |psi_s>. The kinetic and local parts are
//    per-CTA partial sums produced by the density kernel (same link products as the current); the
//    nonlocal part sum_s f_s sum_u D_u |C_us|^2 uses C = dV B^H Psi from the DMMA GEMM-1.
//  * remap_occ: occ_k = sum_s f_s |C_ks|^2 with C = dV Ref^H Psi from the same GEMM-1 (the
//    shadow-dynamics handshake maps the propagated orbitals back to occupation numbers).
// Fixed-order reductions only (deterministic).
#include "lfd_internal.h"

namespace lfd {

// One block per domain. E[dom] = {kinetic, local, nonlocal, total}.
__global__ void __launch_bounds__(256) k_energy_final(const double* __restrict__ epart, int blocks,
                                                      const double2* __restrict__ C, const double* __restrict__ D,
                                                      const double* __restrict__ occ, int nproj, int norb, double dV,
                                                      double* __restrict__ E) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  __shared__ double sh[3][256];
  const int dom = blockIdx.x, tid = threadIdx.x;
  double ek = 0.0, el = 0.0, en = 0.0;
  for (int b = tid; b < blocks; b += blockDim.x) {
    ek += epart[((long long)dom * blocks + b) * 2];
    el += epart[((long long)dom * blocks + b) * 2 + 1];
  }
  if (C) {
    const long long mn = (long long)nproj * norb;
    for (long long e = tid; e < mn; e += blockDim.x) {
      const int u = (int)(e / norb), s = (int)(e - (long long)u * norb);
      const double2 c = C[(long long)dom * mn + e];
      en += occ[(long long)dom * norb + s] * D[(long long)dom * nproj + u] * (c.x * c.x + c.y * c.y);
    }
  }
  sh[0][tid] = ek;
  sh[1][tid] = el;
  sh[2][tid] = en;
  __syncthreads();
  for (int w = 128; w > 0; w >>= 1) {
    if (tid < w)
      for (int k = 0; k < 3; ++k) sh[k][tid] += sh[k][tid + w];
    __syncthreads();
  }
  if (tid == 0) {
    const double kin = dV * sh[0][0], loc = dV * sh[1][0], nl = sh[2][0];
    E[dom * 4 + 0] = kin;
    E[dom * 4 + 1] = loc;
    E[dom * 4 + 2] = nl;
    E[dom * 4 + 3] = kin + loc + nl;
  }
}

cudaError_t launch_energy_final(const Geometry& g, const double* epart, int blocks, const double2* C,
                                const double* D, const double* occ, double* E, cudaStream_t st) {
  launch_k(k_energy_final, g.ndom, 256, 0, st, epart, blocks, C, D, occ, g.nproj, g.norb, g.dV, E);
  return cudaGetLastError();
}

// occ_out[dom][k] = sum_s f_s |C[dom][k][s]|^2 : one warp per (dom, k), lanes over s, fixed-order tree.
__global__ void __launch_bounds__(256) k_remap(int ndom, int nref, int norb, const double2* __restrict__ C,
                                               const double* __restrict__ occ, double* __restrict__ out) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  const long long w = ((long long)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  if (w >= (long long)ndom * nref) return;
  const int dom = (int)(w / nref), k = (int)(w - (long long)dom * nref);
  const double2* row = C + ((long long)dom * nref + k) * norb;
  const double* f = occ + (long long)dom * norb;
  double acc = 0.0;
  for (int s = lane; s < norb; s += 32) {
    const double2 c = row[s];
    acc = fma(f[s], fma(c.x, c.x, c.y * c.y), acc);
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
  if (lane == 0) out[w] = acc;
}

cudaError_t launch_remap(const Geometry& g, int nref, const double2* C, const double* occ, double* out,
                         cudaStream_t st) {
  const long long threads = (long long)g.ndom * nref * 32;
  launch_k(k_remap, (unsigned)((threads + 255) / 256), 256, 0, st, g.ndom, nref, g.norb, C, occ, out);
  return cudaGetLastError();
}

}  // namespace lfd
