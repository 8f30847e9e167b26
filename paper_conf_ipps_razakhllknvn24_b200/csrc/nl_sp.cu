// nl_sp.cu -- the projector GEMMs of the SP variant (complex64 Psi / B) for sm_100a.
//
// Same operations as nl.cu (Eq. 7 / Eq. 9, P:68 / P:210; readings R9-R12):
//   GEMM-1  part[dom][split][m][n] = sum_{r in split} conj(A[r][m]) X[r][n]  (+ column norms of X)
//   GEMM-2  psi[r][n] <- nfac[n] psi[r][n] + sum_m B[r][m] Xc[m][n]
// in single precision on the tensor pipe: B200 has no FP32 tensor-core kind, so every real product runs as
// 3xTF32 on the warp-level HMMA path (mma.sync m16n8k8 tf32, 279 TF/s measured on this pool vs 72 TF/s
// FFMA, profiles/r01_sp_peaks.txt): x = hi + lo with hi = trunc_tf32(x), lo = x - hi, and
// a b ~ hi_a hi_b + hi_a lo_b + lo_a hi_b (relative error ~2^-20 per product), FP32 accumulation -- close to
// the accuracy of an FP32 GEMM. Complex products use the 3M form (3 real products; 9 HMMA per complex
// tile-step instead of 12). GEMM-1 writes its split partials in FP64, so the split reduction, the
// norm / carry / merge kernels and everything downstream of them are the FP64 kernels of nl.cu; GEMM-2
// reads the coefficient X'' rounded to complex64 once per call (k_to_c64).
// Operands are staged in shared memory by cp.async (8-byte, zero fill past the edges) in a 2-deep ring
// over K chunks of 32; CTA tile 64 x 64 complex, 8 warps of 32 x 16.
#include "lfd_internal.h"

namespace lfd {

namespace {

constexpr int kSpT = 64;              // CTA tile (rows of the output) x 64 columns
constexpr int kSpKC = 32;             // K chunk
constexpr int kSpLdA = kSpT + 4;      // smem row stride (float2) of [k][m] / [k][n] tiles
constexpr int kSpLdK = kSpKC + 4;     // smem row stride (float2) of [m][k] tiles
constexpr int kSpThreads = 256;

// 8-byte async copy global -> shared; zero fill when !ok (then nothing is read; `base` is a valid address)
__device__ __forceinline__ void cp8(void* smem, const void* gmem, bool ok, const void* base) {
  const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;" ::"r"(s), "l"(ok ? gmem : base), "r"(ok ? 8 : 0)
               : "memory");
}
__device__ __forceinline__ void cp_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
__device__ __forceinline__ void cp_wait1() { asm volatile("cp.async.wait_group 1;" ::: "memory"); }
__device__ __forceinline__ void cp_wait0() { asm volatile("cp.async.wait_group 0;" ::: "memory"); }

// 3xTF32 split of an FP32 operand: the tensor core reads only the top 19 bits of a tf32 operand (the low 13
// mantissa bits are ignored: truncation), so hi = x itself acts as trunc(x), and lo = x - trunc(x) is exact
// in FP32 (one LOP3 + one FADD per value).
struct TF {
  unsigned hi, lo;
};
__device__ __forceinline__ TF split_tf32(float x) {
  const unsigned xb = __float_as_uint(x);
  return {xb, __float_as_uint(x - __uint_as_float(xb & 0xffffe000u))};
}
// Not volatile: the compiler may interleave the independent HMMAs of different accumulators.
__device__ __forceinline__ void hmma(float* c, unsigned a0, unsigned a1, unsigned a2, unsigned a3, unsigned b0,
                                     unsigned b1) {
  asm("mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
      "{%0,%1,%2,%3};"
      : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
      : "r"(a0), "r"(a1), "r"(a2), "r"(a3), "r"(b0), "r"(b1));
}

// One k8 step of a warp tile of MT x NT (16 x 8) tiles, complex, in the 3M form (three real products per
// complex product), each real product in 3xTF32: a b ~ lo_a hi_b + hi_a lo_b + hi_a hi_b (small terms
// first; lo_a lo_b ~ 2^-20 |ab| dropped).
// a[mi][0..3]: complex A fragment (rows g, g+8, cols t, t+4), b[ni][0..1]: complex B fragment (k t, t+4).
//   plain (GEMM-2): T1 = Ar Br, T2 = Ai Bi, T3 = (Ar + Ai)(Br + Bi);  Re = T1 - T2, Im = T3 - T1 - T2
//   kConj (GEMM-1): T1 = Ar Br, T2 = Ai Bi, T3 = (Ar - Ai)(Br + Bi);  Re = T1 + T2, Im = T3 - T1 + T2
// (cmma_finish forms Re, Im.) Issue order: term-major, then product, then tile, so consecutive HMMAs update
// different accumulators.
template <int MT, int NT, bool kConj>
__device__ __forceinline__ void cmma_k8(float (&acc)[3][MT][NT][4], const float2 (&a)[MT][4], const float2 (&b)[NT][2]) {
  TF as[3][MT][4], bs[3][NT][2];
#pragma unroll
  for (int mi = 0; mi < MT; ++mi)
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      as[0][mi][q] = split_tf32(a[mi][q].x);
      as[1][mi][q] = split_tf32(a[mi][q].y);
      as[2][mi][q] = split_tf32(kConj ? a[mi][q].x - a[mi][q].y : a[mi][q].x + a[mi][q].y);
    }
#pragma unroll
  for (int ni = 0; ni < NT; ++ni)
#pragma unroll
    for (int q = 0; q < 2; ++q) {
      bs[0][ni][q] = split_tf32(b[ni][q].x);
      bs[1][ni][q] = split_tf32(b[ni][q].y);
      bs[2][ni][q] = split_tf32(b[ni][q].x + b[ni][q].y);
    }
#pragma unroll
  for (int term = 0; term < 3; ++term)  // 0: lo_a hi_b, 1: hi_a lo_b, 2: hi_a hi_b
#pragma unroll
    for (int p = 0; p < 3; ++p)
#pragma unroll
      for (int mi = 0; mi < MT; ++mi)
#pragma unroll
        for (int ni = 0; ni < NT; ++ni) {
          const TF* A = as[p][mi];
          const TF* B = bs[p][ni];
          if (term == 0) hmma(acc[p][mi][ni], A[0].lo, A[1].lo, A[2].lo, A[3].lo, B[0].hi, B[1].hi);
          else if (term == 1) hmma(acc[p][mi][ni], A[0].hi, A[1].hi, A[2].hi, A[3].hi, B[0].lo, B[1].lo);
          else hmma(acc[p][mi][ni], A[0].hi, A[1].hi, A[2].hi, A[3].hi, B[0].hi, B[1].hi);
        }
}

template <bool kConj>
__device__ __forceinline__ float2 cmma_finish(float t1, float t2, float t3) {
  return kConj ? make_float2(t1 + t2, t3 - t1 + t2) : make_float2(t1 - t2, t3 - t1 - t2);
}

// ------------------------------------------------------------------------------------------------
// GEMM-1 (SP). grid (nsplit, mtiles * ntiles, ndom); 8 warps = 2 (M) x 4 (N), warp tile 32 x 16.
// smem per stage: As[k][m] = A rows (conjugated in the product), Xs[k][n] = X rows.
// ------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(kSpThreads) k_gemm1_sp(const float2* __restrict__ A, const float2* __restrict__ X,
                                                          double2* __restrict__ part, double* __restrict__ norms,
                                                          int mrows, int ncols, int nsplit, long long ng,
                                                          long long rps, long long a_ds, long long x_ds) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  extern __shared__ __align__(16) float2 sp_smem[];
  auto As = reinterpret_cast<float2(*)[kSpKC][kSpLdA]>(sp_smem);                       // [2][KC][LdA]
  auto Xs = reinterpret_cast<float2(*)[kSpKC][kSpLdA]>(sp_smem + 2 * kSpKC * kSpLdA);  // [2][KC][LdA]
  const int split = blockIdx.x, dom = blockIdx.z;
  const int ntn = (ncols + kSpT - 1) / kSpT;
  const int m0 = (blockIdx.y / ntn) * kSpT, n0 = (blockIdx.y % ntn) * kSpT;
  const long long rb = (long long)split * rps, re_ = min(ng, rb + rps);
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, g = lane >> 2, t = lane & 3;
  const int wm = warp >> 2, wn = warp & 3;
  const float2* Ad = A + dom * a_ds;
  const float2* Xd = X + dom * x_ds;
  const int nchunks = (int)((max(re_ - rb, 0LL) + kSpKC - 1) / kSpKC);

  auto load = [&](int c, int st) {
    const long long r0 = rb + (long long)c * kSpKC;
    for (int i = tid; i < kSpKC * kSpT; i += kSpThreads) {
      const int k = i / kSpT, m = i % kSpT;
      const long long r = r0 + k;
      const bool rok = r < re_;
      cp8(&As[st][k][m], Ad + r * mrows + m0 + m, rok && m0 + m < mrows, A);
      cp8(&Xs[st][k][m], Xd + r * ncols + n0 + m, rok && n0 + m < ncols, X);
    }
    cp_commit();
  };

  float acc[3][2][2][4];
#pragma unroll
  for (int p = 0; p < 3; ++p)
#pragma unroll
    for (int mi = 0; mi < 2; ++mi)
#pragma unroll
      for (int ni = 0; ni < 2; ++ni)
#pragma unroll
        for (int q = 0; q < 4; ++q) acc[p][mi][ni][q] = 0.f;
  float nrm[2] = {0.f, 0.f};  // |X|^2 of columns (wn*16 + ni*8 + g), k = t, t+4 (warps wm == 0)

  if (nchunks > 0) load(0, 0);
  for (int c = 0; c < nchunks; ++c) {
    const int st = c & 1;
    if (c + 1 < nchunks) {
      load(c + 1, st ^ 1);
      cp_wait1();
    } else {
      cp_wait0();
    }
    __syncthreads();
#pragma unroll
    for (int k8 = 0; k8 < kSpKC / 8; ++k8) {
      const int k = k8 * 8 + t;
      float2 a[2][4], b[2][2];
#pragma unroll
      for (int mi = 0; mi < 2; ++mi) {
        const int m = wm * 32 + mi * 16 + g;
        a[mi][0] = As[st][k][m];
        a[mi][1] = As[st][k][m + 8];
        a[mi][2] = As[st][k + 4][m];
        a[mi][3] = As[st][k + 4][m + 8];
      }
#pragma unroll
      for (int ni = 0; ni < 2; ++ni) {
        const int n = wn * 16 + ni * 8 + g;
        b[ni][0] = Xs[st][k][n];
        b[ni][1] = Xs[st][k + 4][n];
        if (wm == 0)
          nrm[ni] += b[ni][0].x * b[ni][0].x + b[ni][0].y * b[ni][0].y + b[ni][1].x * b[ni][1].x +
                     b[ni][1].y * b[ni][1].y;
      }
      cmma_k8<2, 2, true>(acc, a, b);
    }
    __syncthreads();
  }
  // partials (FP64): rows m0 + wm*32 + mi*16 + g (+8), columns n0 + wn*16 + ni*8 + 2t (+1)
  double2* P = part + ((long long)dom * nsplit + split) * (long long)mrows * ncols;
#pragma unroll
  for (int mi = 0; mi < 2; ++mi)
#pragma unroll
    for (int ni = 0; ni < 2; ++ni)
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int m = m0 + wm * 32 + mi * 16 + g + (q >> 1) * 8;
        const int n = n0 + wn * 16 + ni * 8 + 2 * t + (q & 1);
        if (m < mrows && n < ncols) {
          const float2 v = cmma_finish<true>(acc[0][mi][ni][q], acc[1][mi][ni][q], acc[2][mi][ni][q]);
          P[(long long)m * ncols + n] = make_double2(v.x, v.y);
        }
      }
  if (norms && wm == 0 && blockIdx.y < ntn) {  // first M tile only (the norms do not depend on m)
#pragma unroll
    for (int ni = 0; ni < 2; ++ni) {
      float v = nrm[ni];
      v += __shfl_xor_sync(0xffffffffu, v, 1);
      v += __shfl_xor_sync(0xffffffffu, v, 2);
      const int n = n0 + wn * 16 + ni * 8 + g;
      if (t == 0 && n < ncols) norms[((long long)dom * nsplit + split) * ncols + n] = v;
    }
  }
}

// ------------------------------------------------------------------------------------------------
// GEMM-2 (SP). grid (row blocks of 64, column tiles of 64, ndom); K = nproj in chunks of 32.
// smem per stage: Bs[m][k] (B rows), Xs[k][n] (the complex64 coefficient X'').
// ------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(kSpThreads) k_gemm2_sp(const float2* psi, float2* pout, const float2* __restrict__ B,
                                                          const float2* __restrict__ Xc, const double* __restrict__ nfac,
                                                          int np, int norb, long long ng) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  extern __shared__ __align__(16) float2 sp_smem[];
  auto Bs = reinterpret_cast<float2(*)[kSpT][kSpLdK]>(sp_smem);                        // [2][T][LdK]
  auto Xs = reinterpret_cast<float2(*)[kSpKC][kSpLdA]>(sp_smem + 2 * kSpT * kSpLdK);   // [2][KC][LdA]
  const int dom = blockIdx.z;
  const long long r0 = (long long)blockIdx.x * kSpT;
  const int n0 = blockIdx.y * kSpT;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, g = lane >> 2, t = lane & 3;
  const int wm = warp >> 2, wn = warp & 3;
  const float2* Bd = B + (long long)dom * ng * np;
  const float2* Xd = Xc + (long long)dom * np * norb;
  const float2* Pd = psi + (long long)dom * ng * norb;
  float2* Po = pout + (long long)dom * ng * norb;
  const int nchunks = (np + kSpKC - 1) / kSpKC;
  {  // the epilogue's Psi tile to L2 now (one 128-byte line per thread covers rows x 64 columns)
    const int rr = tid / 4, cc = n0 + (tid % 4) * 16;
    if (r0 + rr < ng && cc < norb)
      asm volatile("prefetch.global.L2 [%0];" ::"l"(Pd + (r0 + rr) * norb + cc));
  }

  auto load = [&](int c, int st) {
    const int k0 = c * kSpKC;
    for (int i = tid; i < kSpT * kSpKC; i += kSpThreads) {
      const int r = i / kSpKC, k = i % kSpKC;  // B rows: consecutive threads along k (contiguous in HBM)
      cp8(&Bs[st][r][k], Bd + (r0 + r) * np + k0 + k, r0 + r < ng && k0 + k < np, B);
      const int kk = i / kSpT, n = i % kSpT;
      cp8(&Xs[st][kk][n], Xd + (long long)(k0 + kk) * norb + n0 + n, k0 + kk < np && n0 + n < norb, Xc);
    }
    cp_commit();
  };

  float acc[3][2][2][4];
#pragma unroll
  for (int p = 0; p < 3; ++p)
#pragma unroll
    for (int mi = 0; mi < 2; ++mi)
#pragma unroll
      for (int ni = 0; ni < 2; ++ni)
#pragma unroll
        for (int q = 0; q < 4; ++q) acc[p][mi][ni][q] = 0.f;

  load(0, 0);
  for (int c = 0; c < nchunks; ++c) {
    const int st = c & 1;
    if (c + 1 < nchunks) {
      load(c + 1, st ^ 1);
      cp_wait1();
    } else {
      cp_wait0();
    }
    __syncthreads();
#pragma unroll
    for (int k8 = 0; k8 < kSpKC / 8; ++k8) {
      const int k = k8 * 8 + t;
      float2 a[2][4], b[2][2];
#pragma unroll
      for (int mi = 0; mi < 2; ++mi) {
        const int m = wm * 32 + mi * 16 + g;
        a[mi][0] = Bs[st][m][k];
        a[mi][1] = Bs[st][m + 8][k];
        a[mi][2] = Bs[st][m][k + 4];
        a[mi][3] = Bs[st][m + 8][k + 4];
      }
#pragma unroll
      for (int ni = 0; ni < 2; ++ni) {
        const int n = wn * 16 + ni * 8 + g;
        b[ni][0] = Xs[st][k][n];
        b[ni][1] = Xs[st][k + 4][n];
      }
      cmma_k8<2, 2, false>(acc, a, b);
    }
    __syncthreads();
  }
  // epilogue: psi <- n psi + B X'' in place (columns 2t, 2t+1 of a fragment are adjacent orbitals)
  const double* nf = nfac + (long long)dom * norb;
#pragma unroll
  for (int mi = 0; mi < 2; ++mi)
#pragma unroll
    for (int ni = 0; ni < 2; ++ni)
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const long long r = r0 + wm * 32 + mi * 16 + g + (q >> 1) * 8;
        const int n = n0 + wn * 16 + ni * 8 + 2 * t + (q & 1);
        if (r < ng && n < norb) {
          const float f = (float)nf[n];
          const float2 v = Pd[r * norb + n];
          const float2 u = cmma_finish<false>(acc[0][mi][ni][q], acc[1][mi][ni][q], acc[2][mi][ni][q]);
          Po[r * norb + n] = make_float2(fmaf(f, v.x, u.x), fmaf(f, v.y, u.y));
        }
      }
}

__global__ void k_to_c64(const double2* __restrict__ in, float2* __restrict__ out, long long n) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  const long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) out[i] = make_float2((float)in[i].x, (float)in[i].y);
}

constexpr size_t kSmem1 = 2 * 2 * kSpKC * kSpLdA * sizeof(float2);
constexpr size_t kSmem2 = (2 * kSpT * kSpLdK + 2 * kSpKC * kSpLdA) * sizeof(float2);

}  // namespace

cudaError_t gemm_sp_set_attributes() {
  cudaError_t e = cudaFuncSetAttribute(k_gemm1_sp, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmem1);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(k_gemm2_sp, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmem2);
  return e;
}

cudaError_t launch_gemm1_sp(const Gemm1Args& a, const float2* A, const float2* X, cudaStream_t st) {
  const int mt = (a.mrows + kSpT - 1) / kSpT, nt = (a.ncols + kSpT - 1) / kSpT;
  dim3 grid(a.nsplit, mt * nt, a.ndom);
  launch_k(k_gemm1_sp, grid, kSpThreads, kSmem1, st, A, X, a.part, a.norms, a.mrows, a.ncols, a.nsplit, a.ng, a.rows_per_split,
                                          a.a_dom_stride, a.x_dom_stride);
  return cudaGetLastError();
}

cudaError_t launch_gemm2_sp(float2* psi, const float2* B, const double2* Cp, float2* X32, const double* nfac,
                            int ndom, int nproj, int norb, long long ng, cudaStream_t st, float2* psi_out) {
  const long long n = (long long)ndom * nproj * norb;
  launch_k(k_to_c64, (unsigned)((n + 255) / 256), 256, 0, st, Cp, X32, n);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  dim3 grid((unsigned)((ng + kSpT - 1) / kSpT), (norb + kSpT - 1) / kSpT, ndom);
  launch_k(k_gemm2_sp, grid, kSpThreads, kSmem2, st, psi, psi_out ? psi_out : psi, B, X32, nfac, nproj, norb, ng);
  return cudaGetLastError();
}

}  // namespace lfd
