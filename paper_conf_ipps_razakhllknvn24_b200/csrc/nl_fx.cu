// nl_fx.cu -- the first nonlocal factor's GEMM-2 fused with the x pass of the local propagator.
//
// Eq. 6 applies N, then the local factor Phi . K_z K_y K_x (Phi . ), then N. The GEMM-2 of the first N
// (Psi <- n Psi + B C'', Eq. 9; nl_i8.cu) writes Psi and the x pass (Psi <- K_x (Phi . Psi), kin.cu)
// reads it straight back: one full read + write of Psi per step (722 MB at C2) that this kernel removes.
// A work item is one x-line (y, z) of a domain: all nx points x of all orbitals. The int8-digit products
// (nl_i8.cu's scheme: 6 balanced digits, 21 digit pairs in int32 TMEM accumulators, FP64 recombination) run
// with the line as the MMA's N = 80 (zero rows past nx); the epilogue writes n Psi + B C'' into the line's
// shared-memory copy of Psi, and two march warps (one thread per orbital: the paper's psi_old carry,
// Alg. 3 l.6, in registers) stream K_x (Phi . ) along the line from shared memory into HBM.
//
// Roles (20 warps): 16 epilogue warps (4 TMEM lane quarters x 4 groups of 20 x), the MMA issuer (which also
// loads B's digit tile of the next line as soon as the previous line's MMAs are done: one 4-D TMA copy
// [6 digits][80 x][128 B], 128B-swizzled by the TMA, rows past nx zero-filled), a producer of the line (one TMA copy each of Psi [nx][2 norb] and Phi [nx], one bulk copy of
// B's row scales) and the two march warps. Shared memory: one digit tile (60 KB) + two line buffers
// (ping-pong: the epilogue fills one while the march drains the other). TMEM: the W digits (A operand,
// 192 columns) + a 4-slot ring of 80-column diagonal accumulators.
#include <algorithm>
#include <new>
#ifdef LFD_FX_TIMING
#include <cstdio>
#endif

#include "lfd_internal.h"
#include "lfd_march.cuh"  // PairCoef, pair_coef
#include "lfd_tc.cuh"
#include "lfd_tma.cuh"

namespace lfd {

// Role-wait instrumentation for A/B experiments only (compiled in with -DLFD_FX_TIMING; printf from two CTAs)
#ifdef LFD_FX_TIMING
#define FX_T0(v) long long v = clock64()
#define FX_ACC(acc, v) acc += clock64() - v
#else
#define FX_T0(v)
#define FX_ACC(acc, v)
#endif

constexpr int kFxN = 80;                     // MMA N: x points of a line tile (nx <= 80)
constexpr int kFxK = 128;                    // bytes per digit row (K = 2 nproj padded to 128)
constexpr int kFxSliceB = kFxN * kFxK;       // 10 KB per digit
constexpr int kFxTileB = kI8S * kFxSliceB;   // 60 KB
constexpr int kFxSlots = 4;                  // TMEM ring of diagonal accumulators (80 columns each)
constexpr int kFxWCols = kI8S * (kFxK / 4);  // 192 TMEM columns of W^T digits
constexpr int kFxAcc = kI8S;                 // diagonals d = 2 .. S+1
constexpr int kFxEpi = 16;                   // epilogue warps
constexpr int kFxXg = kFxN / 4;              // x points per epilogue warp
constexpr int kFxMarch = 4;                  // march warps (one warpgroup): 64 orbitals x 2 segments of each line
constexpr int kFxSeg = 2;                    // segments of a periodic line marched in parallel
constexpr int kFxWMarch0 = kFxEpi, kFxWMma = kFxEpi + kFxMarch, kFxWLine = kFxWMma + 1;  // + 2 idle warps
constexpr int kFxThreads = (kFxEpi + kFxMarch + 4) * 32;  // 24 warps = 6 warpgroups (setmaxnreg: 96 / 64)
constexpr int kFxXchB = 2 * kFxSeg * 64 * 32;             // segment boundary E outputs [parity][seg][s][2]
// named barriers: epilogue -> march "ready" (2, 3 by line parity), march -> epilogue "free" (4, 5), march only (6)
constexpr int kFxBarReady = 2, kFxBarFree = 4, kFxBarMarch = 6;
constexpr int kFxHandoff = (kFxEpi + kFxMarch) * 32;
constexpr int kFxMaxSmem = 225 * 1024;  // dynamic (the static barriers and tau table take the rest)

struct FxMaps {
  CUtensorMap dig, psi, phi;
};

__host__ __device__ inline int fx_al128(int b) { return (b + 127) & ~127; }
// bytes of one line buffer: Psi [nx][2 norb] doubles + Phi [nx] complex + B's row scales [80]
__host__ __device__ inline int fx_line_bytes(int nx, int norb) {
  return fx_al128(nx * norb * 16) + fx_al128(nx * 16) + kFxN * 8;
}
static size_t fx_smem(int nx, int norb) { return (size_t)kFxTileB + 2 * fx_line_bytes(nx, norb) + kFxXchB + 1024; }

bool gemm2x_supported(const Geometry& g) {
  return g.i8 && !g.sp && g.nx <= kFxN && g.nx >= 2 && g.norb <= 64 && g.nproj <= 64 &&
         (long long)g.ny * g.nz < (1LL << 31) && fx_smem(g.nx, g.norb) <= (size_t)kFxMaxSmem &&
         (size_t)kFxTileB + (size_t)g.nproj * g.norb * 16 + 1024 <= (size_t)kFxMaxSmem;
}
size_t gemm2x_digit_bytes(const Geometry& g) { return (size_t)g.ndom * g.ny * g.nz * kI8S * g.nx * kFxK; }
size_t gemm2x_sig_bytes(const Geometry& g) { return (size_t)g.ndom * g.ny * g.nz * kFxN * sizeof(double); }

// ---- B's digits in x-line order (once per lfd_init): warp per grid row ------------------------------------
// dig [dom][line][6][nx][128 B] plain (the TMA applies the 128B swizzle), sig [dom][line][80] (0 past nx)
__global__ void __launch_bounds__(256) k_bslicex_i8(const double2* __restrict__ B, int nproj, int nx, int nyz,
                                                    int8_t* __restrict__ out, double* __restrict__ sig) {
  pdl_wait();
  pdl_trigger();
  const int dom = blockIdx.y, lane = threadIdx.x & 31;
  const long long r = (long long)blockIdx.x * 8 + (threadIdx.x >> 5);  // grid row x * nyz + line
  const long long ngp = (long long)nx * nyz;
  if (r >= ngp) return;
  double v[4] = {0.0, 0.0, 0.0, 0.0};
  const int u0 = 2 * lane;
  const double2* row = B + ((long long)dom * ngp + r) * nproj;
  if (u0 < nproj) { const double2 a = row[u0]; v[0] = a.x; v[1] = a.y; }
  if (u0 + 1 < nproj) { const double2 a = row[u0 + 1]; v[2] = a.x; v[3] = a.y; }
  double mx = fmax(fmax(fabs(v[0]), fabs(v[1])), fmax(fabs(v[2]), fabs(v[3])));
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  const int e = mx > 0.0 ? row_exponent(mx) : 0;
  uint32_t d[kI8S];
  digits4(v, e, !(mx > 0.0), d);
  const int x = (int)(r / nyz), line = (int)(r - (long long)x * nyz);
  int8_t* tb = out + ((long long)dom * nyz + line) * kI8S * nx * kFxK + (long long)x * kFxK + 4 * lane;
#pragma unroll
  for (int i = 0; i < kI8S; ++i) *reinterpret_cast<uint32_t*>(tb + (long long)i * nx * kFxK) = d[i];
  if (lane == 0) sig[((long long)dom * nyz + line) * kFxN + x] = mx > 0.0 ? ldexp(1.0, e) : 0.0;
}

cudaError_t launch_bslicex_i8(const Geometry& g, const double2* B, int8_t* dig, double* sig, cudaStream_t st) {
  const int nyz = g.ny * g.nz;
  cudaError_t e = cudaMemsetAsync(sig, 0, gemm2x_sig_bytes(g), st);
  if (e != cudaSuccess) return e;
  dim3 grid((unsigned)((g.ng + 7) / 8), g.ndom);
  launch_k(k_bslicex_i8, grid, 256, 0, st, B, g.nproj, g.nx, nyz, dig, sig);
  return cudaGetLastError();
}

// ---- K_x on lane components ------------------------------------------------------------------------------
// The epilogue lane n = 2 s + c holds component c (0 re, 1 im) of orbital s; z_p, its partner component, is the
// neighbour lane's (shfl_xor 1). For complex w: (w z)_c = w.x z_c + sgn w.y z_p with sgn = -1 (c = 0), +1 (c = 1).
__device__ __forceinline__ double cmul_c(double2 w, double zc, double zp, double sgn) {
  return fma(w.x, zc, sgn * w.y * zp);
}
// K_x of one periodic line (nx even, >= 8) for one orbital, as march_line2 (lfd_march.cuh: two segments marched
// side by side) with explicit shared-memory loads and running store pointers (the generic lambda form recomputed
// the shared-window base and 64-bit addresses every pair)
__device__ __forceinline__ double2 ld_sh2(uint32_t a) {
  double2 v;
  asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "r"(a));
  return v;
}
template <bool kS>
__device__ __forceinline__ void fx_march2(int n, const PairCoef& c, uint32_t l0, uint32_t ls, double2* out,
                                          long long xs) {
  const int PA = (n / 2 + 1) / 2, PB = n / 2 - PA, LA = 2 * PA;
  LineMarch<kS> A, B;
  A.init();
  B.init();
  uint32_t la = l0, lb = l0 + (uint32_t)LA * ls;
  A.first(c, ld_sh2(la), ld_sh2(la + ls));
  B.first(c, ld_sh2(lb), ld_sh2(lb + ls));
  la += 2 * ls;
  lb += 2 * ls;
  A.second(c, ld_sh2(la), ld_sh2(la + ls));
  B.second(c, ld_sh2(lb), ld_sh2(lb + ls));
  la += 2 * ls;
  lb += 2 * ls;
  double2* oa = out + 2 * xs;  // stores of the steady loop at pair p: points 2p-2, 2p-1 (A), LA + 2p-2 .. (B)
  double2* ob = out + (long long)(LA + 2) * xs;
  for (int p = 2; p < PA; ++p) {
    const double2 aa = ld_sh2(la), ab = ld_sh2(la + ls);
    A.steady(c, aa, ab, [&](int k, double2 v) { oa[k * xs] = v; });
    la += 2 * ls;
    oa += 2 * xs;
    if (p < PB) {
      const double2 ba = ld_sh2(lb), bb = ld_sh2(lb + ls);
      B.steady(c, ba, bb, [&](int k, double2 v) { ob[k * xs] = v; });
      lb += 2 * ls;
      ob += 2 * xs;
    }
  }
  const double2 OAl = lk_L<kS>(c.a2, c.u2, A.prev_e1, B.E10);
  const double2 OBf = lk_R<kS>(c.a2, c.d2, A.prev_e1, B.E10);
  const double2 OBl = lk_L<kS>(c.a2, c.u2, B.prev_e1, A.E10);
  const double2 OAf = lk_R<kS>(c.a2, c.d2, B.prev_e1, A.E10);
  out[(long long)(LA - 2) * xs] = lk_L<kS>(c.a1, c.u1, A.prev_oR, OAl);
  out[(long long)(LA - 1) * xs] = lk_R<kS>(c.a1, c.d1, A.prev_oR, OAl);
  out[(long long)(n - 2) * xs] = lk_L<kS>(c.a1, c.u1, B.prev_oR, OBl);
  out[(long long)(n - 1) * xs] = lk_R<kS>(c.a1, c.d1, B.prev_oR, OBl);
  out[0] = lk_L<kS>(c.a1, c.u1, OAf, A.O1);
  out[xs] = lk_R<kS>(c.a1, c.d1, OAf, A.O1);
  out[(long long)LA * xs] = lk_L<kS>(c.a1, c.u1, OBf, B.O1);
  out[(long long)(LA + 1) * xs] = lk_R<kS>(c.a1, c.d1, OBf, B.O1);
}

// ---- the fused kernel ------------------------------------------------------------------------------------
struct FxArgs {
  double2* psi;
  const DomCoef* coef;
  const double* nfac;
  const double2* Cp;
  const double* sig;
  int ndom, nproj, norb, nx, nyz;
  long long ng;
};

template <bool kPer, bool kS>
__global__ void __launch_bounds__(kFxThreads, 1) k_gemm2x_i8(const __grid_constant__ CUtensorMap tDig,
                                                             const __grid_constant__ CUtensorMap tPsi,
                                                             const __grid_constant__ CUtensorMap tPhi, FxArgs p) {
  // programmatic dependent launch: set-up and the first digit tile (B's digits are constant since lfd_init)
  // overlap the previous kernel; every other load waits for it (C'', n, Psi, Phi)
  pdl_trigger();
  extern __shared__ __align__(1024) unsigned char dsm_raw[];
  unsigned char* dsm = dsm_raw + ((1024u - (smem_addr(dsm_raw) & 1023u)) & 1023u);
  const int nx = p.nx, norb = p.norb, nproj = p.nproj, nyz = p.nyz;
  const int psiB = fx_al128(nx * norb * 16), phiB = fx_al128(nx * 16);
  const int lineB = psiB + phiB + kFxN * 8;
  unsigned char* Tsm = dsm;             // [6][80][128 B] digit tile (128B-swizzled)
  unsigned char* Lsm = dsm + kFxTileB;  // 2 line buffers
  auto lpsi = [&](int b) { return reinterpret_cast<double*>(Lsm + b * lineB); };
  auto lphi = [&](int b) { return reinterpret_cast<const double2*>(Lsm + b * lineB + psiB); };
  auto lsig = [&](int b) { return reinterpret_cast<const double*>(Lsm + b * lineB + psiB + phiB); };
  unsigned char* Csm = Lsm;  // C'' of the domain, staged before the first line load
  double2* Xsm = reinterpret_cast<double2*>(Lsm + 2 * lineB);  // march segments' boundary values
  __shared__ __align__(8) uint64_t bfull, bempty, dfull[kFxSlots], dempty[kFxSlots];
  __shared__ __align__(8) uint64_t lfull[2], lempty[2], cbar;
  __shared__ uint32_t tmem_base_sh;
  __shared__ double taus[kI8M];

  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int dom = blockIdx.y;

  if (warp == kFxWMma) {  // TMEM: W^T digits (192 columns) + 4 accumulator slots x 80 columns
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_addr(&tmem_base_sh)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    mbar_init(&bfull, 1);
    mbar_init(&bempty, 1);
    for (int s = 0; s < kFxSlots; ++s) { mbar_init(&dfull[s], 1); mbar_init(&dempty[s], kFxEpi); }
    for (int b = 0; b < 2; ++b) { mbar_init(&lfull[b], 1); mbar_init(&lempty[b], kFxMarch); }
    mbar_init(&cbar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_base_sh;
  const uint32_t tacc = tmem + kFxWCols;
  const long long nlines = nyz;
  if (warp == kFxWMma && lane == 0 && blockIdx.x < nlines) {  // first digit tile, before the dependency wait
    mbar_expect_tx(&bfull, kFxTileB);
    tma_4d(Tsm, &tDig, 0, 0, 0, (int)((long long)dom * nyz + blockIdx.x), &bfull);
  }
  pdl_wait();

  if (warp < kFxEpi) {
    // W^T digits from C'' (one bulk copy into shared memory) into TMEM, as in k_gemm2_i8: thread (warp w, lane)
    // owns row n = 32 (w & 3) + lane of W^T and the 8 columns of chunk c8 = w >> 2 of each digit
    if (tid == 0) {
      mbar_expect_tx(&cbar, (uint32_t)(nproj * norb * 16));
      tma_row(Csm, p.Cp + (long long)dom * nproj * norb, (uint32_t)(nproj * norb * 16), &cbar);
    }
    const int q = warp & 3, c8 = warp >> 2;
    const int n = 32 * q + lane, s = n >> 1, cn = n & 1;
    const bool sv = s < norb;
    mbar_wait(&cbar, 0);
    const double2* X = reinterpret_cast<const double2*>(Csm) + s;
    double mx = 0.0;
    if (sv)
      for (int u = 0; u < nproj; ++u) {
        const double2 x = X[u * norb];
        mx = fmax(mx, fmax(fabs(x.x), fabs(x.y)));
      }
    const int e = mx > 0.0 ? row_exponent(mx) : 0;
    if (c8 == 0) taus[n] = mx > 0.0 ? ldexp(1.0, e - 12) : 0.0;
    const uint32_t trow = tmem + ((uint32_t)(32 * q) << 16);
    uint32_t dg[kI8S][8];
#pragma unroll
    for (int w = 0; w < 8; ++w) {
      double v[4] = {0.0, 0.0, 0.0, 0.0};
      const int u0 = 16 * c8 + 2 * w;
      if (sv && u0 < nproj) {
        const double2 x = X[u0 * norb];
        v[0] = cn ? x.y : x.x; v[1] = cn ? x.x : -x.y;
      }
      if (sv && u0 + 1 < nproj) {
        const double2 x = X[(u0 + 1) * norb];
        v[2] = cn ? x.y : x.x; v[3] = cn ? x.x : -x.y;
      }
      uint32_t d[kI8S];
      digits_i64(v, mx > 0.0 ? ldexp(1.0, 41 - e) : 0.0, d);
#pragma unroll
      for (int i = 0; i < kI8S; ++i) dg[i][w] = d[i];
    }
#pragma unroll
    for (int i = 0; i < kI8S; ++i) tmem_st8(trow + i * 32 + 8 * c8, dg[i]);
    asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
  }
  // W ready and the staged C'' consumed (the line producer then reuses its space)
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  // registers (setmaxnreg, per warpgroup at the top of each role): the epilogue warpgroups hold 20 FP64
  // accumulators + two 16-wide TMEM loads per lane (96); the march and MMA / producer warpgroups need 64

  if (warp < kFxEpi) {
    asm volatile("setmaxnreg.inc.sync.aligned.u32 88;\n" ::: "memory");
    // epilogue: lanes 32 (w & 3) .. (TMEM lane = output double n of a Psi row), x group 20 (w >> 2) ..;
    // diagonals drained two at a time ((P_d 2^7 + P_{d+1}) is an exact int32), then Psi1 = n Psi + sigma tau acc
    // written over the line's staged Psi
    const int q = warp & 3, h = warp >> 2;
    const int n = 32 * q + lane;
    const bool nvalid = n < 2 * norb;
    const double nf = nvalid ? p.nfac[(long long)dom * norb + (n >> 1)] : 0.0;
    const double tau = taus[n];
    const int x0 = kFxXg * h;
    const int nxc = min(max(nx - x0, 0), kFxXg);  // valid x of this warp
    const int ld2 = 2 * norb;
    long long w_d = 0, w_l = 0;
    FX_T0(t_all);
    int it = 0;
    for (long long t = blockIdx.x; t < nlines; t += gridDim.x, ++it) {
      const int b = it & 1;
      double fa[kFxXg];
#pragma unroll
      for (int c = 0; c < kFxXg; ++c) fa[c] = 0.0;
#pragma unroll 1
      for (int dp = 0; dp < kFxAcc / 2; ++dp) {
        const int g = it * kFxAcc + 2 * dp, s0 = g % kFxSlots, s1 = (g + 1) % kFxSlots;
        FX_T0(c3);
        mbar_wait(&dfull[s0], (uint32_t)((g / kFxSlots) & 1));
        mbar_wait(&dfull[s1], (uint32_t)(((g + 1) / kFxSlots) & 1));
        FX_ACC(w_d, c3);
        tc_fence_after();
        const uint32_t lb = ((uint32_t)(32 * q) << 16) + x0;
        const double wd = ldexp(1.0, -14 * dp - 7);
        {  // x 0..15 of the warp's group, then 16..19 (two loads keep the register peak low)
          int32_t a0[16], a1[16];
          tmem_ld16(tacc + s0 * kFxN + lb, a0);
          tmem_ld16(tacc + s1 * kFxN + lb, a1);
          tmem_wait_ld();
          if (dp == 0) {
#pragma unroll
            for (int c = 0; c < 16; ++c) fa[c] = fma(i2d_raw(a0[c] * 128 + a1[c]), wd, -kI2dM * wd);
          } else {
#pragma unroll
            for (int c = 0; c < 16; ++c) fa[c] = fma(i2d(a0[c] * 128 + a1[c]), wd, fa[c]);
          }
        }
        {
          int32_t c0[4], c1[4];
          tmem_ld4(tacc + s0 * kFxN + lb + 16, c0);
          tmem_ld4(tacc + s1 * kFxN + lb + 16, c1);
          tmem_wait_ld();
          if (dp == 0) {
#pragma unroll
            for (int c = 0; c < 4; ++c) fa[16 + c] = fma(i2d_raw(c0[c] * 128 + c1[c]), wd, -kI2dM * wd);
          } else {
#pragma unroll
            for (int c = 0; c < 4; ++c) fa[16 + c] = fma(i2d(c0[c] * 128 + c1[c]), wd, fa[16 + c]);
          }
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {
          mbar_arrive(&dempty[s0]);
          mbar_arrive(&dempty[s1]);
        }
      }
      FX_T0(c4);
      mbar_wait(&lfull[b], (uint32_t)((it >> 1) & 1));
      FX_ACC(w_l, c4);
      // Psi1 = n Psi + sigma tau acc, written over the line's staged Psi for the march warps. The handoffs with the
      // march warps are named barriers (epilogue + march warps): "free" b (the march of line it - 2 is done with
      // the buffer -- also implied by lfull, whose load waited for it) and "ready" b (Psi1 written)
      if (it >= 2) asm volatile("bar.sync %0, %1;" ::"r"(kFxBarFree + b), "n"(kFxHandoff) : "memory");
      if (nvalid) {
        double* ps = lpsi(b) + (long long)x0 * ld2 + n;
        const double* sg = lsig(b) + x0;
#pragma unroll
        for (int c = 0; c < kFxXg; ++c) {
          if (c < nxc) *ps = fma(nf, *ps, fa[c] * (sg[c] * tau));  // (powers of two: exact scaling)
          ps += ld2;
        }
      }
      asm volatile("bar.arrive %0, %1;" ::"r"(kFxBarReady + b), "n"(kFxHandoff) : "memory");
    }
#ifdef LFD_FX_TIMING
    if (warp == 0 && lane == 0 && (blockIdx.x == 0 || blockIdx.x == 100))
      printf("fx cta %d epi0: total %lld wait-diag %lld wait-line %lld\n", blockIdx.x, clock64() - t_all, w_d, w_l);
#endif
    (void)w_d; (void)w_l;
  } else if (warp < kFxEpi + kFxMarch) {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 72;\n" ::: "memory");
    // march warps: thread (segment g, orbital s) streams K_x over segment g of the line for orbital s (Phi . Psi1
    // from shared memory, HBM out); the links across segment ends (and the periodic wrap) are taken after a
    // barrier from the neighbouring segments' first / last E outputs (as finish() takes the wrap of one line).
    // Lines that do not split (zero BC, nx < 12): segment-0 threads march the whole line (march_line).
    const int gi = tid - kFxWMarch0 * 32;
    const int g = gi / 64, s = gi % 64;
    const bool active = s < norb;
    const bool split = kPer && nx >= 4 * kFxSeg;
    const int P = nx / 2;  // pairs (periodic: nx even)
    const int p0 = split ? (g * P) / kFxSeg : 0, p1 = split ? ((g + 1) * P) / kFxSeg : 0;  // this segment's pairs
    const PairCoef cf = pair_coef<kS>(p.coef + dom, 0);
    const long long xs = (long long)nyz * norb;  // element stride between x points
    long long w_r = 0;
    FX_T0(t_all);
    int it = 0;
    for (long long t = blockIdx.x; t < nlines; t += gridDim.x, ++it) {
      const int b = it & 1;
      FX_T0(c5);
      asm volatile("bar.sync %0, %1;" ::"r"(kFxBarReady + b), "n"(kFxHandoff) : "memory");
      FX_ACC(w_r, c5);
      const double2* L = reinterpret_cast<const double2*>(lpsi(b)) + s;
      double2* out = p.psi + ((long long)dom * p.ng + t) * norb + s;
      if (split) {
        LineMarch<kS> M;
        M.init();
        // plain shared-memory loads (ordered by the named barriers' memory clobbers, free to be scheduled early)
        const double2* la = L + (2 * p0) * norb;
        const double2* lf = lphi(b) + 2 * p0;  // Phi (the x pass's pre-phase)
        if (active) {
          M.first(cf, cmul(lf[0], la[0]), cmul(lf[1], la[norb]));
          la += 2 * norb;
          lf += 2;
          M.second(cf, cmul(lf[0], la[0]), cmul(lf[1], la[norb]));
          la += 2 * norb;
          lf += 2;
          double2* o = out + (long long)(2 * p0 + 2) * xs;
#pragma unroll 2
          for (int q = p0 + 2; q < p1; ++q) {
            const double2 a = cmul(lf[0], la[0]), c = cmul(lf[1], la[norb]);
            M.steady(cf, a, c, [&](int k, double2 v) { o[k * xs] = v; });
            la += 2 * norb;
            lf += 2;
            o += 2 * xs;
          }
        }
        double2* xb = Xsm + ((b * kFxSeg + g) * 64 + s) * 2;  // [E output at the first point, at the last point]
        xb[0] = M.E10;
        xb[1] = M.prev_e1;
        asm volatile("bar.sync %0, %1;" ::"n"(kFxBarMarch), "n"(kFxMarch * 32) : "memory");
        if (active) {
          const int gl = g > 0 ? g - 1 : kFxSeg - 1, gr = g + 1 < kFxSeg ? g + 1 : 0;
          const double2 lft = Xsm[((b * kFxSeg + gl) * 64 + s) * 2 + 1];  // left segment's last E output
          const double2 rgt = Xsm[((b * kFxSeg + gr) * 64 + s) * 2];      // right segment's first E output
          const double2 Ol = lk_L<kS>(cf.a2, cf.u2, M.prev_e1, rgt);       // O output at the segment's last point
          const double2 Of = lk_R<kS>(cf.a2, cf.d2, lft, M.E10);           // O output at its first point
          const int e = 2 * p1;
          out[(long long)(e - 2) * xs] = lk_L<kS>(cf.a1, cf.u1, M.prev_oR, Ol);
          out[(long long)(e - 1) * xs] = lk_R<kS>(cf.a1, cf.d1, M.prev_oR, Ol);
          out[(long long)(2 * p0) * xs] = lk_L<kS>(cf.a1, cf.u1, Of, M.O1);
          out[(long long)(2 * p0 + 1) * xs] = lk_R<kS>(cf.a1, cf.d1, Of, M.O1);
        }
      } else if (g == 0 && active) {
        const double2* ph = lphi(b);
        march_line<kPer, kS, double2, double2>(
            nx, cf, [&](int i) { return cmul(ph[i], L[i * norb]); }, [&](int i, double2 v) { out[i * xs] = v; });
      }
      __syncwarp();
      if (lane == 0) mbar_arrive(&lempty[b]);  // the line producer may reload the buffer
      if (t + 2 * (long long)gridDim.x < nlines)  // the epilogue syncs on this for line it + 2
        asm volatile("bar.arrive %0, %1;" ::"r"(kFxBarFree + b), "n"(kFxHandoff) : "memory");
    }
#ifdef LFD_FX_TIMING
    if (tid == kFxWMarch0 * 32 && (blockIdx.x == 0 || blockIdx.x == 100))
      printf("fx cta %d march: total %lld wait-ready %lld\n", blockIdx.x, clock64() - t_all, w_r);
#endif
    (void)w_r;
  } else {
    asm volatile("setmaxnreg.dec.sync.aligned.u32 56;\n" ::: "memory");
    if (warp == kFxWLine) {  // the line: Psi [nx][2 norb], Phi [nx], B's row scales
      if (lane == 0) {
        long long w_m = 0;
        int it = 0;
        for (long long t = blockIdx.x; t < nlines; t += gridDim.x, ++it) {
          const int b = it & 1;
          FX_T0(c6);
          if (it >= 2) mbar_wait(&lempty[b], (uint32_t)(((it >> 1) - 1) & 1));
          FX_ACC(w_m, c6);
          mbar_expect_tx(&lfull[b], (uint32_t)(nx * norb * 16 + nx * 16 + kFxN * 8));
          tma_4d(lpsi(b), &tPsi, 0, (int)t, 0, dom, &lfull[b]);
          tma_4d(const_cast<double2*>(lphi(b)), &tPhi, 0, (int)t, 0, dom, &lfull[b]);
          tma_row(const_cast<double*>(lsig(b)), p.sig + ((long long)dom * nyz + t) * kFxN, kFxN * 8, &lfull[b]);
        }
  #ifdef LFD_FX_TIMING
        if (blockIdx.x == 0 || blockIdx.x == 100) printf("fx cta %d line: wait-empty %lld\n", blockIdx.x, w_m);
  #endif
        (void)w_m;
      }
    } else if (warp == kFxWMma) {  // D_d += W_j^T (TMEM) x b_i (smem), i + j = d; one ring slot per diagonal
      const uint64_t db0 = umma_desc_sw128(smem_addr(Tsm));
      long long w_b = 0, w_s = 0, w_e = 0;
      FX_T0(t_all);
      int it = 0;
      for (long long t = blockIdx.x; t < nlines; t += gridDim.x, ++it) {
        FX_T0(c0);
        mbar_wait(&bfull, (uint32_t)(it & 1));
        FX_ACC(w_b, c0);
        tc_fence_after();
#pragma unroll
        for (int d = 2; d <= kI8S + 1; ++d) {
          const int g = it * kFxAcc + (d - 2), sl = g % kFxSlots;
          if (g >= kFxSlots) {
            FX_T0(c1);
            mbar_wait(&dempty[sl], (uint32_t)(((g / kFxSlots) - 1) & 1));
            FX_ACC(w_s, c1);
            tc_fence_after();
          }
          const uint32_t acc = tacc + sl * kFxN;
          uint32_t accum = 0;  // 0 for the diagonal's first MMA
#pragma unroll
          for (int i = 1; i <= kI8S; ++i) {
            const int j = d - i;
            if (j < 1 || j > kI8S) continue;
            uint64_t db = db0 + (uint64_t)(((i - 1) * kFxSliceB) >> 4);
            uint32_t ta = tmem + (j - 1) * 32;
#pragma unroll 1
            for (int kk = 0; kk < kFxK / 32; ++kk) {  // (not unrolled: the 64-register warpgroup)
              umma_i8_ts(acc, ta, db, accum, i8_idesc(kFxN));
              accum = 1;
              db += 2;  // 32 bytes >> 4
              ta += 8;
            }
          }
          umma_commit(&dfull[sl]);
        }
        umma_commit(&bempty);  // the digit tile may be overwritten once these MMAs are done
        const long long tn = t + gridDim.x;
        if (tn < nlines) {  // the next line's digit tile
          FX_T0(c2);
          mbar_wait(&bempty, (uint32_t)(it & 1));
          FX_ACC(w_e, c2);
          if (lane == 0) {
            mbar_expect_tx(&bfull, kFxTileB);
            tma_4d(Tsm, &tDig, 0, 0, 0, (int)((long long)dom * nyz + tn), &bfull);
          }
          __syncwarp();
        }
      }
  #ifdef LFD_FX_TIMING
      if (lane == 0 && (blockIdx.x == 0 || blockIdx.x == 100))
        printf("fx cta %d mma: total %lld wait-digits %lld wait-slot %lld wait-mma-done %lld lines %d\n", blockIdx.x,
               clock64() - t_all, w_b, w_s, w_e, it);
  #endif
      (void)w_b; (void)w_s; (void)w_e;
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == kFxWMma) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
  }
}

FxMaps* gemm2x_maps_create(const Geometry& g, const int8_t* dig, double2* psi, const double2* phi) {
  FxMaps* m = new (std::nothrow) FxMaps;
  if (!m) return nullptr;
  const uint64_t nyz = (uint64_t)g.ny * g.nz;
  // digits [dom*nyz lines][6][nx][128 B], box [1][6][80][128] with the 128B swizzle (x rows past nx zero)
  const uint64_t dd[4] = {(uint64_t)kFxK, (uint64_t)g.nx, (uint64_t)kI8S, (uint64_t)g.ndom * nyz};
  const uint64_t sd[3] = {(uint64_t)kFxK, (uint64_t)g.nx * kFxK, (uint64_t)kI8S * g.nx * kFxK};
  const uint32_t bd[4] = {(uint32_t)kFxK, (uint32_t)kFxN, (uint32_t)kI8S, 1};
  // Psi as doubles [dom][x][yz][2 norb], box [1][nx][1][2 norb]: the line (y, z) of all orbitals
  const uint64_t dp[4] = {(uint64_t)2 * g.norb, nyz, (uint64_t)g.nx, (uint64_t)g.ndom};
  const uint64_t sp[3] = {(uint64_t)g.norb * 16, nyz * g.norb * 16, (uint64_t)g.ng * g.norb * 16};
  const uint32_t bp[4] = {(uint32_t)(2 * g.norb), 1, (uint32_t)g.nx, 1};
  // Phi as doubles [dom][x][yz][2], box [1][nx][1][2]
  const uint64_t df[4] = {2, nyz, (uint64_t)g.nx, (uint64_t)g.ndom};
  const uint64_t sf[3] = {16, nyz * 16, (uint64_t)g.ng * 16};
  const uint32_t bf[4] = {2, 1, (uint32_t)g.nx, 1};
  if (encode_tmap(&m->dig, CU_TENSOR_MAP_DATA_TYPE_UINT8, 4, dig, dd, sd, bd, CU_TENSOR_MAP_SWIZZLE_128B) !=
          cudaSuccess ||
      encode_tmap(&m->psi, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, psi, dp, sp, bp, CU_TENSOR_MAP_SWIZZLE_NONE) !=
          cudaSuccess ||
      encode_tmap(&m->phi, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, phi, df, sf, bf, CU_TENSOR_MAP_SWIZZLE_NONE) !=
          cudaSuccess) {
    delete m;
    return nullptr;
  }
  return m;
}

void gemm2x_maps_destroy(FxMaps* m) { delete m; }

cudaError_t launch_gemm2x_i8(const Geometry& g, const FxMaps* m, double2* psi, const DomCoef* coef, const double* nfac,
                             const double2* Cp, const double* sig, bool scaled, int num_sms, cudaStream_t st) {
  FxArgs a;
  a.psi = psi; a.coef = coef; a.nfac = nfac; a.Cp = Cp; a.sig = sig;
  a.ndom = g.ndom; a.nproj = g.nproj; a.norb = g.norb; a.nx = g.nx; a.nyz = g.ny * g.nz; a.ng = g.ng;
  int cpd = num_sms / g.ndom;
  if (cpd < 1) cpd = 1;
  if (cpd > a.nyz) cpd = a.nyz;
  dim3 grid(cpd, g.ndom);
  // the C'' staging (nproj x norb complex) lives in the line-buffer region before the first line load
  const size_t sm = std::max(fx_smem(g.nx, g.norb), (size_t)kFxTileB + (size_t)g.nproj * g.norb * 16 + 1024);
  if (g.bc == 0) {
    if (scaled) launch_k(k_gemm2x_i8<true, true>, grid, kFxThreads, sm, st, m->dig, m->psi, m->phi, a);
    else launch_k(k_gemm2x_i8<true, false>, grid, kFxThreads, sm, st, m->dig, m->psi, m->phi, a);
  } else {
    if (scaled) launch_k(k_gemm2x_i8<false, true>, grid, kFxThreads, sm, st, m->dig, m->psi, m->phi, a);
    else launch_k(k_gemm2x_i8<false, false>, grid, kFxThreads, sm, st, m->dig, m->psi, m->phi, a);
  }
  return cudaGetLastError();
}

cudaError_t gemm2x_set_attributes() {
  for (auto f : {k_gemm2x_i8<true, true>, k_gemm2x_i8<true, false>, k_gemm2x_i8<false, true>,
                 k_gemm2x_i8<false, false>}) {
    cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, kFxMaxSmem);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

}  // namespace lfd
