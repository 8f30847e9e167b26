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
constexpr int kFxSlots = 4;                  // TMEM ring of diagonal accumulators (80 columns each)
// shapes by the digit count S (6 for FP64 contexts, 4 for the SP variant)
template <int S>
struct FxG {
  static constexpr int TileB = S * kFxSliceB;     // 60 KB / 40 KB
  static constexpr int WCols = S * (kFxK / 4);    // TMEM columns of W^T digits
  static constexpr int Acc = S;                   // diagonals d = 2 .. S+1
};
constexpr int fx_digits(bool sp) { return sp ? 4 : kI8S; }
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
constexpr int kFxMaxSmem = 225 * 1024;  // dynamic (the static barriers, tau table and coefficients take the rest)

struct FxMaps {
  CUtensorMap dig, psi, phi;
};

__host__ __device__ inline int fx_al128(int b) { return (b + 127) & ~127; }
// bytes of one line buffer: Psi [nx][norb] complex (esz bytes each) + Phi [nx] x 16 bytes (complex128, or two
// complex64: the TMA box needs 16 bytes) + B's row scales [80]
__host__ __device__ inline int fx_line_bytes(int nx, int norb, int esz) {
  return fx_al128(nx * norb * esz) + fx_al128(nx * 16) + kFxN * 8;
}
static size_t fx_smem(int nx, int norb, bool sp) {
  return (size_t)fx_digits(sp) * kFxSliceB + 2 * fx_line_bytes(nx, norb, sp ? 8 : 16) + kFxXchB + 1024;
}

bool gemm2x_supported(const Geometry& g) {
  const size_t tile = (size_t)fx_digits(g.sp) * kFxSliceB;
  // (complex64: TMA strides of 16-byte multiples -- norb even, and ny nz even for the Phi map)
  return g.i8 && g.nx <= kFxN && g.nx >= 2 && g.norb <= 64 && g.nproj <= 64 &&
         (!g.sp || (g.norb % 2 == 0 && (g.ny * g.nz) % 2 == 0)) &&
         (long long)g.ny * g.nz < (1LL << 31) && fx_smem(g.nx, g.norb, g.sp) <= (size_t)kFxMaxSmem &&
         tile + (size_t)g.nproj * g.norb * 16 + 1024 <= (size_t)kFxMaxSmem;
}
size_t gemm2x_digit_bytes(const Geometry& g) {
  return (size_t)g.ndom * g.ny * g.nz * fx_digits(g.sp) * g.nx * kFxK;
}
size_t gemm2x_sig_bytes(const Geometry& g) { return (size_t)g.ndom * g.ny * g.nz * kFxN * sizeof(double); }

// ---- B's digits in x-line order (once per lfd_init): warp per grid row ------------------------------------
// dig [dom][line][S][nx][128 B] plain (the TMA applies the 128B swizzle), sig [dom][line][80] (0 past nx)
template <class T, int S>
__global__ void __launch_bounds__(256) k_bslicex_i8(const T* __restrict__ B, int nproj, int nx, int nyz,
                                                    int8_t* __restrict__ out, double* __restrict__ sig) {
  pdl_wait();
  pdl_trigger();
  const int dom = blockIdx.y, lane = threadIdx.x & 31;
  const long long r = (long long)blockIdx.x * 8 + (threadIdx.x >> 5);  // grid row x * nyz + line
  const long long ngp = (long long)nx * nyz;
  if (r >= ngp) return;
  double v[4] = {0.0, 0.0, 0.0, 0.0};
  const int u0 = 2 * lane;
  const T* row = B + ((long long)dom * ngp + r) * nproj;
  if (u0 < nproj) { const T a = row[u0]; v[0] = a.x; v[1] = a.y; }
  if (u0 + 1 < nproj) { const T a = row[u0 + 1]; v[2] = a.x; v[3] = a.y; }
  double mx = fmax(fmax(fabs(v[0]), fabs(v[1])), fmax(fabs(v[2]), fabs(v[3])));
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  const int e = mx > 0.0 ? row_exponent(mx) : 0;
  uint32_t d[S];
  digits4<S>(v, e, !(mx > 0.0), d);
  const int x = (int)(r / nyz), line = (int)(r - (long long)x * nyz);
  int8_t* tb = out + ((long long)dom * nyz + line) * S * nx * kFxK + (long long)x * kFxK + 4 * lane;
#pragma unroll
  for (int i = 0; i < S; ++i) *reinterpret_cast<uint32_t*>(tb + (long long)i * nx * kFxK) = d[i];
  if (lane == 0) sig[((long long)dom * nyz + line) * kFxN + x] = mx > 0.0 ? ldexp(1.0, e) : 0.0;
}

cudaError_t launch_bslicex_i8(const Geometry& g, const void* B, int8_t* dig, double* sig, cudaStream_t st) {
  const int nyz = g.ny * g.nz;
  cudaError_t e = cudaMemsetAsync(sig, 0, gemm2x_sig_bytes(g), st);
  if (e != cudaSuccess) return e;
  dim3 grid((unsigned)((g.ng + 7) / 8), g.ndom);
  if (g.sp)
    launch_k(k_bslicex_i8<float2, 4>, grid, 256, 0, st, static_cast<const float2*>(B), g.nproj, g.nx, nyz, dig, sig);
  else
    launch_k(k_bslicex_i8<double2, kI8S>, grid, 256, 0, st, static_cast<const double2*>(B), g.nproj, g.nx, nyz, dig, sig);
  return cudaGetLastError();
}

// ---- the fused kernel ------------------------------------------------------------------------------------
struct FxArgs {
  void* psi;  // complex128, or complex64 (SP)
  const DomCoef* coef;
  const double* nfac;
  const double2* Cp;
  const double* sig;
  int ndom, nproj, norb, nx, nyz;
  long long ng;
};

// T = double2 (S = 6 digits) or float2 (the SP variant: S = 4 digits, complex64 Psi, the march in FP32)
template <bool kPer, bool kS, class T = double2, int S = kI8S>
__global__ void __launch_bounds__(kFxThreads, 1) k_gemm2x_i8(const __grid_constant__ CUtensorMap tDig,
                                                             const __grid_constant__ CUtensorMap tPsi,
                                                             const __grid_constant__ CUtensorMap tPhi, FxArgs p) {
  // programmatic dependent launch: set-up and the first digit tile (B's digits are constant since lfd_init)
  // overlap the previous kernel; every other load waits for it (C'', n, Psi, Phi)
  pdl_trigger();
  extern __shared__ __align__(1024) unsigned char dsm_raw[];
  unsigned char* dsm = dsm_raw + ((1024u - (smem_addr(dsm_raw) & 1023u)) & 1023u);
  using R = decltype(T::x);  // real component type of Psi
  constexpr int kTileB = FxG<S>::TileB, kWCols = FxG<S>::WCols, kAcc = FxG<S>::Acc;
  constexpr int kPhiStep = sizeof(T) == 8 ? 2 : 1;  // complex64 Phi staged two lines at a time (16-byte box)
  const int nx = p.nx, norb = p.norb, nproj = p.nproj, nyz = p.nyz;
  const int psiB = fx_al128(nx * norb * (int)sizeof(T)), phiB = fx_al128(nx * 16);
  const int lineB = psiB + phiB + kFxN * 8;
  unsigned char* Tsm = dsm;           // [S][80][128 B] digit tile (128B-swizzled)
  unsigned char* Lsm = dsm + kTileB;  // 2 line buffers
  auto lpsi = [&](int b) { return reinterpret_cast<R*>(Lsm + b * lineB); };
  auto lphi = [&](int b) { return reinterpret_cast<const T*>(Lsm + b * lineB + psiB); };  // Phi(x) at [x kPhiStep]
  auto lsig = [&](int b) { return reinterpret_cast<const double*>(Lsm + b * lineB + psiB + phiB); };
  unsigned char* Csm = Lsm;  // C'' of the domain, staged before the first line load
  T* Xsm = reinterpret_cast<T*>(Lsm + 2 * lineB);  // march segments' boundary values
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
  const uint32_t tacc = tmem + kWCols;
  const long long nlines = nyz;
  if (warp == kFxWMma && lane == 0 && blockIdx.x < nlines) {  // first digit tile, before the dependency wait
    mbar_expect_tx(&bfull, kTileB);
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
    uint32_t dg[S][8];
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
      uint32_t d[S];
      digits_x<S>(v, mx > 0.0 ? ldexp(1.0, 7 * S - 1 - e) : 0.0, d);
#pragma unroll
      for (int i = 0; i < S; ++i) dg[i][w] = d[i];
    }
#pragma unroll
    for (int i = 0; i < S; ++i) tmem_st8(trow + i * 32 + 8 * c8, dg[i]);
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
#pragma unroll  // (unrolled: 223 -> 221 us; in k_gemm2_i8 the same unroll took 174 -> 165 us)
      for (int dp = 0; dp < kAcc / 2; ++dp) {
        const int g = it * kAcc + 2 * dp, s0 = g % kFxSlots, s1 = (g + 1) % kFxSlots;
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
        R* ps = lpsi(b) + (long long)x0 * ld2 + n;
        const double* sg = lsig(b) + x0;
#pragma unroll
        for (int c = 0; c < kFxXg; ++c) {
          if (c < nxc) *ps = (R)fma(nf, (double)*ps, fa[c] * (sg[c] * tau));  // (powers of two: exact scaling)
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
    const PairCoefT<T> cf = pair_coef_t<kS, T>(p.coef + dom, 0);  // (complex64: rounded once from FP64)
    const long long xs = (long long)nyz * norb;  // element stride between x points
    long long w_r = 0;
    FX_T0(t_all);
    int it = 0;
    for (long long t = blockIdx.x; t < nlines; t += gridDim.x, ++it) {
      const int b = it & 1;
      FX_T0(c5);
      asm volatile("bar.sync %0, %1;" ::"r"(kFxBarReady + b), "n"(kFxHandoff) : "memory");
      FX_ACC(w_r, c5);
      const T* L = reinterpret_cast<const T*>(lpsi(b)) + s;
      T* out = static_cast<T*>(p.psi) + ((long long)dom * p.ng + t) * norb + s;
      if (split) {
        LineMarch<kS, T, T> M;
        M.init();
        // plain shared-memory loads (ordered by the named barriers' memory clobbers, free to be scheduled early)
        const T* la = L + (2 * p0) * norb;
        const T* lf = lphi(b) + 2 * p0 * kPhiStep + (kPhiStep == 2 ? (int)(t & 1) : 0);  // Phi (the pre-phase)
        if (active) {
          M.first(cf, cmul(lf[0], la[0]), cmul(lf[kPhiStep], la[norb]));
          la += 2 * norb;
          lf += 2 * kPhiStep;
          M.second(cf, cmul(lf[0], la[0]), cmul(lf[kPhiStep], la[norb]));
          la += 2 * norb;
          lf += 2 * kPhiStep;
          T* o = out + (long long)(2 * p0 + 2) * xs;
#pragma unroll(sizeof(T) == 16 ? 2 : 1)  // measured: FP64 217.6 vs 231.2 us unrolled by 2 vs 1, SP 135.8 vs 132.2
          for (int q = p0 + 2; q < p1; ++q) {
            const T a = cmul(lf[0], la[0]), c = cmul(lf[kPhiStep], la[norb]);
            M.steady(cf, a, c, [&](int k, T v) { o[k * xs] = v; });
            la += 2 * norb;
            lf += 2 * kPhiStep;
            o += 2 * xs;
          }
        }
        T* xb = Xsm + ((b * kFxSeg + g) * 64 + s) * 2;  // [E output at the first point, at the last point]
        xb[0] = M.E10;
        xb[1] = M.prev_e1;
        asm volatile("bar.sync %0, %1;" ::"n"(kFxBarMarch), "n"(kFxMarch * 32) : "memory");
        if (active) {
          const int gl = g > 0 ? g - 1 : kFxSeg - 1, gr = g + 1 < kFxSeg ? g + 1 : 0;
          const T lft = Xsm[((b * kFxSeg + gl) * 64 + s) * 2 + 1];  // left segment's last E output
          const T rgt = Xsm[((b * kFxSeg + gr) * 64 + s) * 2];      // right segment's first E output
          const T Ol = lk_L<kS>(cf.a2, cf.u2, M.prev_e1, rgt);       // O output at the segment's last point
          const T Of = lk_R<kS>(cf.a2, cf.d2, lft, M.E10);           // O output at its first point
          const int e = 2 * p1;
          out[(long long)(e - 2) * xs] = lk_L<kS>(cf.a1, cf.u1, M.prev_oR, Ol);
          out[(long long)(e - 1) * xs] = lk_R<kS>(cf.a1, cf.d1, M.prev_oR, Ol);
          out[(long long)(2 * p0) * xs] = lk_L<kS>(cf.a1, cf.u1, Of, M.O1);
          out[(long long)(2 * p0 + 1) * xs] = lk_R<kS>(cf.a1, cf.d1, Of, M.O1);
        }
      } else if (g == 0 && active) {
        const T* ph = lphi(b) + (kPhiStep == 2 ? (int)(t & 1) : 0);
        march_line<kPer, kS, T, T>(
            nx, cf, [&](int i) { return cmul(ph[i * kPhiStep], L[i * norb]); }, [&](int i, T v) { out[i * xs] = v; });
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
          mbar_expect_tx(&lfull[b], (uint32_t)(nx * norb * (int)sizeof(T) + nx * 16 + kFxN * 8));
          tma_4d(lpsi(b), &tPsi, 0, (int)t, 0, dom, &lfull[b]);
          if (sizeof(T) == 16) tma_4d(const_cast<T*>(lphi(b)), &tPhi, 0, (int)t, 0, dom, &lfull[b]);
          else tma_4d(const_cast<T*>(lphi(b)), &tPhi, (int)(t & ~1LL), 0, dom, 0, &lfull[b]);  // (16-byte aligned)
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
        // (the issuing warp shares its sub-partition with epilogue and march warps: every MMA issue instruction
        // counts -- the K loop unrolled, and for S = 6 the diagonals too: C2 231 -> 219 us; for S = 4 rolled
        // diagonals measured faster, 143 vs 137 us)
#pragma unroll(S == 6 ? S : 1)
        for (int d = 2; d <= S + 1; ++d) {
          const int g = it * kAcc + (d - 2), sl = g % kFxSlots;
          if (g >= kFxSlots) {
            FX_T0(c1);
            mbar_wait(&dempty[sl], (uint32_t)(((g / kFxSlots) - 1) & 1));
            FX_ACC(w_s, c1);
            tc_fence_after();
          }
          const uint32_t acc = tacc + sl * kFxN;
          uint32_t accum = 0;  // 0 for the diagonal's first MMA
#pragma unroll
          for (int i = 1; i <= S; ++i) {
            const int j = d - i;
            if (j < 1 || j > S) continue;
            uint64_t db = db0 + (uint64_t)(((i - 1) * kFxSliceB) >> 4);
            uint32_t ta = tmem + (j - 1) * 32;
#pragma unroll
            for (int kk = 0; kk < kFxK / 32; ++kk) {
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
            mbar_expect_tx(&bfull, kTileB);
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

FxMaps* gemm2x_maps_create(const Geometry& g, const int8_t* dig, void* psi, const void* phi) {
  FxMaps* m = new (std::nothrow) FxMaps;
  if (!m) return nullptr;
  const uint64_t nyz = (uint64_t)g.ny * g.nz, S = (uint64_t)fx_digits(g.sp);
  // digits [dom*nyz lines][S][nx][128 B], box [1][S][80][128] with the 128B swizzle (x rows past nx zero)
  const uint64_t dd[4] = {(uint64_t)kFxK, (uint64_t)g.nx, S, (uint64_t)g.ndom * nyz};
  const uint64_t sd[3] = {(uint64_t)kFxK, (uint64_t)g.nx * kFxK, S * g.nx * kFxK};
  const uint32_t bd[4] = {(uint32_t)kFxK, (uint32_t)kFxN, (uint32_t)S, 1};
  // Psi as 8-byte elements [dom][x][yz][E norb] (E = 2 doubles per complex128, 1 per complex64), box [1][nx][1][E norb]:
  // the line (y, z) of all orbitals
  const uint64_t E = g.sp ? 1 : 2, esz = g.sp ? 8 : 16;
  const uint64_t dp[4] = {E * g.norb, nyz, (uint64_t)g.nx, (uint64_t)g.ndom};
  const uint64_t sp[3] = {(uint64_t)g.norb * esz, nyz * g.norb * esz, (uint64_t)g.ng * g.norb * esz};
  const uint32_t bp[4] = {(uint32_t)(E * g.norb), 1, (uint32_t)g.nx, 1};
  // Phi: complex128 [dom][x][yz][2 doubles], box [1][nx][1][2]; complex64 [1][dom][x][yz] (8-byte elements), box
  // [1][1][nx][2]: the line pair (2k, 2k + 1) holding the line (a 16-byte box that starts 16-byte aligned)
  const uint64_t df[4] = {2, nyz, (uint64_t)g.nx, (uint64_t)g.ndom};
  const uint64_t sf[3] = {16, nyz * 16, (uint64_t)g.ng * 16};
  const uint32_t bf[4] = {2, 1, (uint32_t)g.nx, 1};
  const uint64_t df32[4] = {nyz, (uint64_t)g.nx, (uint64_t)g.ndom, 1};
  const uint64_t sf32[3] = {nyz * 8, (uint64_t)g.ng * 8, (uint64_t)g.ndom * g.ng * 8};
  const uint32_t bf32[4] = {2, (uint32_t)g.nx, 1, 1};
  if (encode_tmap(&m->dig, CU_TENSOR_MAP_DATA_TYPE_UINT8, 4, dig, dd, sd, bd, CU_TENSOR_MAP_SWIZZLE_128B) !=
          cudaSuccess ||
      encode_tmap(&m->psi, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, psi, dp, sp, bp, CU_TENSOR_MAP_SWIZZLE_NONE) !=
          cudaSuccess ||
      encode_tmap(&m->phi, CU_TENSOR_MAP_DATA_TYPE_FLOAT64, 4, phi, g.sp ? df32 : df, g.sp ? sf32 : sf,
                  g.sp ? bf32 : bf, CU_TENSOR_MAP_SWIZZLE_NONE) != cudaSuccess) {
    delete m;
    return nullptr;
  }
  return m;
}

void gemm2x_maps_destroy(FxMaps* m) { delete m; }

cudaError_t launch_gemm2x_i8(const Geometry& g, const FxMaps* m, void* psi, const DomCoef* coef, const double* nfac,
                             const double2* Cp, const double* sig, bool scaled, int num_sms, cudaStream_t st) {
  FxArgs a;
  a.psi = psi; a.coef = coef; a.nfac = nfac; a.Cp = Cp; a.sig = sig;
  a.ndom = g.ndom; a.nproj = g.nproj; a.norb = g.norb; a.nx = g.nx; a.nyz = g.ny * g.nz; a.ng = g.ng;
  int cpd = num_sms / g.ndom;
  if (cpd < 1) cpd = 1;
  if (cpd > a.nyz) cpd = a.nyz;
  dim3 grid(cpd, g.ndom);
  // the C'' staging (nproj x norb complex128) lives in the line-buffer region before the first line load
  const size_t sm = std::max(fx_smem(g.nx, g.norb, g.sp),
                             (size_t)fx_digits(g.sp) * kFxSliceB + (size_t)g.nproj * g.norb * 16 + 1024);
#define LFD_FX(P, K)                                                                                             \
  (g.sp ? launch_k(k_gemm2x_i8<P, K, float2, 4>, grid, kFxThreads, sm, st, m->dig, m->psi, m->phi, a)         \
        : launch_k(k_gemm2x_i8<P, K, double2, kI8S>, grid, kFxThreads, sm, st, m->dig, m->psi, m->phi, a))
  if (g.bc == 0) {
    if (scaled) LFD_FX(true, true); else LFD_FX(true, false);
  } else {
    if (scaled) LFD_FX(false, true); else LFD_FX(false, false);
  }
#undef LFD_FX
  return cudaGetLastError();
}

cudaError_t gemm2x_set_attributes() {
  for (auto f : {k_gemm2x_i8<true, true, double2, kI8S>, k_gemm2x_i8<true, false, double2, kI8S>,
                 k_gemm2x_i8<false, true, double2, kI8S>, k_gemm2x_i8<false, false, double2, kI8S>,
                 k_gemm2x_i8<true, true, float2, 4>, k_gemm2x_i8<true, false, float2, 4>,
                 k_gemm2x_i8<false, true, float2, 4>, k_gemm2x_i8<false, false, float2, 4>}) {
    cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, kFxMaxSmem);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

}  // namespace lfd
