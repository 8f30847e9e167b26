// nl_i8.cu -- the projector GEMMs of the nonlocal factor (Eq. 9 / P:210) on the
// tcgen05 tensor cores with (emulated) FP64 accuracy: the FP64 operands are split exactly into int8 digit
// slices (an Ozaki-type scheme), the digit products run as tcgen05.mma kind::i8 with exact int32
// accumulation in TMEM, and the epilogues recombine them in FP64. GEMM-2 first, GEMM-1 further down.
//
//   Psi[r][s] <- n_s Psi[r][s] + sum_u B[r][u] X[u][s]          (X = C'' = C' diag(n), nl.cu)
//
// Real form. With n = 2s + c (Psi's interleaved re/im doubles) and k = 2u + c' (B's), the complex product
// is one real GEMM out[r][n] = sum_k Bre[r][k] W[k][n], W[2u][2s] = Re X, W[2u+1][2s] = -Im X,
// W[2u][2s+1] = Im X, W[2u+1][2s+1] = Re X (K = 2 nproj <= 128, N = 2 norb <= 128).
//
// Digits. Every row r of B (over k) and every column n of W (over k) gets a power-of-two scale
// sigma_r = 2^e (max_k |B[r][k]| < 2^e), and x = B / sigma_r in (-1, 1) is written exactly as
//   x = sum_{i=1..S} d_i 2^{-6-7(i-1)} + rest,  d_1 = rint(64 x),  d_{i+1} = rint(128 (residual_i)),
// |d_i| <= 64, |rest| <= 2^{-7S-1} (each step is exact in FP64: scaling by powers of two and subtracting
// an integer). The same for W with tau_n. Then
//   out[r][n] ~= sigma_r tau_n sum_{d=2..S+1} 2^{-12-7(d-2)} P_d[r][n],  P_d = sum_{i+j=d} sum_k b_i w_j,
// and each P_d is an exact int32 sum (|P_d| <= 6 * 128 * 64 * 64 < 2^22). The terms dropped (i+j > S+1)
// and the digit remainders are O(2^-42) relative to sigma_r tau_n: with S = 6 the product is accurate to
// ~1e-12 relative (tools/i8_model.py), and since the update B X is O(eps = Delta Delta_sci / 2 ~ 1.4e-3)
// of Psi, the error on Psi per factor is ~1e-15 -- the north star's 1e-10 after 100 steps holds with a
// wide margin (tests/test_gpu_i8.py checks the same bound as the FP64 path).
//
// Kernel (B200-first). The B digits are built ONCE at lfd_init (B is constant: P:216's resident Psi_u(0))
// into tiles of 64 grid points, each tile [S][64 rows][128 B] already in the canonical K-major SWIZZLE_128B
// shared-memory image, so one cp.async.bulk per tile stages it (2-stage ring), plus the row scales sigma_r.
// Per call every CTA builds the W digits (S x 16 KB) from C'' (one bulk copy) straight into TMEM
// (tcgen05.st), where they are the MMA's A operand. Transposed MMA: D[n][r] = sum_k W^T[n][k] b[r][k]
// (M = 128 output doubles n on the TMEM lanes, N = 64 grid points), so each epilogue lane owns one Psi double
// n of a row. Roles: warp 16 = producer of the digit tiles, warp 18 = producer of the tile's Psi rows and
// their sigma_r (16-row sub-tiles, contiguous in HBM, one bulk copy each into a 7-slot ring), warp 17 = MMA
// issuer (the 21 digit pairs x 4 K-steps of a tile into S diagonal accumulators d = i + j, each in a slot of
// a TMEM ring of (512 - 32 S) / 64 slots), warps 0-15 = epilogue (4 TMEM lane quarters x 4 row quarters:
// tcgen05.ld of the diagonals two at a time, (P_d 2^7 + P_{d+1}) exact in int32, FP64 recombination with
// the scales applied by exponent arithmetic, Psi <- n_s Psi + sigma_r tau_n acc stored to HBM). The epilogue
// releases each accumulator slot as soon as it is in registers, so the MMAs run up to a ring ahead of it.
// S = 6 for FP64 contexts, 4 for the SP variant (complex64 Psi, float epilogue stores).
// GEMM-1 (below) uses a different, base-256 digit scheme; the first nonlocal factor's GEMM-2 fused with
// the x pass is nl_fx.cu.
#include "lfd_internal.h"
#include "lfd_tc.cuh"
#include "lfd_tma.cuh"

#include <type_traits>
#ifdef LFD_G1_TIMING
#include <cstdio>
#endif

namespace lfd {

// Role-wait instrumentation of k_gemm1_i8 for A/B experiments only (compiled in with -DLFD_G1_TIMING; printf
// from two CTAs)
#ifdef LFD_G1_TIMING
#define G1_T0(v) long long v = clock64()
#define G1_ACC(acc, v) acc += clock64() - v
#else
#define G1_T0(v)
#define G1_ACC(acc, v)
#endif

constexpr int kI8NT = 64;                           // grid points per tile (MMA N)
constexpr int kI8K = 128;                           // bytes per digit row: K = 2 nproj padded to 128
constexpr int kI8Stages = 2;                        // digit-tile ring
constexpr int kI8EpiWarps = 16;                     // epilogue warps: 4 lane quarters x 4 row quarters
constexpr int kI8Rows = kI8NT / 4;                  // tile rows per epilogue warp
constexpr int kI8SliceB = kI8NT * kI8K;             // 8 KB: one digit slice of a tile
constexpr int kI8SubR = 16;                         // Psi rows per staged sub-tile (= rows per epilogue warp)
constexpr int kI8PsiSlots = 7;                      // Psi sub-tile ring (the first 64 KB also stage C'')
// Shapes depending on the digit count S (6: FP64 contexts, 4: the SP variant) and the element type T of Psi
// (double2 / float2): digit tile, TMEM columns of W^T (4 int8 per column), diagonal accumulators d = 2 .. S+1 and
// the TMEM ring of them, the staged Psi sub-tile
template <int S, class T>
struct I8G2 {
  static constexpr int TileB = S * kI8SliceB;             // 48 KB (S = 6)
  static constexpr int WCols = S * (kI8K / 4);            // 192 (S = 6)
  static constexpr int Acc = S;
  static constexpr int Slots = (512 - WCols) / kI8NT;     // 5 (S = 6), 6 (S = 4)
  static constexpr int SubRowsB = kI8SubR * 64 * (int)sizeof(T);  // norb <= 64
  static constexpr int SubB = SubRowsB + kI8SubR * 8;     // + the sub-tile's row scales sigma_r
  // (the Psi ring's space first stages C'' -- FP64, up to 64 x 64 complex -- for the W digits)
  static constexpr int RingB = kI8PsiSlots * SubB > 64 * 64 * 16 ? kI8PsiSlots * SubB : 64 * 64 * 16;
  static constexpr int Smem = kI8Stages * TileB + RingB + 1024;  // + alignment slack
};
constexpr int kI8Threads = (kI8EpiWarps + 3) * 32;  // epilogue warps + 2 producers + MMA
constexpr int kWDig = kI8EpiWarps, kWMma = kI8EpiWarps + 1, kWPsi = kI8EpiWarps + 2;  // role warps

// ---- B digits (once per lfd_init): warp per grid row -------------------------------------------------
template <class T, int S>
__global__ void __launch_bounds__(256) k_bslice_i8(const T* __restrict__ B, int nproj, long long ng,
                                                   long long tiles, int8_t* __restrict__ out,
                                                   double* __restrict__ sig) {
  pdl_wait();
  pdl_trigger();
  const int dom = blockIdx.y, lane = threadIdx.x & 31;
  const long long r = (long long)blockIdx.x * 8 + (threadIdx.x >> 5);
  if (r >= tiles * kI8NT) return;
  double v[4] = {0.0, 0.0, 0.0, 0.0};
  const int u0 = 2 * lane;
  if (r < ng) {
    const T* row = B + ((long long)dom * ng + r) * nproj;
    if (u0 < nproj) { const T a = row[u0]; v[0] = a.x; v[1] = a.y; }
    if (u0 + 1 < nproj) { const T a = row[u0 + 1]; v[2] = a.x; v[3] = a.y; }
  }
  double mx = fmax(fmax(fabs(v[0]), fabs(v[1])), fmax(fabs(v[2]), fabs(v[3])));
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
  const int e = mx > 0.0 ? row_exponent(mx) : 0;
  uint32_t d[S];
  digits4<S>(v, e, !(mx > 0.0), d);
  const long long t = r / kI8NT;
  const int rr = (int)(r - t * kI8NT);
  int8_t* tb = out + ((long long)dom * tiles + t) * (S * kI8SliceB);
#pragma unroll
  for (int i = 0; i < S; ++i) *reinterpret_cast<uint32_t*>(tb + i * kI8SliceB + sw128(rr, 4 * lane)) = d[i];
  if (lane == 0) sig[(long long)dom * tiles * kI8NT + r] = mx > 0.0 ? ldexp(1.0, e) : 0.0;
}

// ---- GEMM-2 -----------------------------------------------------------------------------------------
// grid (CTAs per domain, ndom); CTA b of a domain takes tiles b, b + gridDim.x, ...
template <bool kOut, class T, int S>
__global__ void __launch_bounds__(kI8Threads, 1) k_gemm2_i8(Gemm2Args p) {
  using G = I8G2<S, T>;
  using R = decltype(T::x);  // real component type of Psi (double / float)
  constexpr int kI8TileB = G::TileB, kI8WCols = G::WCols, kI8Acc = G::Acc, kI8Slots = G::Slots;
  constexpr int kI8SubRowsB = G::SubRowsB, kI8SubB = G::SubB;
  // programmatic dependent launch: the set-up below (TMEM, barriers) and the digit producer (B's digits are
  // constant since lfd_init) overlap the previous kernel; every other warp waits for it (C'', n, Psi)
  pdl_trigger();
  extern __shared__ __align__(1024) unsigned char dsm_raw[];
  // SWIZZLE_128B images need 1024-byte aligned shared addresses
  unsigned char* dsm = dsm_raw + ((1024u - (smem_addr(dsm_raw) & 1023u)) & 1023u);
  unsigned char* Tsm = dsm;                            // [stages][S][64 r][128 B] swizzled digit tiles
  unsigned char* Psm = Tsm + kI8Stages * kI8TileB;     // [slots][16 r][norb] complex + sigma: Psi sub-tiles
  unsigned char* Csm = Psm;                            // C'' of the domain (staged before the Psi ring starts)
  __shared__ __align__(8) uint64_t full[kI8Stages], empty[kI8Stages], dfull[kI8Slots], dempty[kI8Slots];
  __shared__ __align__(8) uint64_t pfull[kI8PsiSlots], pempty[kI8PsiSlots];
  __shared__ __align__(8) uint64_t cbar;
  __shared__ uint32_t tmem_base_sh;
  __shared__ double taus[kI8M];

  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int dom = blockIdx.y;
  const int norb = p.norb, nproj = p.nproj;
  const long long ng = p.ng;
  const long long tiles = (ng + kI8NT - 1) / kI8NT;

  if (warp == kWMma) {  // TMEM: W^T digits (A operand, 6 x 32 columns) + the ring of diagonal accumulators
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_addr(&tmem_base_sh)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    for (int s = 0; s < kI8Stages; ++s) { mbar_init(&full[s], 1); mbar_init(&empty[s], 1); }
    for (int s = 0; s < kI8Slots; ++s) { mbar_init(&dfull[s], 1); mbar_init(&dempty[s], kI8EpiWarps); }
    for (int s = 0; s < kI8PsiSlots; ++s) { mbar_init(&pfull[s], 1); mbar_init(&pempty[s], 4); }
    mbar_init(&cbar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_base_sh;
  const uint32_t tacc = tmem + kI8WCols;  // accumulator slot columns
  if (warp != kWDig) pdl_wait();

  if (warp < kI8EpiWarps) {
    // W^T digits from C'' (staged by one bulk copy) into TMEM: thread (warp w, lane) owns row
    // n = 32 (w & 3) + lane of W^T (TMEM lane n) and the 8 columns (32 K bytes, projectors 16 c8 ..
    // 16 c8 + 15) of chunk c8 = w >> 2 of each digit; k = 4 c + byte. tau_n = 2^f, max_k |W^T[n][k]| < 2^f.
    if (tid == 0) {
      mbar_expect_tx(&cbar, (uint32_t)(nproj * norb * 16));
      tma_row(Csm, p.Cp + (long long)dom * nproj * norb, (uint32_t)(nproj * norb * 16), &cbar);
    }
    const int q = warp & 3, c8 = warp >> 2;
    const int n = 32 * q + lane, s = n >> 1, cn = n & 1;
    const bool sv = s < norb;
    mbar_wait(&cbar, 0);
    const double2* X = reinterpret_cast<const double2*>(Csm) + s;  // X[u][s] at u * norb
    double mx = 0.0;
    if (sv)
      for (int u = 0; u < nproj; ++u) {
        const double2 x = X[u * norb];
        mx = fmax(mx, fmax(fabs(x.x), fabs(x.y)));
      }
    const int e = mx > 0.0 ? row_exponent(mx) : 0;
    if (c8 == 0) taus[n] = mx > 0.0 ? ldexp(1.0, e - 12) : 0.0;  // x 2^-12: the weight of diagonal 2
    const uint32_t trow = tmem + ((uint32_t)(32 * q) << 16);
    uint32_t dg[S][8];
#pragma unroll
    for (int w = 0; w < 8; ++w) {
      double v[4] = {0.0, 0.0, 0.0, 0.0};
      const int u0 = 16 * c8 + 2 * w;  // k = 4 (8 c8 + w) .. + 3 -> projectors u0, u0 + 1
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
  // W ready (TMEM digits, taus[]) and the staged C'' consumed: named barrier 1 over every warp except the
  // digit producer (warp 8), which streams from the start
  if (warp != kWDig) {
    tc_fence_before();
    asm volatile("bar.sync 1, %0;" ::"n"(kI8Threads - 32) : "memory");
    tc_fence_after();
  }

  const int rowb = norb * (int)sizeof(T);  // bytes per Psi row
  if (warp == kWDig) {  // producer of the digit tiles (one bulk copy each)
    if (lane == 0) {
      const int8_t* src = p.bsl + (long long)dom * tiles * kI8TileB;
      int it = 0;
      for (long long t = blockIdx.x; t < tiles; t += gridDim.x, ++it) {
        const int s = it % kI8Stages;
        if (it >= kI8Stages) mbar_wait(&empty[s], (uint32_t)(((it / kI8Stages) - 1) & 1));
        mbar_expect_tx(&full[s], kI8TileB);
        tma_row(Tsm + s * kI8TileB, src + t * kI8TileB, kI8TileB, &full[s]);
      }
    }
  } else if (warp == kWPsi) {  // producer of the Psi sub-tiles (16 contiguous rows + their 16 row scales)
    if (lane == 0) {
      const T* prow = reinterpret_cast<const T*>(p.psi) + (long long)dom * ng * norb;
      const double* sig = p.bsig + (long long)dom * tiles * kI8NT;
      int u = 0;
      for (long long t = blockIdx.x; t < tiles; t += gridDim.x)
        for (int k = 0; k < kI8NT / kI8SubR; ++k, ++u) {
          const int s = u % kI8PsiSlots;
          if (u >= kI8PsiSlots) mbar_wait(&pempty[s], (uint32_t)(((u / kI8PsiSlots) - 1) & 1));
          const long long r0 = t * kI8NT + k * kI8SubR;
          const long long nr = (ng - r0) < kI8SubR ? (ng - r0) : kI8SubR;
          if (nr <= 0) {  // past the domain end: nothing to stage, the slot completes at once
            mbar_arrive(&pfull[s]);
            continue;
          }
          tma_row8(Psm + s * kI8SubB, prow + r0 * norb, (uint32_t)(nr * rowb), &pfull[s], kI8SubR * 8);
          tma_row(Psm + s * kI8SubB + kI8SubRowsB, sig + r0, kI8SubR * 8, &pfull[s]);
        }
    }
  } else if (warp == kWMma) {  // MMA issuer: D_d += W_j^T (TMEM) x b_i (smem), i + j = d; one ring slot per d
    {  // the whole warp runs the loop (warp-uniform values stay in uniform registers); one elected lane issues
      const uint32_t tbase = smem_addr(Tsm);
      int it = 0;
      for (long long t = blockIdx.x; t < tiles; t += gridDim.x, ++it) {
        const int s = it % kI8Stages;
        mbar_wait(&full[s], (uint32_t)((it / kI8Stages) & 1));
        tc_fence_after();
        const uint64_t db0 = umma_desc_sw128(tbase + s * kI8TileB);
#pragma unroll
        for (int d = 2; d <= S + 1; ++d) {
          const int g = it * kI8Acc + (d - 2), sl = g % kI8Slots;
          if (g >= kI8Slots) {
            mbar_wait(&dempty[sl], (uint32_t)(((g / kI8Slots) - 1) & 1));
            tc_fence_after();
          }
          const uint32_t acc = tacc + sl * kI8NT;
          uint32_t first = 1;
#pragma unroll
          for (int i = 1; i <= S; ++i) {
            const int j = d - i;
            if (j < 1 || j > S) continue;
#pragma unroll
            for (int kk = 0; kk < kI8K / 32; ++kk) {
              // descriptor arithmetic is linear in the (>> 4) start address: one add per MMA (the issuing
              // warp shares its scheduler with four epilogue warps, so its instruction count matters)
              umma_i8_ts(acc, tmem + (j - 1) * 32 + kk * 8, db0 + (uint64_t)(((i - 1) * kI8SliceB + kk * 32) >> 4),
                         first ? 0u : 1u, i8_idesc(kI8NT));
              first = 0;
            }
          }
          umma_commit(&dfull[sl]);  // diagonal d of tile t ready
        }
        umma_commit(&empty[s]);  // the digit tile may be overwritten once these MMAs are done
      }
    }
  } else if (warp < kI8EpiWarps) {
    // epilogue: warp w reads TMEM lanes 32 (w & 3) .. + 31 (output double n of a Psi row) and tile rows
    // 16 (w >> 2) .. + 15; it drains the diagonals two at a time as they complete, (P_d 2^7 + P_{d+1}) an
    // exact int32, into FP64 sums acc_c = sum_d P_d 2^{-7(d-2)}; then Psi <- n_s Psi + sigma_r tau_n 2^-12 acc.
    const int q = warp & 3, h = warp >> 2;
    const int n = 32 * q + lane;
    const bool nvalid = n < 2 * norb;
    const double nf = nvalid ? p.nfac[(long long)dom * norb + (n >> 1)] : 0.0;
    const double tau = taus[n];
    R* pout = reinterpret_cast<R*>(reinterpret_cast<T*>(kOut ? p.psi_out : p.psi) + (long long)dom * ng * norb) + n;
    const int ld = 2 * norb;
    int it = 0;
    for (long long t = blockIdx.x; t < tiles; t += gridDim.x, ++it) {
      const long long r0 = t * kI8NT + kI8Rows * h;
      const int nc = (int)((ng - r0) < kI8Rows ? (ng - r0) : kI8Rows);  // valid rows of this warp
      // SP (R = float): each diagonal converted exactly (|P_d| < 2^21 for S = 4) and accumulated in FP32, the
      // scaling by exponent arithmetic on the float -- no FP64 pipe work in the SP epilogue
      constexpr bool kF32 = sizeof(R) == 4;
      using A = std::conditional_t<kF32, float, double>;
      A fa[kI8Rows];
#pragma unroll
      for (int c = 0; c < kI8Rows; ++c) fa[c] = A(0);
#pragma unroll  // (unrolled: C2 174 -> 165 us, the loads of the next pair overlap this pair's FP64 work)
      for (int dp = 0; dp < kI8Acc / 2; ++dp) {  // diagonals d = 2 + 2 dp and d + 1
        const int g = it * kI8Acc + 2 * dp, s0 = g % kI8Slots, s1 = (g + 1) % kI8Slots;
        mbar_wait(&dfull[s0], (uint32_t)((g / kI8Slots) & 1));
        mbar_wait(&dfull[s1], (uint32_t)(((g + 1) / kI8Slots) & 1));
        tc_fence_after();
        int32_t a0[kI8Rows], a1[kI8Rows];
        const uint32_t lb = ((uint32_t)(32 * q) << 16) + kI8Rows * h;
        tmem_ld16(tacc + s0 * kI8NT + lb, a0);
        tmem_ld16(tacc + s1 * kI8NT + lb, a1);
        tmem_wait_ld();
        tc_fence_before();
        __syncwarp();
        if (lane == 0) {  // the slots may take the next diagonals
          mbar_arrive(&dempty[s0]);
          mbar_arrive(&dempty[s1]);
        }
        if constexpr (kF32) {
          const float w0 = __int_as_float((127 - 14 * dp) << 23), w1 = __int_as_float((120 - 14 * dp) << 23);
#pragma unroll
          for (int c = 0; c < kI8Rows; ++c) fa[c] = fmaf(i2f(a1[c]), w1, fmaf(i2f(a0[c]), w0, fa[c]));
        } else {
          const double wd = ldexp(1.0, -14 * dp - 7);
          if (dp == 0) {  // fa = (m - M) wd in one fma: m = M + x built from bits, exact result x wd
#pragma unroll
            for (int c = 0; c < kI8Rows; ++c) fa[c] = fma(i2d_raw(a0[c] * 128 + a1[c]), wd, -kI2dM * wd);
          } else {
#pragma unroll
            for (int c = 0; c < kI8Rows; ++c) fa[c] = fma(i2d(a0[c] * 128 + a1[c]), wd, fa[c]);
          }
        }
      }
      // the warp's staged Psi sub-tile (rows 16 h .. 16 h + 15 of the tile)
      {
        const int u = it * (kI8NT / kI8SubR) + h, s = u % kI8PsiSlots;
        mbar_wait(&pfull[s], (uint32_t)((u / kI8PsiSlots) & 1));
        const R* ps = reinterpret_cast<const R*>(Psm + s * kI8SubB) + n;
        const double* sg = reinterpret_cast<const double*>(Psm + s * kI8SubB + kI8SubRowsB);
        if (nvalid) {  // running row pointers (16 precomputed row offsets would spill)
          R* po = pout + r0 * ld;
#pragma unroll
          for (int c = 0; c < kI8Rows; ++c) {
            if constexpr (kF32) {
              if (c < nc) *po = fmaf((float)nf, (float)*ps, scale_pow2f(fa[c], sg[c], tau));
            } else {
              if (c < nc) *po = (R)fma(nf, (double)*ps, scale_pow2(fa[c], sg[c], tau));
            }
            po += ld;
            ps += ld;
          }
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&pempty[s]);
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == kWMma) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
  }
}

// ================================================================================================
// GEMM-1 (Eq. 7 / Eq. 9): split partials of C[u][s] = sum_r conj(B[r][u]) Psi[r][s]
// and the column norms sum_r |Psi[r][s]|^2, on the int8 tensor cores with base-256 digits.
//
// Real form: D[m][u] = sum_k A[m][k] Bd[u][k] with m = 2s + c (M = 128) and k over the grid rows of a 64-row
// block in groups of 4 rows, k = 8 (rr / 4) + 4 c' + rr % 4 (K = 128 per block): A[2s][.] = (Re Psi, Im Psi)
// of the group's 4 rows, A[2s+1][.] = (Im Psi, -Re Psi), Bd[u][.] = (Re B, Im B); then D[2s][u] = Re C[u][s],
// D[2s+1][u] = Im C[u][s].
//
// Digits (S bytes per value: S = 5 for FP64 contexts, 3 for the SP variant). Psi, per orbital scale
// tau_s = 2^(E_s - 1022) (every |Re|, |Im| < tau_s; E_s recorded by the K_y K_z pass that wrote Psi, k_kin_yz /
// the SP z pass, integer max of the FP64 exponent fields, cleared here by the last CTA):
// X = rint(x 2^(8S-2) / tau_s), written OFFSET-BINARY -- the S bytes u_k of X + 2^(8S-1) are unsigned digits
// (tcgen05 kind::i8 takes u8 A x s8 B), and they are the low mantissa bytes of ONE DFMA against
// 1.5 2^52 + 2^(8S-1) (the sum is an integer below 2^53, so the DFMA rounds to it exactly). B, per column scale
// sigma_u (once at lfd_init): Y = rint(b 2^(8S-2) / sigma_u) as balanced base-256 digits d_i in [-128, 127]
// (the bytes of Y + 128 (1 + 256 + ... + 256^(S-1)) minus 128, from one DFMA the same way). With a_k the
// signed digits of X (a_k = u_k below the top byte, a_{S-1} = u_{S-1} - 128):
//   sum_K X Y = sum_{k,i} 256^(k+i) sum_K u_k d_i  -  128 sum_i 256^(S-1+i) sum_K d_i,
// the second term from the column sums of B's digits over the CTA's rows (exact, once at lfd_init). The pairs
// with k + i >= S - 2 are kept (19 of 25 for S = 5), grouped by diagonal d = k + i into S + 1 exact int32
// accumulators in TMEM (|P_d| <= S x 2 rps x 255 x 128 < 2^31 for rps <= 6144); the dropped pairs and the
// digit remainders are ~2^-38 relative to sigma_u tau_s (S = 5; the old base-128 scheme: ~2^-40), so the
// update B C'' stays within ~1e-15 of Psi per factor. C = sigma_u tau_s 2^-12 sum_d 256^(d-2S+2) (P_d - corr_d).
//
// Kernel: B's digits per 64-row block [S][64 u][128 B] in the SWIZZLE_128B image (one bulk copy, 2-stage
// ring); Psi rows staged per 16-row quarter block (bulk copies, 6-slot ring). 16 worker warps: lane (m, h)
// loads its orbital's two components of 4 grid rows, makes their digits (2 DFMA per row: digits, norm) and
// transposes them with byte permutes into the A words of its TMEM lane (2 per digit), into one of NBuf A
// buffers; one thread issues the quarter block's MMAs (S = 5: 7 MMAs of N = 64 w, w <= 4 consecutive
// diagonals each) as soon as its buffer is full. TMEM: NBuf x 8S A columns + (S + 1) x 64 accumulators.
// ================================================================================================
constexpr int kG1Rows = 64;                        // grid rows per B-digit block (K = 128 bytes)
constexpr int kG1Half = 16;                        // grid rows per A (Psi-digit) quarter block (K = 32 bytes)
constexpr int kG1SliceB = 64 * 128;                // 8 KB: one digit slice of a B block (64 u rows)
constexpr int kG1Stages = 2;                       // B-digit ring
constexpr int kG1PsiSlots = 6;                     // Psi quarter-block ring
constexpr int kG1Workers = 16;                     // worker warps: 4 lane quarters x 4 row groups
constexpr int kG1Threads = (kG1Workers + 2) * 32;  // + producer + MMA
constexpr int kG1WProd = kG1Workers, kG1WMma = kG1Workers + 1;
constexpr long long kG1MaxRps = 6144;              // int32 diagonals: S x 2 rps x 255 x 128 < 2^31 (S <= 5)
__host__ __device__ constexpr int g1_digits(bool sp) { return sp ? 3 : 5; }
// shapes depending on the digit count S and Psi's element type T
template <int S, class T>
struct I8G1 {
  static constexpr int Acc = S + 1;                           // diagonals d = S-2 .. 2S-2
  static constexpr int NBuf = S >= 5 ? 3 : 4;                 // TMEM A buffers
  static constexpr int ABuf = S * 8;                          // TMEM columns of one A buffer (K = 32 bytes)
  static constexpr int BlkB = S * kG1SliceB;                  // 40 KB (S = 5)
  static constexpr int PsiB = kG1Half * 64 * (int)sizeof(T);  // Psi rows of a quarter block (norb <= 64)
  static constexpr int Smem = kG1Stages * BlkB + kG1PsiSlots * PsiB + 1024;
  static_assert(NBuf * ABuf + 64 * Acc <= 512, "TMEM columns");
};
// s32 <- u8 (A, Psi digits) x s8 (B digits), both K-major, M = 128, N = n (a multiple of 64 here)
__host__ __device__ constexpr uint32_t g1_idesc(int n) {
  return (2u << 4) | (0u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
}
// 1.5 2^52 + the digit offset: the low 8S mantissa bits of fma(x, sc, M) are the integer rint(x sc) + offset
template <int S>
__host__ __device__ constexpr double g1_madd_a() { return 6755399441055744.0 + (double)(1LL << (8 * S - 1)); }
template <int S>
__host__ __device__ constexpr double g1_madd_b() {  // offset 128 (1 + 256 + ... + 256^(S-1))
  long long c = 0;
  for (int k = 0; k < S; ++k) c = (c << 8) | 128;
  return 6755399441055744.0 + (double)c;
}

// the S low bytes of rint(v[q] sc) + offset (q = 0..3) transposed: out[k] = byte k of the four values
template <int S>
__device__ __forceinline__ void g1_bytes(const double v[4], double sc, double madd, uint32_t out[S]) {
  uint32_t lo[4], hi[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const long long b = __double_as_longlong(fma(v[q], sc, madd));
    lo[q] = (uint32_t)b;
    hi[q] = (uint32_t)(b >> 32);
  }
  const uint32_t a = __byte_perm(lo[0], lo[1], 0x5140), b = __byte_perm(lo[0], lo[1], 0x7362);
  const uint32_t c = __byte_perm(lo[2], lo[3], 0x5140), d = __byte_perm(lo[2], lo[3], 0x7362);
  out[0] = __byte_perm(a, c, 0x5410);
  out[1] = __byte_perm(a, c, 0x7632);
  out[2] = __byte_perm(b, d, 0x5410);
  if constexpr (S >= 4) out[3] = __byte_perm(b, d, 0x7632);
  if constexpr (S >= 5) out[4] = __byte_perm(__byte_perm(hi[0], hi[1], 0x0040), __byte_perm(hi[2], hi[3], 0x0040), 0x5410);
  (void)hi;
}

// The SP variant (S = 3) from FP32 values: fma(v, sc, 1.5 2^23) is 1.5 2^23 + X exactly for |X| <= 2^22, its
// low 24 bits are X + 2^22 (the exponent's low bit is 0 below 2^24 and 1 at X = 2^22 exactly), so adding 2^22
// to the word gives the offset-binary X + 2^23 in the low 3 bytes, as the FP64 form's low bytes (g1_madd_a<3>).
__device__ __forceinline__ void g1_bytes3f(const float v[4], float sc, uint32_t out[3]) {
  uint32_t lo[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) lo[q] = __float_as_uint(fmaf(v[q], sc, 12582912.0f)) + 0x400000u;
  const uint32_t a = __byte_perm(lo[0], lo[1], 0x5140), b = __byte_perm(lo[0], lo[1], 0x7362);
  const uint32_t c = __byte_perm(lo[2], lo[3], 0x5140), d = __byte_perm(lo[2], lo[3], 0x7362);
  out[0] = __byte_perm(a, c, 0x5410);
  out[1] = __byte_perm(a, c, 0x7632);
  out[2] = __byte_perm(b, d, 0x5410);
}

__device__ __forceinline__ void umma_g1_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t db, uint32_t accumulate,
                                           uint32_t idesc) {
  asm volatile(
      "{\n.reg .pred p, e;\nelect.sync _|e, 0xffffffff;\nsetp.ne.b32 p, %4, 0;\n"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n}\n" ::"r"(tmem_d),
      "r"(tmem_a), "l"(db), "r"(idesc), "r"(accumulate));
}
__device__ __forceinline__ void tmem_st2(uint32_t taddr, const uint32_t v[2]) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x2.b32 [%0], {%1,%2};" ::"r"(taddr), "r"(v[0]), "r"(v[1]) : "memory");
}

// The MMAs of one quarter block: entry j = (A digit k, first B digit i0, width w) is one MMA of N = 64 w into the
// consecutive diagonals k + i0 .. k + i0 + w - 1 (B's digit slices i0 .. are consecutive 64-row K-major tiles,
// the diagonals consecutive 64-column TMEM blocks). The first two entries cover every diagonal exactly once
// (accumulate = 0 at a split's first quarter block); all pairs k + i >= S - 2 appear once.
template <int S>
__host__ __device__ constexpr int g1_sched_n() { return S == 5 ? 7 : 4; }
template <int S>
__host__ __device__ constexpr int g1_sched(int j) {  // k | i0 << 4 | w << 8
  if (S == 5) {
    constexpr int t[7] = {3 | 0 << 4 | 4 << 8, 4 | 3 << 4 | 2 << 8, 3 | 4 << 4 | 1 << 8, 4 | 0 << 4 | 3 << 8,
                          0 | 3 << 4 | 2 << 8, 1 | 2 << 4 | 3 << 8, 2 | 1 << 4 | 4 << 8};
    return t[j];
  }
  constexpr int t[4] = {1 | 0 << 4 | 3 << 8, 2 | 2 << 4 | 1 << 8, 2 | 0 << 4 | 2 << 8, 0 | 1 << 4 | 2 << 8};
  return t[j];
}
template <int S>
__device__ __forceinline__ void g1_mmas(uint32_t tacc, uint32_t ta, uint64_t db0, int kq, bool first) {
#pragma unroll
  for (int j = 0; j < g1_sched_n<S>(); ++j) {
    const int e = g1_sched<S>(j);
    const int k = e & 15, i0 = (e >> 4) & 15, w = e >> 8;
    umma_g1_ts(tacc + (k + i0 - (S - 2)) * 64, ta + k * 8, db0 + (uint64_t)((i0 * kG1SliceB + kq * 32) >> 4),
               (first && j < 2) ? 0u : 1u, g1_idesc(64 * w));
  }
}

// B's GEMM-1 scales: bexp[dom][u] = max over the domain of the biased exponent of Re / Im B[r][u]
template <class T>
__global__ void __launch_bounds__(256) k_bexp1_i8(const T* __restrict__ B, int nproj, long long ng,
                                                  int* __restrict__ bexp) {
  pdl_wait();
  pdl_trigger();
  __shared__ int sm[64];
  const int dom = blockIdx.y;
  for (int u = threadIdx.x; u < 64; u += blockDim.x) sm[u] = 0;
  __syncthreads();
  const long long n = ng * nproj;
  const T* b = B + (long long)dom * n;
  for (long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (long long)gridDim.x * blockDim.x) {
    const T v = b[i];
    const double vx = v.x, vy = v.y;  // (complex64 values widened exactly)
    const int e = max(__double2hiint(vx) & 0x7ff00000, __double2hiint(vy) & 0x7ff00000) >> 20;
    if (e > 0) atomicMax(sm + (int)(i % nproj), e);  // shared-memory atomics, then one global per column
  }
  __syncthreads();
  for (int u = threadIdx.x; u < nproj; u += blockDim.x)
    if (sm[u] > 0) atomicMax(bexp + (long long)dom * nproj + u, sm[u]);
}

// B's GEMM-1 digits: warp per (64-row block, u); lane l holds K bytes 4l .. 4l+3, i.e. component c' = l & 1 of
// rows 4 (l >> 1) .. + 3. Also the per-split column sums of each digit (integer atomics: order-independent).
template <class T, int S>
__global__ void __launch_bounds__(256) k_bslice1_i8(const T* __restrict__ B, int nproj, long long ng,
                                                    long long nblk, const int* __restrict__ bexp, int blk_per_split,
                                                    int nsplit, int8_t* __restrict__ out, int* __restrict__ colsum) {
  pdl_wait();
  pdl_trigger();
  const int dom = blockIdx.y, lane = threadIdx.x & 31;
  const long long wid = (long long)blockIdx.x * 8 + (threadIdx.x >> 5);
  if (wid >= nblk * 64) return;
  const long long blk = wid >> 6;
  const int u = (int)(wid & 63);
  double v[4] = {0.0, 0.0, 0.0, 0.0};
  const int E = u < nproj ? bexp[(long long)dom * nproj + u] : 0;
  if (u < nproj) {
    const T* col = B + (long long)dom * ng * nproj + u;
#pragma unroll
    for (int t = 0; t < 4; ++t) {
      const long long r = blk * kG1Rows + 4 * (lane >> 1) + t;
      if (r < ng) {
        const T a = col[r * nproj];
        v[t] = (lane & 1) ? a.y : a.x;
      }
    }
  }
  uint32_t d[S];
  g1_bytes<S>(v, E == 0 ? 0.0 : ldexp(1.0, 8 * S - 2 - (E - 1022)), g1_madd_b<S>(), d);  // |Y| <= 2^(8S-2)
  int8_t* tb = out + ((long long)dom * nblk + blk) * (S * kG1SliceB);
#pragma unroll
  for (int i = 0; i < S; ++i) {
    d[i] ^= 0x80808080u;  // byte f -> digit f - 128 (balanced)
    *reinterpret_cast<uint32_t*>(tb + i * kG1SliceB + sw128(u, 4 * lane)) = d[i];
  }
  if (u < nproj) {
    const int split = (int)(blk / blk_per_split);
#pragma unroll
    for (int i = 0; i < S; ++i) {
      int s = __dp4a((int)d[i], 0x01010101, 0);  // the 4 signed digits
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
      if (lane == 0 && s != 0) atomicAdd(colsum + (((long long)dom * nsplit + split) * S + i) * nproj + u, s);
    }
  }
}

// grid (splits, ndom); CTA = one split of rps rows (a multiple of 64)
template <class T, int S>
__global__ void __launch_bounds__(kG1Threads, 1) k_gemm1_i8(Gemm1I8Args p) {
  using G = I8G1<S, T>;
  using R = decltype(T::x);
  constexpr int kG1BlkB = G::BlkB, kG1PsiB = G::PsiB, kG1ABuf = G::ABuf, kNBuf = G::NBuf;
  // programmatic dependent launch: set-up and the first B-digit blocks (constant since lfd_init) overlap the
  // previous kernel; the Psi loads and everything reading colE / writing the partials wait for it
  pdl_trigger();
  extern __shared__ __align__(1024) unsigned char dsm_raw[];
  unsigned char* dsm = dsm_raw + ((1024u - (smem_addr(dsm_raw) & 1023u)) & 1023u);
  unsigned char* Bsm = dsm;                            // [stages][S][64 u][128 B] swizzled B digits
  unsigned char* Psm = Bsm + kG1Stages * kG1BlkB;      // [slots][16 rows][norb] complex
  __shared__ __align__(8) uint64_t bfull[kG1Stages], bempty[kG1Stages], pfull[kG1PsiSlots], pempty[kG1PsiSlots];
  __shared__ __align__(8) uint64_t afull[kNBuf], afree[kNBuf], done;
  __shared__ uint32_t tmem_base_sh;
  __shared__ double nsum[4][64];
  __shared__ int last_sh;

  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int dom = blockIdx.y, split = blockIdx.x;
  const int norb = p.norb, nproj = p.nproj;
  const long long ng = p.ng;
  const long long nblk = (ng + kG1Rows - 1) / kG1Rows;
  const long long r0 = (long long)split * p.rps;
  const long long r1 = min(ng, r0 + p.rps);
  const int nhalf = (int)((r1 - r0 + kG1Half - 1) / kG1Half);  // quarter blocks of this split
  const int rowb = norb * (int)sizeof(T);

  if (warp == kG1WMma) {  // TMEM: NBuf A buffers (Psi digits, 8 S columns each) + S + 1 accumulators x 64 columns
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_addr(&tmem_base_sh)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (tid == 0) {
    for (int s = 0; s < kG1Stages; ++s) { mbar_init(&bfull[s], 1); mbar_init(&bempty[s], 1); }
    for (int s = 0; s < kG1PsiSlots; ++s) { mbar_init(&pfull[s], 1); mbar_init(&pempty[s], kG1Workers); }
    for (int b = 0; b < kNBuf; ++b) { mbar_init(&afull[b], kG1Workers); mbar_init(&afree[b], 1); }
    mbar_init(&done, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = tmem_base_sh;
  const uint32_t tacc = tmem + kNBuf * kG1ABuf;

  if (warp == kG1WProd) {  // producer: B-digit blocks and Psi quarter blocks, in the order the MMAs use them
    if (lane == 0) {
      const int8_t* src = p.bsl1 + (long long)dom * nblk * kG1BlkB;
      const T* prow = reinterpret_cast<const T*>(p.psi) + (long long)dom * ng * norb;
      const int nb = (nhalf + 3) >> 2;  // B-digit blocks of this split
      for (int b = 0; b < kG1Stages && b < nb; ++b) {  // before the dependency wait: B is constant
        mbar_expect_tx(&bfull[b], kG1BlkB);
        tma_row(Bsm + b * kG1BlkB, src + (r0 / kG1Rows + b) * kG1BlkB, kG1BlkB, &bfull[b]);
      }
      pdl_wait();
      long long w_be = 0, w_pe = 0;
      G1_T0(t_all);
      for (int g = 0; g < nhalf; ++g) {
        if ((g & 3) == 0 && (g >> 2) >= kG1Stages) {
          const int b = g >> 2, s = b % kG1Stages;
          G1_T0(c0);
          mbar_wait(&bempty[s], (uint32_t)(((b / kG1Stages) - 1) & 1));
          G1_ACC(w_be, c0);
          mbar_expect_tx(&bfull[s], kG1BlkB);
          tma_row(Bsm + s * kG1BlkB, src + (r0 / kG1Rows + b) * kG1BlkB, kG1BlkB, &bfull[s]);
        }
        const int s = g % kG1PsiSlots;
        G1_T0(c1);
        if (g >= kG1PsiSlots) mbar_wait(&pempty[s], (uint32_t)(((g / kG1PsiSlots) - 1) & 1));
        G1_ACC(w_pe, c1);
        const long long ra = r0 + (long long)g * kG1Half;
        const long long nr = (r1 - ra) < kG1Half ? (r1 - ra) : kG1Half;
        tma_row8(Psm + s * kG1PsiB, prow + ra * norb, (uint32_t)(nr * rowb), &pfull[s], 0);
      }
#ifdef LFD_G1_TIMING
      if (blockIdx.x == 0 || blockIdx.x == 100)
        printf("g1 cta %d prod: total %lld wait-bempty %lld wait-pempty %lld blocks %d\n", blockIdx.x,
               clock64() - t_all, w_be, w_pe, nhalf);
#endif
      (void)w_be; (void)w_pe;
    }
  } else if (warp == kG1WMma) {  // MMA issuer
    {  // the whole warp runs the loop (warp-uniform values stay in uniform registers); one elected lane issues
      const uint32_t bbase = smem_addr(Bsm);
      long long w_bf = 0, w_af = 0;
      G1_T0(t_all);
      for (int g = 0, ab = 0, aph = 0; g < nhalf; ++g) {  // ab = g % NBuf, aph = (g / NBuf) & 1
        const int b = g >> 2, s = b % kG1Stages, kq = g & 3;
        G1_T0(c0);
        if (kq == 0) mbar_wait(&bfull[s], (uint32_t)((b / kG1Stages) & 1));
        G1_ACC(w_bf, c0);
        G1_T0(c1);
        mbar_wait(&afull[ab], (uint32_t)aph);
        G1_ACC(w_af, c1);
        tc_fence_after();
        g1_mmas<S>(tacc, tmem + ab * kG1ABuf, umma_desc_sw128(bbase + s * kG1BlkB), kq, g == 0);
        umma_commit(&afree[ab]);  // A buffer ab may take quarter block g + NBuf
        if (kq == 3 || g + 1 == nhalf) umma_commit(&bempty[s]);
        if (++ab == kNBuf) { ab = 0; aph ^= 1; }
      }
      umma_commit(&done);
#ifdef LFD_G1_TIMING
      if (lane == 0 && (blockIdx.x == 0 || blockIdx.x == 100))
        printf("g1 cta %d mma: total %lld wait-bfull %lld wait-afull %lld\n", blockIdx.x, clock64() - t_all, w_bf, w_af);
#endif
      (void)w_bf; (void)w_af;
    }
  } else {  // workers: Psi digits into TMEM, column norms; at the end the accumulators into FP64 partials
    pdl_wait();
    const int q = warp & 3, h = warp >> 2;    // lane quarter, row group (4 rows of each quarter block)
    const int m = 32 * q + lane, sIdx = m >> 1, cm = m & 1;
    const bool sv = sIdx < norb;
    const int E = sv ? p.colE[(long long)dom * norb + sIdx] : 0;
    const bool zc = E == 0;                   // an all-zero orbital (or none): tau = 0
    const double sc = zc ? 0.0 : ldexp(1.0, 8 * S - 2 - (E - 1022));  // x 2^(8S-2) / tau_s
    const double sc2 = cm ? -sc : sc;         // the odd row's second component is -Re
    constexpr double kMA = g1_madd_a<S>();
    // SP: the digits from the FP32 values (g1_bytes3f) and the norm per quarter block in FP32, so the workers do
    // no FP64 conversions; the scale 2^(22 - (E - 1022)) is a normal float unless max |psi_s| < 2^-106, and such
    // an orbital is taken as zero (its contribution to C is below 1e-32)
    constexpr bool kF = sizeof(R) == 4;
    static_assert(!kF || S == 3, "the FP32 digit path is the 3-digit SP scheme");
    const int esc = 8 * S - 2 - (E - 1022);
    const float scf = (zc || esc > 127) ? 0.0f : __int_as_float((esc + 127) << 23);
    const float scf2 = cm ? -scf : scf;
    double nrm = 0.0;
    const uint32_t trow = tmem + ((uint32_t)(32 * q) << 16);
    long long w_pf = 0, w_afr = 0, w_st = 0;
    G1_T0(t_all);
#pragma unroll(S == 5 ? 2 : 4)  // (FP64 129.1 -> 128.1 us; SP by 4: 89.4 -> 87.9)
    for (int g = 0, s = 0, ph = 0, ab = 0, aph = 0; g < nhalf; ++g) {
      G1_T0(c0);
      mbar_wait(&pfull[s], (uint32_t)ph);
      G1_ACC(w_pf, c0);
      const long long ra = r0 + (long long)g * kG1Half;
      // this lane's components of Psi[row][sIdx] for rows 4h .. 4h+3: (Re, Im) for the even row m = 2s, (Im, Re)
      // for the odd row (its Re enters negated: sc2)
      const R* P = reinterpret_cast<const R*>(Psm + s * kG1PsiB) + 2 * sIdx + 8 * h * norb;
      using V = std::conditional_t<kF, float, double>;
      V v1[4], v2[4];
      if (sv && ra + 4 * h + 4 <= r1) {  // all 4 rows present (every quarter block but a split's ragged last)
#pragma unroll
        for (int t = 0; t < 4; ++t) { v1[t] = P[t * 2 * norb + cm]; v2[t] = P[t * 2 * norb + 1 - cm]; }
      } else {
#pragma unroll
        for (int t = 0; t < 4; ++t) {
          const bool ok = sv && ra + 4 * h + t < r1;
          v1[t] = ok ? (V)P[t * 2 * norb + cm] : V(0);
          v2[t] = ok ? (V)P[t * 2 * norb + 1 - cm] : V(0);
        }
      }
      // this lane's share of the column norm: Re^2 (even lane, v1 = Re) or Im^2 (odd lane, v1 = Im); the pair
      // is summed once at the end. Absent rows add +0.
      uint32_t d1[S], d2[S];
      if constexpr (kF) {
        const float nq = fmaf(v1[3], v1[3], fmaf(v1[2], v1[2], fmaf(v1[1], v1[1], v1[0] * v1[0])));
        nrm += (double)nq;
        g1_bytes3f(v1, scf, d1);
        g1_bytes3f(v2, scf2, d2);
      } else {
        nrm = fma(v1[0], v1[0], nrm);
        nrm = fma(v1[1], v1[1], nrm);
        nrm = fma(v1[2], v1[2], nrm);
        nrm = fma(v1[3], v1[3], nrm);
        g1_bytes<S>(v1, sc, kMA, d1);
        g1_bytes<S>(v2, sc2, kMA, d2);
      }
      G1_T0(c1);
      if (g >= kNBuf) mbar_wait(&afree[ab], (uint32_t)(aph ^ 1));  // the MMAs of quarter block g - NBuf are done
      G1_ACC(w_afr, c1);
      tc_fence_after();
      G1_T0(c2);
#pragma unroll
      for (int k = 0; k < S; ++k) {
        const uint32_t w2[2] = {d1[k], d2[k]};
        tmem_st2(trow + ab * kG1ABuf + k * 8 + 2 * h, w2);
      }
      asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory");
      G1_ACC(w_st, c2);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) {
        mbar_arrive(&afull[ab]);
        // the Psi rows are free: the digits just stored depend on every load of them, so those have returned
        // (the hazard mbar_release guards against cannot occur here)
        mbar_arrive(&pempty[s]);
      }
      if (++s == kG1PsiSlots) { s = 0; ph ^= 1; }
      if (++ab == kNBuf) { ab = 0; aph ^= 1; }
    }
#ifdef LFD_G1_TIMING
    if (tid == 0 && (blockIdx.x == 0 || blockIdx.x == 100))
      printf("g1 cta %d work0: total %lld wait-pfull %lld wait-afree %lld tmem-st %lld\n", blockIdx.x, clock64() - t_all,
             w_pf, w_afr, w_st);
#endif
    (void)w_pf; (void)w_afr; (void)w_st;
    // column norms: Re^2 (even lane) + Im^2 (odd lane), then a fixed-order sum over the 4 row groups
    nrm += __shfl_xor_sync(0xffffffffu, nrm, 1);
    if (!cm && sv) nsum[h][sIdx] = nrm;
    mbar_wait(&done, 0);
    tc_fence_after();
    // accumulators: warp (q, h) reads lanes 32 q .. (rows m) and columns u = 16 h .. 16 h + 15
    const int* cs = p.colsum + ((long long)dom * p.nsplit + split) * S * nproj;  // [S][nproj]
    double cacc[16];
#pragma unroll
    for (int c = 0; c < 16; ++c) cacc[c] = 0.0;
#pragma unroll 1
    for (int d = S - 2; d <= 2 * S - 2; ++d) {
      int32_t a[16];
      tmem_ld16(tacc + (d - (S - 2)) * 64 + ((uint32_t)(32 * q) << 16) + 16 * h, a);
      tmem_wait_ld();
      const double wd = ldexp(1.0, -8 * (2 * S - 2 - d));
      const int i = d - (S - 1);  // the pair (S-1, i) carries the offset of the top A digit
#pragma unroll
      for (int c = 0; c < 16; ++c) {
        const int u = 16 * h + c;
        double pd = i2d(a[c]);
        if (i >= 0 && u < nproj) pd -= 128.0 * (double)cs[i * nproj + u];
        cacc[c] = fma(pd, wd, cacc[c]);
      }
    }
    // C[u][s] = sigma_u tau_s 2^-12 cacc; m = 2 s + cm -> Re (cm 0) / Im (cm 1)
    const double tau = zc ? 0.0 : ldexp(1.0, E - 1022 - 12);
    double* part = reinterpret_cast<double*>(p.part + ((long long)dom * p.nsplit + split) * nproj * norb);
#pragma unroll
    for (int c = 0; c < 16; ++c) {
      const int u = 16 * h + c;
      if (!sv || u >= nproj) continue;
      const int eb = p.bexp[(long long)dom * nproj + u];
      const double sig = eb == 0 ? 0.0 : ldexp(1.0, eb - 1022);
      part[2 * ((long long)u * norb + sIdx) + cm] = sig * tau * cacc[c];
    }
    asm volatile("bar.sync 1, %0;" ::"n"(kG1Workers * 32) : "memory");
    if (tid < norb)
      p.norms[((long long)dom * p.nsplit + split) * norb + tid] =
          (nsum[0][tid] + nsum[1][tid]) + (nsum[2][tid] + nsum[3][tid]);
  }
  tc_fence_before();
  __syncthreads();
  // the last CTA of the domain clears the orbital exponents for the next K_y K_z pass
  if (tid == 0) {
    __threadfence();
    last_sh = atomicAdd(p.counter + dom, 1) == (int)gridDim.x - 1;
  }
  __syncthreads();
  if (last_sh) {
    for (int i = tid; i < norb; i += blockDim.x) p.colE[(long long)dom * norb + i] = 0;
    if (tid == 0) p.counter[dom] = 0;
  }
  if (warp == kG1WMma) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
  }
}

size_t gemm1_i8_bytes(int ndom, long long ng, bool sp) {
  const long long nblk = (ng + kG1Rows - 1) / kG1Rows;
  return (size_t)ndom * nblk * g1_digits(sp) * kG1SliceB;
}
size_t gemm1_i8_colsum_bytes(int ndom, int nsplit, int nproj, bool sp) {
  return (size_t)ndom * nsplit * g1_digits(sp) * nproj * sizeof(int);
}
long long gemm1_i8_rows_per_split(long long ng, int ndom, int num_sms) {
  int cpd = num_sms / ndom;
  if (cpd < 1) cpd = 1;
  long long rps = (ng + cpd - 1) / cpd;
  rps = (rps + kG1Rows - 1) / kG1Rows * kG1Rows;
  if (rps > kG1MaxRps) rps = kG1MaxRps;
  return rps;
}
cudaError_t launch_bslice1_i8(const void* B, bool sp, int ndom, int nproj, long long ng, long long rps, int nsplit,
                              int* bexp, int8_t* out, int* colsum, cudaStream_t st) {
  cudaError_t e = cudaMemsetAsync(bexp, 0, sizeof(int) * ndom * nproj, st);
  if (e == cudaSuccess) e = cudaMemsetAsync(colsum, 0, gemm1_i8_colsum_bytes(ndom, nsplit, nproj, sp), st);
  if (e != cudaSuccess) return e;
  const long long nblk = (ng + kG1Rows - 1) / kG1Rows;
  const int bps = (int)(rps / kG1Rows);
  dim3 grid((unsigned)((nblk * 64 + 7) / 8), ndom);
  if (sp) {
    const float2* b = static_cast<const float2*>(B);
    launch_k(k_bexp1_i8<float2>, dim3(296, ndom), 256, 0, st, b, nproj, ng, bexp);
    launch_k(k_bslice1_i8<float2, 3>, grid, 256, 0, st, b, nproj, ng, nblk, (const int*)bexp, bps, nsplit, out, colsum);
  } else {
    const double2* b = static_cast<const double2*>(B);
    launch_k(k_bexp1_i8<double2>, dim3(296, ndom), 256, 0, st, b, nproj, ng, bexp);
    launch_k(k_bslice1_i8<double2, 5>, grid, 256, 0, st, b, nproj, ng, nblk, (const int*)bexp, bps, nsplit, out, colsum);
  }
  return cudaGetLastError();
}
cudaError_t launch_gemm1_i8(const Gemm1I8Args& a, cudaStream_t st) {
  dim3 grid(a.nsplit, a.ndom);
  if (a.sp) launch_k(k_gemm1_i8<float2, 3>, grid, kG1Threads, I8G1<3, float2>::Smem, st, a);
  else launch_k(k_gemm1_i8<double2, 5>, grid, kG1Threads, I8G1<5, double2>::Smem, st, a);
  return cudaGetLastError();
}

size_t gemm2_i8_bytes(int ndom, long long ng, int S) {
  const long long tiles = (ng + kI8NT - 1) / kI8NT;
  return (size_t)ndom * tiles * S * kI8SliceB;
}
size_t gemm2_i8_sig_bytes(int ndom, long long ng) {
  const long long tiles = (ng + kI8NT - 1) / kI8NT;
  return (size_t)ndom * tiles * kI8NT * sizeof(double);
}
bool gemm2_i8_supported(int nproj, int norb) { return nproj >= 1 && nproj <= 64 && norb >= 1 && norb <= 64; }

cudaError_t launch_bslice_i8(const void* B, bool sp, int ndom, int nproj, long long ng, int8_t* out, double* sig,
                             cudaStream_t st) {
  const long long tiles = (ng + kI8NT - 1) / kI8NT;
  dim3 grid((unsigned)((tiles * kI8NT + 7) / 8), ndom);
  if (sp) launch_k(k_bslice_i8<float2, 4>, grid, 256, 0, st, static_cast<const float2*>(B), nproj, ng, tiles, out, sig);
  else launch_k(k_bslice_i8<double2, 6>, grid, 256, 0, st, static_cast<const double2*>(B), nproj, ng, tiles, out, sig);
  return cudaGetLastError();
}

cudaError_t launch_gemm2_i8(const Gemm2Args& a, cudaStream_t st) {
  const long long tiles = (a.ng + kI8NT - 1) / kI8NT;
  int cpd = a.num_sms / a.ndom;
  if (cpd < 1) cpd = 1;
  if (cpd > tiles) cpd = (int)tiles;
  dim3 grid(cpd, a.ndom);
  if (a.sp) {
    constexpr int sm = I8G2<4, float2>::Smem;
    if (a.psi_out) launch_k(k_gemm2_i8<true, float2, 4>, grid, kI8Threads, sm, st, a);
    else launch_k(k_gemm2_i8<false, float2, 4>, grid, kI8Threads, sm, st, a);
  } else {
    constexpr int sm = I8G2<6, double2>::Smem;
    if (a.psi_out) launch_k(k_gemm2_i8<true, double2, 6>, grid, kI8Threads, sm, st, a);
    else launch_k(k_gemm2_i8<false, double2, 6>, grid, kI8Threads, sm, st, a);
  }
  return cudaGetLastError();
}

cudaError_t gemm_i8_set_attributes() {
  cudaError_t e = cudaSuccess;
#define LFD_ATTR(f, sm) \
  if ((e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, sm)) != cudaSuccess) return e
  LFD_ATTR((k_gemm2_i8<false, double2, 6>), (I8G2<6, double2>::Smem));
  LFD_ATTR((k_gemm2_i8<true, double2, 6>), (I8G2<6, double2>::Smem));
  LFD_ATTR((k_gemm2_i8<false, float2, 4>), (I8G2<4, float2>::Smem));
  LFD_ATTR((k_gemm2_i8<true, float2, 4>), (I8G2<4, float2>::Smem));
  LFD_ATTR((k_gemm1_i8<double2, 5>), (I8G1<5, double2>::Smem));
  LFD_ATTR((k_gemm1_i8<float2, 3>), (I8G1<3, float2>::Smem));
#undef LFD_ATTR
  return cudaSuccess;
}

}  // namespace lfd
