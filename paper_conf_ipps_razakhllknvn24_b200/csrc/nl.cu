// nl.cu -- the "BLASified" nonlocal factor of Eq. 6/7/9 for sm_100a.
//
// Paper: Eq. 7 projects v_nl on the unoccupied KS orbitals at t = 0; §III-D casts it as
// two BLAS-3 calls on the Ngrid x Norb matrix Psi (Eq. 9); Eq. 6 divides by the norm.
// Readings R9-R12: C = dV B^H Psi; Psi <- (Psi - i (Delta/2) B diag(D) C) diag(n), with n_s restoring
// each orbital's norm, computed here from the Gram closed form ||Psi'_s||^2 = s_s + eps^2 (DC)^H G (DC).
//
// Both GEMMs are FP64 complex and really are dense contractions, so they run on the FP64 tensor pipe:
// warp-level DMMA (mma.sync m8n8k4 f64 -> SASS DMMA.8x8x4; tcgen05 has no f64 kind on sm_100a).
// Complex products use 4 real DMMAs. Operand rows are staged into shared memory by the TMA engine
// (cp.async.bulk, one bulk copy per row segment, completion on an mbarrier with expect_tx) through a
// 4-stage ring; rows are padded (66 / 20 complex) so every DMMA fragment load (LDS.128) is
// bank-conflict free.
//  * GEMM-1 (k_gemm1): C partials over a fixed split of the grid rows (tall-skinny, K = Ngrid), plus
//    the column norms s_s from the same operand fragments. Split partials are reduced in a fixed order
//    (k_reduce) -- deterministic, no atomics.
//  * GEMM-2 (k_gemm2): persistent CTAs over (domain, 64-row block, 64-column tile); the epilogue fuses
//    Psi + B C' and the per-orbital renormalisation and writes Psi in place.
#include "lfd_complex.cuh"
#include "lfd_internal.h"
#include "lfd_tma.cuh"

namespace lfd {

namespace {

constexpr int kThreads = 256;  // 8 warps: 2 (M) x 4 (N), warp tile 32 x 16 complex
constexpr int kTile = 64;      // CTA tile 64 x 64 complex

// GEMM-1 stage: A rows [KC1][kLd1] (B rows, m along the row) and X rows [KC1][kLd1].
constexpr int kKC1 = 32;
constexpr int kLd1 = kTile + 2;
constexpr int kStages1 = 3;
constexpr int kConsWarps1 = 8;
constexpr int kThreads1 = kConsWarps1 * 32 + 32;  // + producer warp
// GEMM-2 stage: A rows [64][kLdA2] (B rows, k = projector along the row) and C' rows [KC2][kLd1].
constexpr int kKC2 = 32;
constexpr int kLdA2 = kKC2 + 4;  // 36 == 4 mod 8: conflict-free A-fragment loads

__device__ __forceinline__ void dmma(double& c0, double& c1, double a, double b) {
  asm("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
      : "+d"(c0), "+d"(c1)
      : "d"(a), "d"(b));
}


#ifndef LFD_3M
#define LFD_3M 1  // Gauss/3M complex product: 3 real DMMAs per complex tile instead of 4
#endif

// Accumulators of one warp: 4 (M) x 2 (N) DMMA tiles. With 3M, for A = a_r + i a_i and
// B = b_r + i b_i the three real products are T1 = a_r b_r, T2 = a_i b_i, T3 = (a_r + a_i)(b_r + b_i),
// so Re = T1 - T2 and Im = T3 - T1 - T2 (GEMM-2). GEMM-1 multiplies by conj(A): there T3 uses
// (a_r - a_i), Re = T1 + T2, Im = T3 - T1 + T2. The flop count reported is always 8 per complex
// multiply-add ("label any 3M 'effective' rate").
struct Frag {
  double t1[4][2][2];
  double t2[4][2][2];
  double t3[4][2][2];
  __device__ __forceinline__ void zero() {
#pragma unroll
    for (int i = 0; i < 4; ++i)
#pragma unroll
      for (int j = 0; j < 2; ++j)
#pragma unroll
        for (int c = 0; c < 2; ++c) t1[i][j][c] = t2[i][j][c] = t3[i][j][c] = 0.0;
  }
  // GEMM-2 (plain product) results
  __device__ __forceinline__ double re(int i, int j, int c) const {
#if LFD_3M
    return t1[i][j][c] - t2[i][j][c];
#else
    return t1[i][j][c];
#endif
  }
  __device__ __forceinline__ double im(int i, int j, int c) const {
#if LFD_3M
    return t3[i][j][c] - t1[i][j][c] - t2[i][j][c];
#else
    return t2[i][j][c];
#endif
  }
};

// acc += a (4 row fragments) * c (2 column fragments), complex. Passes over the 8 tiles keep the
// updates of one accumulator 8 independent DMMAs apart.
__device__ __forceinline__ void mma_4x2(Frag& acc, const double2 (&a)[4], const double2 (&c)[2]) {
#if LFD_3M
  double as[4], cs[2];
#pragma unroll
  for (int mi = 0; mi < 4; ++mi) as[mi] = a[mi].x + a[mi].y;
#pragma unroll
  for (int ni = 0; ni < 2; ++ni) cs[ni] = c[ni].x + c[ni].y;
#pragma unroll
  for (int mi = 0; mi < 4; ++mi)
#pragma unroll
    for (int ni = 0; ni < 2; ++ni) dmma(acc.t1[mi][ni][0], acc.t1[mi][ni][1], a[mi].x, c[ni].x);
#pragma unroll
  for (int mi = 0; mi < 4; ++mi)
#pragma unroll
    for (int ni = 0; ni < 2; ++ni) dmma(acc.t2[mi][ni][0], acc.t2[mi][ni][1], a[mi].y, c[ni].y);
#pragma unroll
  for (int mi = 0; mi < 4; ++mi)
#pragma unroll
    for (int ni = 0; ni < 2; ++ni) dmma(acc.t3[mi][ni][0], acc.t3[mi][ni][1], as[mi], cs[ni]);
#else
#pragma unroll
  for (int mi = 0; mi < 4; ++mi)
#pragma unroll
    for (int ni = 0; ni < 2; ++ni) dmma(acc.t1[mi][ni][0], acc.t1[mi][ni][1], a[mi].x, c[ni].x);  // + ar cr
#pragma unroll
  for (int mi = 0; mi < 4; ++mi)
#pragma unroll
    for (int ni = 0; ni < 2; ++ni) dmma(acc.t2[mi][ni][0], acc.t2[mi][ni][1], a[mi].x, c[ni].y);  // + ar ci
#pragma unroll
  for (int mi = 0; mi < 4; ++mi)
#pragma unroll
    for (int ni = 0; ni < 2; ++ni) dmma(acc.t1[mi][ni][0], acc.t1[mi][ni][1], -a[mi].y, c[ni].y);  // - ai ci
#pragma unroll
  for (int mi = 0; mi < 4; ++mi)
#pragma unroll
    for (int ni = 0; ni < 2; ++ni) dmma(acc.t2[mi][ni][0], acc.t2[mi][ni][1], a[mi].y, c[ni].x);  // + ai cr
#endif
}

}  // namespace

// ------------------------------------------------------------------------------------------------
// GEMM-1: part[dom][split][m][n] = sum_{r in split} conj(A[r][m]) X[r][n];  norms[dom][split][n].
// grid: (nsplit, mtiles*ntiles, ndom), block 8 consumer warps + 1 producer warp. CTA tile kMT x 64
// complex: kMT = 64 uses 2 x 4 warps (warp tile 32 x 16); kMT = 32 / 16 (few projectors, e.g. the
// paper-timing-consistent nproj = 16, R20) use 1 x 8 warps (warp tile kMT x 8) so no DMMA work is spent
// on empty projector rows. Per chunk of kKC1 grid rows the producer issues TWO tiled TMA tensor copies
// (the A and X row blocks, box [kKC1 rows][tile + 2 complex]: the 2 extra columns are the next tile's
// data or zero fill, which pads every smem row to == 2 mod 8 complex so the DMMA fragment LDS.128 are
// bank-conflict free) into a kStages1-deep ring with full/empty mbarriers; consumer warps release a
// stage when done with it (no CTA-wide barrier in the K loop). Rows past the domain end are zero-filled
// by the TMA (rows_per_split is a multiple of kKC1, so every other chunk is whole). The column norms s_s
// are accumulated from the X fragments, the k-steps split between the M-warps of a column slice.
// ------------------------------------------------------------------------------------------------
template <int MI, int NI>
struct FragT {
  double t1[MI][NI][2], t2[MI][NI][2], t3[MI][NI][2];
  __device__ __forceinline__ void zero() {
#pragma unroll
    for (int i = 0; i < MI; ++i)
#pragma unroll
      for (int j = 0; j < NI; ++j)
#pragma unroll
        for (int c = 0; c < 2; ++c) t1[i][j][c] = t2[i][j][c] = t3[i][j][c] = 0.0;
  }
};

// acc += conj(a) * x, 3M (see Frag): T1 = ar xr, T2 = ai xi, T3 = (ar - ai)(xr + xi)
template <int MI, int NI>
__device__ __forceinline__ void mma_conj(FragT<MI, NI>& acc, const double2 (&a)[MI], const double2 (&x)[NI]) {
  double as[MI], xs[NI];
#pragma unroll
  for (int mi = 0; mi < MI; ++mi) as[mi] = a[mi].x - a[mi].y;
#pragma unroll
  for (int ni = 0; ni < NI; ++ni) xs[ni] = x[ni].x + x[ni].y;
#pragma unroll
  for (int mi = 0; mi < MI; ++mi)
#pragma unroll
    for (int ni = 0; ni < NI; ++ni) dmma(acc.t1[mi][ni][0], acc.t1[mi][ni][1], a[mi].x, x[ni].x);
#pragma unroll
  for (int mi = 0; mi < MI; ++mi)
#pragma unroll
    for (int ni = 0; ni < NI; ++ni) dmma(acc.t2[mi][ni][0], acc.t2[mi][ni][1], a[mi].y, x[ni].y);
#pragma unroll
  for (int mi = 0; mi < MI; ++mi)
#pragma unroll
    for (int ni = 0; ni < NI; ++ni) dmma(acc.t3[mi][ni][0], acc.t3[mi][ni][1], as[mi], xs[ni]);
}

// kNT = 32: the N tile for narrow orbital sets (norb <= 32, C5's first row): 4 x 2 warps of 16 x 16, so no DMMA
// work is spent on empty orbital columns either
template <int kMT, int kNT = kTile>
struct G1Shape {
  static constexpr int WM = kNT == 32 ? (kMT >= 64 ? 4 : 2) : (kMT == 64 ? 2 : 1);  // warps along M
  static constexpr int WN = 8 / WM;              // warps along N
  static constexpr int MI = kMT / WM / 8;        // 8-row fragments per warp
  static constexpr int NI = kNT / WN / 8;        // 8-column fragments per warp
  static constexpr int LDA = kMT + 2;            // smem row pitch of the A block (complex)
  static constexpr int LDX = kNT + 2;            // smem row pitch of the X block (== 2 mod 8 complex)
  static constexpr int ABytes = kKC1 * LDA * 16;
  static constexpr int StageBytes = ABytes + kKC1 * LDX * 16;
};

template <int kMT, int kNT = kTile>
__global__ void __launch_bounds__(kThreads1, 1) k_gemm1(const __grid_constant__ CUtensorMap tA,
                                                         const __grid_constant__ CUtensorMap tX, Gemm1Args p) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  using S = G1Shape<kMT, kNT>;
  extern __shared__ __align__(128) unsigned char smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + kStages1 * S::StageBytes);
  uint64_t* empty = full + kStages1;
  __shared__ double nsh[4][kNT];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int split = blockIdx.x;
  const int ntn = (p.ncols + kNT - 1) / kNT;
  const int mt = blockIdx.y / ntn, nt = blockIdx.y - (blockIdx.y / ntn) * ntn;
  const int dom = blockIdx.z;
  const int m0 = mt * kMT, n0 = nt * kNT;
  const long long kbeg = (long long)split * p.rows_per_split;
  const long long kend = min(p.ng, kbeg + p.rows_per_split);
  const int nchunks = (kend > kbeg) ? (int)((kend - kbeg + kKC1 - 1) / kKC1) : 0;

  if (tid == 0) {
    for (int s = 0; s < kStages1; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], kConsWarps1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  if (warp == kConsWarps1) {  // producer warp
    if (lane == 0) {
      for (int i = 0; i < nchunks; ++i) {
        const int s = i % kStages1;
        if (i >= kStages1) mbar_wait(&empty[s], (uint32_t)(((i / kStages1) - 1) & 1));
        mbar_expect_tx(&full[s], (uint32_t)S::StageBytes);
        unsigned char* st = smem + s * S::StageBytes;
        const int r0 = (int)(kbeg + (long long)i * kKC1);
        tma_3d(st, &tA, 2 * m0, r0, dom, &full[s]);
        tma_3d(st + S::ABytes, &tX, 2 * n0, r0, dom, &full[s]);
      }
    }
    return;
  }

  const int g = lane >> 2, t = lane & 3;
  const int wm = warp / S::WN, wn = warp - (warp / S::WN) * S::WN;
  const int mvalid = min(kMT, p.mrows - m0), nvalid = min(kNT, p.ncols - n0);
  FragT<S::MI, S::NI> acc;
  acc.zero();
  double nrm[S::NI];
#pragma unroll
  for (int ni = 0; ni < S::NI; ++ni) nrm[ni] = 0.0;
  const bool do_norm = (p.norms != nullptr) && (mt == 0);

  for (int i = 0; i < nchunks; ++i) {
    const int s = i % kStages1;
    mbar_wait(&full[s], (uint32_t)((i / kStages1) & 1));
    const double2* As = reinterpret_cast<const double2*>(smem + s * S::StageBytes);
    const double2* Xs = reinterpret_cast<const double2*>(smem + s * S::StageBytes + S::ABytes);
    double2 a[S::MI], x[S::NI];
#pragma unroll
    for (int kk = 0; kk < kKC1; kk += 4) {
      const int k = kk + t;
#pragma unroll
      for (int mi = 0; mi < S::MI; ++mi) a[mi] = As[k * S::LDA + wm * (kMT / S::WM) + mi * 8 + g];
#pragma unroll
      for (int ni = 0; ni < S::NI; ++ni) x[ni] = Xs[k * S::LDX + wn * (kNT / S::WN) + ni * 8 + g];
      if (do_norm && ((kk >> 2) % S::WM) == wm) {
#pragma unroll
        for (int ni = 0; ni < S::NI; ++ni) nrm[ni] = fma(x[ni].x, x[ni].x, fma(x[ni].y, x[ni].y, nrm[ni]));
      }
      mma_conj(acc, a, x);
    }
    double dep = 0.0;  // the stage's last loads have returned before it is released (lfd_tma.cuh)
#pragma unroll
    for (int mi = 0; mi < S::MI; ++mi) dep += a[mi].x;
#pragma unroll
    for (int ni = 0; ni < S::NI; ++ni) dep += x[ni].x;
    mbar_release(&empty[s], dep, lane == 0);
  }

  // epilogue: split partials (fixed positions, reduced in order by k_reduce); 3M recombination for
  // conj(A): Re = T1 + T2, Im = T3 - T1 + T2
  double2* out = p.part + (((long long)dom * p.nsplit + split) * p.mrows) * p.ncols;
#pragma unroll
  for (int mi = 0; mi < S::MI; ++mi) {
    const int row = wm * (kMT / S::WM) + mi * 8 + g;
    if (row >= mvalid) continue;
#pragma unroll
    for (int ni = 0; ni < S::NI; ++ni)
#pragma unroll
      for (int c = 0; c < 2; ++c) {
        const int col = wn * (kNT / S::WN) + ni * 8 + 2 * t + c;
        if (col < nvalid) {
          const double t1 = acc.t1[mi][ni][c], t2 = acc.t2[mi][ni][c], t3 = acc.t3[mi][ni][c];
          out[(long long)(m0 + row) * p.ncols + n0 + col] = make_double2(t1 + t2, t3 - t1 + t2);
        }
      }
  }
  if (do_norm) {
#pragma unroll
    for (int ni = 0; ni < S::NI; ++ni) {
      double v = nrm[ni];
      v += __shfl_xor_sync(0xffffffffu, v, 1);
      v += __shfl_xor_sync(0xffffffffu, v, 2);
      if (t == 0) nsh[wm][wn * (kNT / S::WN) + ni * 8 + g] = v;
    }
    asm volatile("bar.sync 1, %0;" ::"n"(kConsWarps1 * 32));  // consumer warps only
    if (tid < nvalid) {
      double v = nsh[0][tid];
#pragma unroll
      for (int q = 1; q < S::WM; ++q) v += nsh[q][tid];
      p.norms[((long long)dom * p.nsplit + split) * p.ncols + n0 + tid] = v;
    }
  }
}

static int gemm1_mt(int mrows) { return mrows <= 16 ? 16 : mrows <= 32 ? 32 : 64; }

// A [dom][ng][mrows] / X [dom][ng][ncols] complex as 3-D float64 tensors, boxes [1][kKC1][tile + 2].
static cudaError_t gemm1_maps(const Gemm1Args& a, int mt, int nt, CUtensorMap* tA, CUtensorMap* tX) {
  const uint32_t boxA[3] = {(uint32_t)(2 * (mt + 2)), kKC1, 1};
  const uint32_t boxX[3] = {(uint32_t)(2 * (nt + 2)), kKC1, 1};
  const uint64_t dA[3] = {(uint64_t)2 * a.mrows, (uint64_t)a.ng, (uint64_t)a.ndom};
  const uint64_t sA[2] = {(uint64_t)a.mrows * 16, (uint64_t)a.a_dom_stride * 16};
  cudaError_t e = encode_tmap_f64(tA, 3, a.A, dA, sA, boxA);
  if (e != cudaSuccess) return e;
  const uint64_t dX[3] = {(uint64_t)2 * a.ncols, (uint64_t)a.ng, (uint64_t)a.ndom};
  const uint64_t sX[2] = {(uint64_t)a.ncols * 16, (uint64_t)a.x_dom_stride * 16};
  return encode_tmap_f64(tX, 3, a.X, dX, sX, boxX);
}

int gemm1_smem_bytes() { return kStages1 * G1Shape<64>::StageBytes + 2 * kStages1 * 8; }

cudaError_t launch_gemm1(const Gemm1Args& a, cudaStream_t st) {
  const int mt = gemm1_mt(a.mrows);
  const int nt = a.ncols <= 32 ? 32 : kTile;
  const int tiles = ((a.mrows + mt - 1) / mt) * ((a.ncols + nt - 1) / nt);
  dim3 grid(a.nsplit, tiles, a.ndom);
  CUtensorMap tA, tX;
  cudaError_t e = gemm1_maps(a, mt, nt, &tA, &tX);
  if (e != cudaSuccess) return e;
#define LFD_G1(M, N) launch_k(k_gemm1<M, N>, grid, kThreads1, kStages1 * G1Shape<M, N>::StageBytes + 2 * kStages1 * 8, \
                              st, tA, tX, a)
  if (nt == 32) {
    if (mt == 16) LFD_G1(16, 32);
    else if (mt == 32) LFD_G1(32, 32);
    else LFD_G1(64, 32);
  } else {
    if (mt == 16) LFD_G1(16, 64);
    else if (mt == 32) LFD_G1(32, 64);
    else LFD_G1(64, 64);
  }
#undef LFD_G1
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// Fixed-order split-K reduction. Block = 32 consecutive output elements x 8 split groups: thread
// (e, sg) sums splits sg, sg+8, ... of element e (coalesced over e), then the 8 group sums are added in
// group order. Blocks past the element range reduce the column norms the same way. Deterministic.
// ------------------------------------------------------------------------------------------------
// 1024 threads: 32 split groups x 32 elements; a thread sums its groups' partials (s = sg, sg + 32, ...: <= 5 at
// C2, all loads in flight) in order, then one thread per element the 32 group sums in order (deterministic).
constexpr int kRedSG = 32;
__global__ void __launch_bounds__(1024) k_reduce(ReduceArgs p, int eblocks) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  __shared__ double2 sh[kRedSG][32];
  const int dom = blockIdx.y;
  const int el = threadIdx.x & 31, sg = threadIdx.x >> 5;
  const long long per_dom = (long long)p.mrows * p.ncols;
  if ((int)blockIdx.x < eblocks) {
    const long long e = (long long)blockIdx.x * 32 + el;
    double sr = 0.0, si = 0.0;
    if (e < per_dom) {
      const double2* src = p.part + (long long)dom * p.nsplit * per_dom + e;
      int s = sg;
      for (; s + 3 * kRedSG < p.nsplit; s += 4 * kRedSG) {  // 4 loads in flight, added in order
        double2 v[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) v[k] = src[(long long)(s + kRedSG * k) * per_dom];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          sr += v[k].x;
          si += v[k].y;
        }
      }
      for (; s < p.nsplit; s += kRedSG) {
        const double2 v = src[(long long)s * per_dom];
        sr += v.x;
        si += v.y;
      }
    }
    sh[sg][el] = make_double2(sr, si);
    __syncthreads();
    if (sg == 0 && e < per_dom) {
      double tr = 0.0, ti = 0.0;
#pragma unroll 8
      for (int q = 0; q < kRedSG; ++q) {
        tr += sh[q][el].x;
        ti += sh[q][el].y;
      }
      const int m = (int)(e / p.ncols);
      const double f = p.scale * (p.D ? p.D[(long long)dom * p.mrows + m] : 1.0);
      const double2 o = make_double2(tr * f, ti * f);
      const long long idx = (long long)dom * per_dom + e;
      p.out[idx] = o;
      if (p.cprime) {
        if (p.W) {  // exactly unitary factor: C'' = (e^{-i eps D_m} - 1) C (W precomputed)
          const double2 w = p.W[(long long)dom * p.mrows + m];
          p.cprime[idx] = make_double2(w.x * o.x - w.y * o.y, w.x * o.y + w.y * o.x);
        } else {
          p.cprime[idx] = make_double2(p.eps * o.y, -p.eps * o.x);  // -i eps (D C)
        }
      }
    }
  } else {
    const int n = ((int)blockIdx.x - eblocks) * 32 + el;
    double acc = 0.0;
    if (n < p.ncols) {
      const double* ns = p.normp + (long long)dom * p.nsplit * p.ncols + n;
      for (int s = sg; s < p.nsplit; s += kRedSG) acc += ns[(long long)s * p.ncols];
    }
    sh[sg][el].x = acc;
    __syncthreads();
    if (sg == 0 && n < p.ncols) {
      double t = 0.0;
      for (int q = 0; q < kRedSG; ++q) t += sh[q][el].x;
      p.s[(long long)dom * p.ncols + n] = p.scale * t;
    }
  }
}

cudaError_t launch_reduce(const ReduceArgs& a, cudaStream_t st) {
  const long long per_dom = (long long)a.mrows * a.ncols;
  const int eblocks = (int)((per_dom + 31) / 32);
  const int nblocks = a.s ? (a.ncols + 31) / 32 : 0;
  dim3 grid(eblocks + nblocks, a.ndom);
  launch_k(k_reduce, grid, kRedSG * 32, 0, st, a, eblocks);
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// n_s = sqrt(s_s / (s_s + eps^2 Re[(DC)_s^H G (DC)_s])). Block per (domain, orbital s): warps take
// projector rows u, lanes run over v (coalesced rows of G), fixed-order warp and block reductions.
// ------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_nlnorm(int nproj, int norb, double eps2, const double2* __restrict__ G,
                                                const double2* __restrict__ DC, const double* __restrict__ s,
                                                double* __restrict__ nfac, double2* __restrict__ Cp) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  extern __shared__ double2 dcs[];  // DC[:, col]
  __shared__ double wq[8];
  const int dom = blockIdx.y, col = blockIdx.x;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const double2* Gd = G + (long long)dom * nproj * nproj;
  const double2* Cd = DC + (long long)dom * nproj * norb;
  for (int u = threadIdx.x; u < nproj; u += blockDim.x) dcs[u] = Cd[(long long)u * norb + col];
  __syncthreads();
  double q = 0.0;
  if (nproj <= 64) {  // the warp's (up to) 8 rows with all G loads in flight and the shuffle trees interleaved;
                      // per row the same fma chain and tree as the loop below (bitwise the same q)
    double tr[8], ti[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const int u = warp + 8 * k;
      tr[k] = 0.0;
      ti[k] = 0.0;
#pragma unroll
      for (int t = 0; t < 2; ++t) {
        const int v = lane + 32 * t;
        if (u < nproj && v < nproj) {
          const double2 gv = Gd[(long long)u * nproj + v], c = dcs[v];
          tr[k] = fma(gv.x, c.x, fma(-gv.y, c.y, tr[k]));
          ti[k] = fma(gv.x, c.y, fma(gv.y, c.x, ti[k]));
        }
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        tr[k] += __shfl_xor_sync(0xffffffffu, tr[k], o);
        ti[k] += __shfl_xor_sync(0xffffffffu, ti[k], o);
      }
    }
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const int u = warp + 8 * k;
      if (u < nproj) {
        const double2 cu = dcs[u];
        q = fma(cu.x, tr[k], fma(cu.y, ti[k], q));
      }
    }
  } else
  for (int u = warp; u < nproj; u += 8) {
    const double2* Gu = Gd + (long long)u * nproj;
    double tr = 0.0, ti = 0.0;
    for (int v = lane; v < nproj; v += 32) {
      const double2 gv = Gu[v], c = dcs[v];
      tr = fma(gv.x, c.x, fma(-gv.y, c.y, tr));
      ti = fma(gv.x, c.y, fma(gv.y, c.x, ti));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      tr += __shfl_xor_sync(0xffffffffu, tr, o);
      ti += __shfl_xor_sync(0xffffffffu, ti, o);
    }
    const double2 cu = dcs[u];
    q = fma(cu.x, tr, fma(cu.y, ti, q));  // Re(conj(cu) * t)
  }
  if (lane == 0) wq[warp] = q;
  __syncthreads();
  if (threadIdx.x == 0) {
    double tq = 0.0;
    for (int w = 0; w < 8; ++w) tq += wq[w];
    const double sv = s[(long long)dom * norb + col];
    const double n = sqrt(sv / (sv + eps2 * tq));
    nfac[(long long)dom * norb + col] = n;
    wq[0] = n;
  }
  __syncthreads();
  const double n = wq[0];  // C'' = C' n (the GEMM-2 epilogue is then Psi n + B C'')
  for (int u = threadIdx.x; u < nproj; u += blockDim.x) {
    double2& c = Cp[((long long)dom * nproj + u) * norb + col];
    c = make_double2(c.x * n, c.y * n);
  }
}

cudaError_t launch_nlnorm(int ndom, int nproj, int norb, double eps, const double2* G, const double2* DC,
                          const double* s, double* nfac, double2* Cp, cudaStream_t st) {
  dim3 grid(norb, ndom);
  launch_k(k_nlnorm, grid, 256, nproj * sizeof(double2), st, nproj, norb, eps * eps, G, DC, s, nfac, Cp);
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// Two consecutive nonlocal factors N(N(Psi)) as ONE factor (lfd_step_sequence; no Psi is observed
// between them). With L(Psi) = Psi + c B D C(Psi), c = -i eps, C = dV B^H Psi and G = dV B^H B:
//   L(L(Psi)) = Psi + B X,   X = M C,   M = 2c D + c^2 D G D,
// and since each N restores the column norm, N(N(Psi))_s = L^2(Psi)_s * sqrt(s_s / ||L^2 Psi_s||^2) with
//   ||Psi_s + B X_s||^2 = s_s + 2 Re(C_s^H X_s) + X_s^H G X_s,  2 Re(C^H X) = -2 eps^2 (DC)^H G (DC).
// Input DC = D C (k_reduce output); writes X to cprime and the factor to nfac. Block per (orbital, dom).
// ------------------------------------------------------------------------------------------------
__global__ void __launch_bounds__(256) k_nlmerge(int nproj, int norb, double eps, const double2* __restrict__ G,
                                                 const double* __restrict__ D, const double2* __restrict__ DC,
                                                 const double* __restrict__ s, double2* __restrict__ X,
                                                 double* __restrict__ nfac) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  extern __shared__ double2 sh[];  // dc[np] | x[np]
  double2* dcs = sh;
  double2* xs = sh + nproj;
  __shared__ double wq[2][8];
  const int dom = blockIdx.y, col = blockIdx.x;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const double2* Gd = G + (long long)dom * nproj * nproj;
  const double* Dd = D + (long long)dom * nproj;
  for (int u = threadIdx.x; u < nproj; u += blockDim.x) dcs[u] = DC[((long long)dom * nproj + u) * norb + col];
  __syncthreads();
  auto gdot = [&](int u, const double2* vec, double& tr, double& ti) {  // (G vec)_u, warp-wide
    const double2* Gu = Gd + (long long)u * nproj;
    tr = 0.0;
    ti = 0.0;
    for (int v = lane; v < nproj; v += 32) {
      const double2 gv = Gu[v], c = vec[v];
      tr = fma(gv.x, c.x, fma(-gv.y, c.y, tr));
      ti = fma(gv.x, c.y, fma(gv.y, c.x, ti));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      tr += __shfl_xor_sync(0xffffffffu, tr, o);
      ti += __shfl_xor_sync(0xffffffffu, ti, o);
    }
  };
  double q1 = 0.0, q2 = 0.0;
  for (int u = warp; u < nproj; u += 8) {
    double yr, yi;
    gdot(u, dcs, yr, yi);
    const double2 cu = dcs[u];
    q1 = fma(cu.x, yr, fma(cu.y, yi, q1));  // Re(conj(DC_u) (G DC)_u)
    const double du = Dd[u];
    // X_u = -2 i eps DC_u - eps^2 D_u (G DC)_u
    const double2 x = make_double2(2.0 * eps * cu.y - eps * eps * du * yr, -2.0 * eps * cu.x - eps * eps * du * yi);
    if (lane == 0) xs[u] = x;
  }
  __syncthreads();
  for (int u = warp; u < nproj; u += 8) {
    double zr, zi;
    gdot(u, xs, zr, zi);
    const double2 xu = xs[u];
    q2 = fma(xu.x, zr, fma(xu.y, zi, q2));  // Re(conj(X_u) (G X)_u)
  }
  if (lane == 0) {
    wq[0][warp] = q1;
    wq[1][warp] = q2;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    double t1 = 0.0, t2 = 0.0;
    for (int w = 0; w < 8; ++w) {
      t1 += wq[0][w];
      t2 += wq[1][w];
    }
    const double sv = s[(long long)dom * norb + col];
    const double n = sqrt(sv / (sv - 2.0 * eps * eps * t1 + t2));
    nfac[(long long)dom * norb + col] = n;
    wq[0][0] = n;
  }
  __syncthreads();
  const double n = wq[0][0];  // X'' = X n (the GEMM-2 epilogue is then Psi n + B X'')
  for (int u = threadIdx.x; u < nproj; u += blockDim.x)
    X[((long long)dom * nproj + u) * norb + col] = make_double2(xs[u].x * n, xs[u].y * n);
}

cudaError_t launch_nlmerge(int ndom, int nproj, int norb, double eps, const double2* G, const double* D,
                           const double2* DC, const double* s, double2* X, double* nfac, cudaStream_t st) {
  dim3 grid(norb, ndom);
  launch_k(k_nlmerge, grid, 256, 2 * nproj * sizeof(double2), st, nproj, norb, eps, G, D, DC, s, X, nfac);
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// Projection carry (no GEMM): the GEMM-2 that just ran wrote Psi_new = (Psi + B X) diag(n), so
//   C_new = dV B^H Psi_new = (C + G X) diag(n)       (G = dV B^H B, exact identity)
// and, with DC = D C, DC_new = (DC + D (G X)) diag(n); C'_new = -i eps DC_new. The column norms are
// unchanged (n restores them), so s is kept. Block per (orbital s, domain); column s only is read and
// written (X and DC are read into shared memory before any write). Replaces GEMM-1 + k_reduce of the
// next nonlocal factor when nothing touched Psi in between (lfd_step: N of step n, then N of n+1).
// ------------------------------------------------------------------------------------------------
template <bool kNorm>
__global__ void __launch_bounds__(256) k_nlcarry(int nproj, int norb, double eps, const double2* __restrict__ G,
                                                 const double* __restrict__ D, double2* DC, double2* X,
                                                 const double* __restrict__ s, double* nfac,
                                                 const double2* __restrict__ W) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  extern __shared__ double2 sh[];  // x[np] | dc[np] (dc is overwritten with DC_new)
  double2* xs = sh;
  double2* dcs = sh + nproj;
  double* ds = reinterpret_cast<double*>(sh + 2 * nproj);  // D[u], staged with x and dc
  __shared__ double wq[8];
  const int dom = blockIdx.y, col = blockIdx.x;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const double2* Gd = G + (long long)dom * nproj * nproj;
  const double* Dd = D + (long long)dom * nproj;
  const long long cb = (long long)dom * nproj * norb + col;
  for (int u = threadIdx.x; u < nproj; u += blockDim.x) {
    xs[u] = X[cb + (long long)u * norb];
    dcs[u] = DC[cb + (long long)u * norb];
    ds[u] = Dd[u];
  }
  __syncthreads();
  const double n = nfac[(long long)dom * norb + col];
  // (G v)_u, warp-wide (lanes over the row of G), fixed-order shuffle tree
  auto gdot = [&](int u, const double2* v, double& tr, double& ti) {
    const double2* Gu = Gd + (long long)u * nproj;
    tr = 0.0;
    ti = 0.0;
    for (int w = lane; w < nproj; w += 32) {
      const double2 gv = Gu[w], x = v[w];
      tr = fma(gv.x, x.x, fma(-gv.y, x.y, tr));
      ti = fma(gv.x, x.y, fma(gv.y, x.x, ti));
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
      tr += __shfl_xor_sync(0xffffffffu, tr, o);
      ti += __shfl_xor_sync(0xffffffffu, ti, o);
    }
  };
  // nproj <= 64: the warp's (up to) 8 rows with all their G loads in flight at once and the 16 shuffle trees
  // interleaved (per row the same fma chain and tree as gdot: bitwise the same values)
  auto gdot8 = [&](const double2* v, double (&tr)[8], double (&ti)[8]) {
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const int u = warp + 8 * k;
      tr[k] = 0.0;
      ti[k] = 0.0;
#pragma unroll
      for (int t = 0; t < 2; ++t) {
        const int w = lane + 32 * t;
        if (u < nproj && w < nproj) {
          const double2 gv = Gd[(long long)u * nproj + w], x = v[w];
          tr[k] = fma(gv.x, x.x, fma(-gv.y, x.y, tr[k]));
          ti[k] = fma(gv.x, x.y, fma(gv.y, x.x, ti[k]));
        }
      }
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        tr[k] += __shfl_xor_sync(0xffffffffu, tr[k], o);
        ti[k] += __shfl_xor_sync(0xffffffffu, ti[k], o);
      }
    }
  };
  const bool small = nproj <= 64;
  double gr[8], gi[8];
  auto row = [&](int u, double tr, double ti) {
    if (lane == 0) {
      const double du = ds[u];
      const double2 d = make_double2(fma(n, dcs[u].x, du * tr), fma(n, dcs[u].y, du * ti));
      DC[cb + (long long)u * norb] = d;
      if (W) {  // exactly unitary factor (D == 1 passed, n == 1): C''_new = W C_new
        const double2 w = W[(long long)dom * nproj + u];
        X[cb + (long long)u * norb] = make_double2(w.x * d.x - w.y * d.y, w.x * d.y + w.y * d.x);
      } else if (!kNorm) {
        X[cb + (long long)u * norb] = make_double2(eps * d.y, -eps * d.x);  // -i eps DC_new
      }
      dcs[u] = d;  // only this lane reads dcs[u] above
    }
  };
  if (small) {  // rows u = warp + 8 k, compile-time k (no register-array selects)
    gdot8(xs, gr, gi);
#pragma unroll
    for (int k = 0; k < 8; ++k)
      if (warp + 8 * k < nproj) row(warp + 8 * k, gr[k], gi[k]);
  } else {
    for (int u = warp; u < nproj; u += 8) {
      double tr, ti;
      gdot(u, xs, tr, ti);
      row(u, tr, ti);
    }
  }
  if (!kNorm) return;
  // n_s of the next factor from the Gram closed form (as k_nlnorm), on DC_new
  __syncthreads();
  double q = 0.0;
  if (small) {
    gdot8(dcs, gr, gi);
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      const int u = warp + 8 * k;
      if (u < nproj) {
        const double2 cu = dcs[u];
        q = fma(cu.x, gr[k], fma(cu.y, gi[k], q));  // Re(conj(cu) (G DC)_u)
      }
    }
  } else {
    for (int u = warp; u < nproj; u += 8) {
      double tr, ti;
      gdot(u, dcs, tr, ti);
      const double2 cu = dcs[u];
      q = fma(cu.x, tr, fma(cu.y, ti, q));  // Re(conj(cu) (G DC)_u)
    }
  }
  if (lane == 0) wq[warp] = q;
  __syncthreads();
  if (threadIdx.x == 0) {
    double tq = 0.0;
    for (int w = 0; w < 8; ++w) tq += wq[w];
    const double sv = s[(long long)dom * norb + col];
    const double nn = sqrt(sv / (sv + eps * eps * tq));
    nfac[(long long)dom * norb + col] = nn;
    wq[0] = nn;
  }
  __syncthreads();
  const double nn = wq[0];  // C'' = -i eps DC_new n_new
  for (int u = threadIdx.x; u < nproj; u += blockDim.x)
    X[cb + (long long)u * norb] = make_double2(eps * dcs[u].y * nn, -eps * dcs[u].x * nn);
}

cudaError_t launch_nlcarry(int ndom, int nproj, int norb, double eps, const double2* G, const double* D,
                           double2* DC, double2* X, const double* s, double* nfac, bool with_norm,
                           const double2* W, cudaStream_t st) {
  dim3 grid(norb, ndom);
  if (with_norm && !W)
    launch_k(k_nlcarry<true>, grid, 256, 2 * nproj * sizeof(double2) + nproj * sizeof(double), st, nproj, norb, eps, G, D, DC, X, s, nfac, W);
  else
    launch_k(k_nlcarry<false>, grid, 256, 2 * nproj * sizeof(double2) + nproj * sizeof(double), st, nproj, norb, eps, G, D, DC, X, s, nfac, W);
  return cudaGetLastError();
}

// ------------------------------------------------------------------------------------------------
// GEMM-2 (persistent, any nproj): psi[r][n] <- nfac[n] psi[r][n] + sum_m B[r][m] Cp[m][n] for every
// (dom, 64-row block, 64-column tile) work item; K = nproj in chunks of kKC2 through a TMA tensor-map
// ring (full/empty mbarriers; thread 0 refills a stage once every warp has released it).
// ------------------------------------------------------------------------------------------------
// Tile shapes of k_gemm2: kRT rows x kCT orbital columns, 8 warps of 32 x 16 (the same fragments): 64 x 64 (2 x 4
// warps, 3-stage ring) or, for narrow orbital sets (norb <= 32, C5's first row), 128 x 32 (4 x 2 warps, 2 stages)
template <int kRT, int kCT>
struct G2Shape {
  static constexpr int WN = kCT / 16, WM = 8 / WN;
  static constexpr int LDC = kCT + 2;                       // == 2 mod 8 complex: conflict-free fragment loads
  static constexpr int Stages = kRT == 64 ? 3 : 2;
  static constexpr int StageBytes = kRT * kLdA2 * 16 + kKC2 * LDC * 16;
  static constexpr int Smem = Stages * StageBytes + 2 * Stages * 8;
};

// returns a value computed from the chunk's last shared loads (for mbar_release)
template <int kLDC>
__device__ __forceinline__ double gemm2_chunk(const double2* As, const double2* Cs, int wm, int wn, int g, int t,
                                              Frag& acc) {
  double2 a[4], c[2];
#pragma unroll
  for (int kk = 0; kk < kKC2; kk += 4) {
    const int k = kk + t;
#pragma unroll
    for (int mi = 0; mi < 4; ++mi) a[mi] = As[(wm * 32 + mi * 8 + g) * kLdA2 + k];
#pragma unroll
    for (int ni = 0; ni < 2; ++ni) c[ni] = Cs[k * kLDC + wn * 16 + ni * 8 + g];
    mma_4x2(acc, a, c);
  }
  return ((a[0].x + a[1].x) + (a[2].x + a[3].x)) + (c[0].x + c[1].x);
}

template <int kRT, int kCT>
__global__ void __launch_bounds__(kThreads, 1) k_gemm2(const __grid_constant__ CUtensorMap tA,
                                                       const __grid_constant__ CUtensorMap tC, Gemm2Args p) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  using S = G2Shape<kRT, kCT>;
  constexpr int kSt = S::Stages;
  extern __shared__ __align__(128) unsigned char smem[];
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + kSt * S::StageBytes);
  uint64_t* empty = full + kSt;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int g = lane >> 2, t = lane & 3;
  const int wm = warp / S::WN, wn = warp % S::WN;
  const int rblocks = (int)((p.ng + kRT - 1) / kRT);
  const int ntn = (p.norb + kCT - 1) / kCT;
  const long long items = (long long)p.ndom * rblocks * ntn;
  const int nk = (p.nproj + kKC2 - 1) / kKC2;

  if (tid == 0) {
    for (int s = 0; s < kSt; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], kConsWarps1);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  // This CTA's chunk sequence: items blockIdx.x, +gridDim.x, ...; nk chunks each.
  const long long my_items = (items > blockIdx.x) ? (items - 1 - blockIdx.x) / gridDim.x + 1 : 0;
  const long long total = my_items * nk;

  auto decode = [&](long long item, int& dom, long long& r0, int& n0) {
    const long long per_dom = (long long)rblocks * ntn;
    dom = (int)(item / per_dom);
    const long long rem = item - dom * per_dom;
    const long long rb = rem / ntn;
    r0 = rb * kRT;
    n0 = (int)(rem - rb * ntn) * kCT;
  };

  // chunk gc -> stage gc % kSt: two tiled tensor copies, the B block [kRT rows][kKC2 + 4 complex]
  // (columns past nproj and rows past ng are zero fill) and the C'' block [kKC2 rows][kCT + 2 complex]
  auto issue = [&](long long gc) {  // thread 0 only
    const int stage = (int)(gc % kSt);
    const long long item = blockIdx.x + (gc / nk) * gridDim.x;
    const int kc = (int)(gc % nk);
    int dom, n0;
    long long r0;
    decode(item, dom, r0, n0);
    double2* As = reinterpret_cast<double2*>(smem + stage * S::StageBytes);
    double2* Cs = As + kRT * kLdA2;
    mbar_expect_tx(&full[stage], (uint32_t)S::StageBytes);
    tma_3d(As, &tA, 2 * kc * kKC2, (int)r0, dom, &full[stage]);
    tma_3d(Cs, &tC, 2 * n0, kc * kKC2, dom, &full[stage]);
  };

  if (tid == 0)
    for (long long s = 0; s < kSt && s < total; ++s) issue(s);

  long long gc = 0;
  for (long long it = 0; it < my_items; ++it) {
    const long long item = blockIdx.x + it * gridDim.x;
    int dom, n0;
    long long r0;
    decode(item, dom, r0, n0);
    const double2* psi = p.psi + (long long)dom * p.ng * p.norb;
    double2* pout = (p.psi_out ? p.psi_out : p.psi) + (long long)dom * p.ng * p.norb;
    if (tid == 32) {  // Psi rows of this item (first) and of the next one -> L2, read in the epilogue
      if (it == 0) l2_prefetch(psi + r0 * p.norb, (uint32_t)(min((long long)kRT, p.ng - r0) * p.norb * 16));
      if (it + 1 < my_items) {
        int d1, n1;
        long long q1;
        decode(item + gridDim.x, d1, q1, n1);
        l2_prefetch(p.psi + ((long long)d1 * p.ng + q1) * p.norb,
                    (uint32_t)(min((long long)kRT, p.ng - q1) * p.norb * 16));
      }
    }
    Frag acc;
    acc.zero();
    for (int kc = 0; kc < nk; ++kc, ++gc) {
      const int stage = (int)(gc % kSt);
      mbar_wait(&full[stage], (uint32_t)((gc / kSt) & 1));
      const double2* As = reinterpret_cast<const double2*>(smem + stage * S::StageBytes);
      const double2* Cs = As + kRT * kLdA2;
      const double dep = gemm2_chunk<S::LDC>(As, Cs, wm, wn, g, t, acc);  // the K tail is zero fill
      mbar_release(&empty[stage], dep, lane == 0);
      if (tid == 0 && gc + kSt < total) {  // refill once every warp has released the stage
        mbar_wait(&empty[stage], (uint32_t)((gc / kSt) & 1));
        issue(gc + kSt);
      }
    }
    // epilogue: Psi <- n_s (Psi + B C'); all 16 loads (L2 hits) are issued before any store
    const double* nf = p.nfac + (long long)dom * p.norb;
    double2 pv[4][2][2];
#pragma unroll
    for (int mi = 0; mi < 4; ++mi) {
      const long long r = r0 + wm * 32 + mi * 8 + g;
#pragma unroll
      for (int ni = 0; ni < 2; ++ni)
#pragma unroll
        for (int c = 0; c < 2; ++c) {
          const int col = n0 + wn * 16 + ni * 8 + 2 * t + c;
          pv[mi][ni][c] = (r < p.ng && col < p.norb) ? psi[r * p.norb + col] : cz();
        }
    }
#pragma unroll
    for (int ni = 0; ni < 2; ++ni)
#pragma unroll
      for (int c = 0; c < 2; ++c) {
        const int col = n0 + wn * 16 + ni * 8 + 2 * t + c;
        if (col >= p.norb) continue;
        const double f = nf[col];
#pragma unroll
        for (int mi = 0; mi < 4; ++mi) {
          const long long r = r0 + wm * 32 + mi * 8 + g;
          if (r < p.ng)
            pout[r * p.norb + col] =
                make_double2(fma(f, pv[mi][ni][c].x, acc.re(mi, ni, c)), fma(f, pv[mi][ni][c].y, acc.im(mi, ni, c)));
        }
      }
  }
}

// Tile geometry of k_gemm2_tma (nproj <= 64): a 2-deep ring of [64 rows][lda] B tiles (lda == 4 mod 8
// complex: conflict-free A-fragment LDS.128) and C' of one (domain, column tile) resident.
constexpr int kFullStages = 2;
constexpr int kFullLdaMax = 68;
constexpr int kFullABytes = kTile * kFullLdaMax * 16;     // [64 rows][<=68] complex
constexpr int kFullCBytes = kTile * kLd1 * 16;            // [<=64 proj][66] complex
constexpr int kFullSmem = kFullStages * kFullABytes + kFullCBytes + 4 * 8;
__host__ __device__ constexpr int full_lda(int np) { return ((np + 3) / 4 * 4) % 8 == 0 ? (np + 3) / 4 * 4 + 4 : (np + 3) / 4 * 4; }

// ------------------------------------------------------------------------------------------------
// GEMM-2, TMA tensor-map variant for nproj <= 64 (the paper-shaped case). Thread 0 issues, per work item,
// ONE tiled tensor copy of the item's 64 B rows (box [64 rows][lda complex]; the columns past nproj are
// zero fill, which pads the smem rows to lda == 4 mod 8 complex so the A-fragment LDS.128 are
// conflict free) into a 2-deep ring (full/empty mbarriers), plus an L2 prefetch of the item's Psi rows
// for the epilogue. C' of the current (domain, column tile) stays resident (one tensor
// copy when it changes), the K loop is fully unrolled for nproj = 64, the epilogue's Psi loads are
// issued mid-loop and Psi <- n_s (Psi + B C') is written in place.
// ------------------------------------------------------------------------------------------------
template <int kNP, bool kOut>
__global__ void __launch_bounds__(kThreads, 1) k_gemm2_tma(const __grid_constant__ CUtensorMap tB,
                                                             const __grid_constant__ CUtensorMap tC, Gemm2Args p) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  extern __shared__ __align__(128) unsigned char smem[];
  double2* Cs = reinterpret_cast<double2*>(smem + kFullStages * kFullABytes);
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + kFullStages * kFullABytes + kFullCBytes);
  uint64_t* empty = full + kFullStages;
  uint64_t* cbar = empty + kFullStages;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int np = kNP > 0 ? kNP : p.nproj;
  const int lda = full_lda(np);
  const long long rblocks = (p.ng + kTile - 1) / kTile;
  const int ntn = (p.norb + kTile - 1) / kTile;
  const long long items = (long long)p.ndom * ntn * rblocks;
  const long long my_items = (items > blockIdx.x) ? (items - 1 - blockIdx.x) / gridDim.x + 1 : 0;
  constexpr int kNK4 = kNP > 0 ? (kNP + 3) / 4 : 16;
  const int nk4 = (np + 3) / 4;
  const int kmid = (kNP > 0 ? kNK4 : nk4) / 2;  // k step at which the epilogue's Psi loads are issued

  if (tid == 0) {
    for (int s = 0; s < kFullStages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], kConsWarps1);
    }
    mbar_init(cbar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  auto decode = [&](long long j, int& dom, int& n0, long long& r0) {
    const long long item = blockIdx.x + j * gridDim.x;
    const long long per_dom = (long long)ntn * rblocks;
    dom = (int)(item / per_dom);
    const long long rem = item - dom * per_dom;
    const int nt = (int)(rem / rblocks);
    n0 = nt * kTile;
    r0 = (rem - (long long)nt * rblocks) * kTile;
  };

  // item j -> stage j % kFullStages: ONE tensor copy of its B rows + L2 prefetch of its Psi rows
  auto issue = [&](long long j) {
    const int s = (int)(j % kFullStages);
    int dom, n0;
    long long r0;
    decode(j, dom, n0, r0);
    mbar_expect_tx(&full[s], (uint32_t)(kTile * lda * 16));
    tma_3d(smem + s * kFullABytes, &tB, 0, (int)r0, dom, &full[s]);
    const long long rows = min((long long)kTile, p.ng - r0);
    l2_prefetch(p.psi + ((long long)dom * p.ng + r0) * p.norb, (uint32_t)(rows * p.norb * 16));
  };
  if (tid == 0)
    for (long long j = 0; j < kFullStages && j < my_items; ++j) issue(j);

  const int g = lane >> 2, t = lane & 3;
  const int wm = warp >> 2, wn = warp & 3;
  int cur_dom = -1, cur_n0 = -1;
  uint32_t cphase = 0;
  for (long long j = 0; j < my_items; ++j) {
    int dom, n0;
    long long r0;
    decode(j, dom, n0, r0);
    if (dom != cur_dom || n0 != cur_n0) {  // (re)load C'[dom][:, n0:n0+64] once every consumer is past Cs
      asm volatile("bar.sync 1, %0;" ::"n"(kConsWarps1 * 32));
      if (tid == 0) {
        mbar_expect_tx(cbar, (uint32_t)(nk4 * 4 * kLd1 * 16));
        tma_3d(Cs, &tC, 2 * n0, 0, dom, cbar);
      }
      mbar_wait(cbar, cphase);
      cphase ^= 1;
      cur_dom = dom;
      cur_n0 = n0;
    }
    // skew: the second M-half of the warps starts half a K loop late, so each half's epilogue overlaps
    // the other half's DMMAs (the halves share only the B stage and C')
    if (j == 0 && wm == 1) asm volatile("bar.sync 2, %0;" ::"n"(kThreads));
    const int s = (int)(j % kFullStages);
    mbar_wait(&full[s], (uint32_t)((j / kFullStages) & 1));
    const double2* As = reinterpret_cast<const double2*>(smem + s * kFullABytes);
    Frag acc;
    acc.zero();
    // kOut: out of place (psi_out); else the in-place code path reads and writes one pointer
    double2* psi = p.psi + (long long)dom * p.ng * p.norb;
    double2* pout = kOut ? p.psi_out + (long long)dom * p.ng * p.norb : psi;
    double2 pv[4][2][2];
    auto load_pv = [&]() {
#pragma unroll
      for (int mi = 0; mi < 4; ++mi) {
        const long long r = r0 + wm * 32 + mi * 8 + g;
#pragma unroll
        for (int ni = 0; ni < 2; ++ni)
#pragma unroll
          for (int c = 0; c < 2; ++c) {
            const int col = n0 + wn * 16 + ni * 8 + 2 * t + c;
            pv[mi][ni][c] = (r < p.ng && col < p.norb) ? psi[r * p.norb + col] : cz();
          }
      }
    };
    double2 a[4], c[2];
#pragma unroll
    for (int kk = 0; kk < kNK4; ++kk) {
      if (kNP == 0 && kk >= nk4) break;
      if (kk == kmid) {
        load_pv();  // Psi loads (L2 hits) in flight during the second half
        if (j == 0 && wm == 0) asm volatile("bar.arrive 2, %0;" ::"n"(kThreads));
      }
      const int k = kk * 4 + t;
#pragma unroll
      for (int mi = 0; mi < 4; ++mi) a[mi] = As[(wm * 32 + mi * 8 + g) * lda + k];
#pragma unroll
      for (int ni = 0; ni < 2; ++ni) c[ni] = Cs[k * kLd1 + wn * 16 + ni * 8 + g];
      mma_4x2(acc, a, c);
    }
    // the stage's last loads have returned before it is released (lfd_tma.cuh)
    mbar_release(&empty[s], ((a[0].x + a[1].x) + (a[2].x + a[3].x)) + (c[0].x + c[1].x), lane == 0);
    if (tid == 0 && j + kFullStages < my_items) {  // refill the stage once every warp has released it
      mbar_wait(&empty[s], (uint32_t)((j / kFullStages) & 1));
      issue(j + kFullStages);
    }
    // epilogue: Psi <- n_s (Psi + B C')
    const double* nf = p.nfac + (long long)dom * p.norb;
#pragma unroll
    for (int ni = 0; ni < 2; ++ni)
#pragma unroll
      for (int c = 0; c < 2; ++c) {
        const int col = n0 + wn * 16 + ni * 8 + 2 * t + c;
        if (col >= p.norb) continue;
        const double f = nf[col];
#pragma unroll
        for (int mi = 0; mi < 4; ++mi) {
          const long long r = r0 + wm * 32 + mi * 8 + g;
          if (r < p.ng)
            pout[r * p.norb + col] =
                make_double2(fma(f, pv[mi][ni][c].x, acc.re(mi, ni, c)), fma(f, pv[mi][ni][c].y, acc.im(mi, ni, c)));
        }
      }
  }
}

// B [dom][ng][nproj] (box [1][64 rows][lda]) and C' [dom][nproj][norb] (box [1][nproj][kLd1]).
static cudaError_t gemm2_maps(const Gemm2Args& a, CUtensorMap* tB, CUtensorMap* tC) {
  const int lda = full_lda(a.nproj);
  const uint64_t dB[3] = {(uint64_t)2 * a.nproj, (uint64_t)a.ng, (uint64_t)a.ndom};
  const uint64_t sB[2] = {(uint64_t)a.nproj * 16, (uint64_t)a.ng * a.nproj * 16};
  const uint32_t bB[3] = {(uint32_t)(2 * lda), kTile, 1};
  cudaError_t e = encode_tmap_f64(tB, 3, a.B, dB, sB, bB);
  if (e != cudaSuccess) return e;
  const uint64_t dC[3] = {(uint64_t)2 * a.norb, (uint64_t)a.nproj, (uint64_t)a.ndom};
  const uint64_t sC[2] = {(uint64_t)a.norb * 16, (uint64_t)a.nproj * a.norb * 16};
  // rows up to the K loop's multiple of 4: the rows past nproj are zero fill (never stale smem)
  const uint32_t bC[3] = {2 * kLd1, (uint32_t)((a.nproj + 3) / 4 * 4), 1};
  return encode_tmap_f64(tC, 3, a.Cp, dC, sC, bC);
}

cudaError_t launch_gemm2(const Gemm2Args& a, cudaStream_t st) {
  if (a.bsl) return launch_gemm2_i8(a, st);
  const long long rblocks = (a.ng + kTile - 1) / kTile;
  const long long items = (long long)a.ndom * rblocks * ((a.norb + kTile - 1) / kTile);
  const int grid = (int)(items < a.num_sms ? items : a.num_sms);
  if (a.nproj <= kTile) {
    CUtensorMap tB, tC;
    cudaError_t e = gemm2_maps(a, &tB, &tC);
    if (e != cudaSuccess) return e;
    const bool o = a.psi_out != nullptr;  // out of place (the self-consistent step's first factor)
    if (a.nproj == kTile) {
      if (o) launch_k(k_gemm2_tma<kTile, true>, grid, kThreads, kFullSmem + 16, st, tB, tC, a);
      else launch_k(k_gemm2_tma<kTile, false>, grid, kThreads, kFullSmem + 16, st, tB, tC, a);
    } else {
      if (o) launch_k(k_gemm2_tma<0, true>, grid, kThreads, kFullSmem + 16, st, tB, tC, a);
      else launch_k(k_gemm2_tma<0, false>, grid, kThreads, kFullSmem + 16, st, tB, tC, a);
    }
  } else {
    // B [dom][ng][nproj] (box [1][kRT rows][kKC2 + 4 complex]) and C'' [dom][nproj][norb] (box [1][kKC2][kCT + 2])
    const bool narrow = a.norb <= 32;
    const int rt = narrow ? 128 : kTile, ct = narrow ? 32 : kTile;
    CUtensorMap tA, tC;
    const uint64_t dA[3] = {(uint64_t)2 * a.nproj, (uint64_t)a.ng, (uint64_t)a.ndom};
    const uint64_t sA[2] = {(uint64_t)a.nproj * 16, (uint64_t)a.ng * a.nproj * 16};
    const uint32_t bA[3] = {2 * kLdA2, (uint32_t)rt, 1};
    cudaError_t e = encode_tmap_f64(&tA, 3, a.B, dA, sA, bA);
    if (e != cudaSuccess) return e;
    const uint64_t dC[3] = {(uint64_t)2 * a.norb, (uint64_t)a.nproj, (uint64_t)a.ndom};
    const uint64_t sC[2] = {(uint64_t)a.norb * 16, (uint64_t)a.nproj * a.norb * 16};
    const uint32_t bC[3] = {(uint32_t)(2 * (ct + 2)), kKC2, 1};
    e = encode_tmap_f64(&tC, 3, a.Cp, dC, sC, bC);
    if (e != cudaSuccess) return e;
    const long long items2 = (long long)a.ndom * ((a.ng + rt - 1) / rt) * ((a.norb + ct - 1) / ct);
    const int grid2 = (int)(items2 < a.num_sms ? items2 : a.num_sms);
    if (narrow) launch_k(k_gemm2<128, 32>, grid2, kThreads, G2Shape<128, 32>::Smem, st, tA, tC, a);
    else launch_k(k_gemm2<64, 64>, grid2, kThreads, G2Shape<64, 64>::Smem, st, tA, tC, a);
  }
  return cudaGetLastError();
}

cudaError_t gemm_set_attributes() {
  cudaError_t e = cudaSuccess;
  for (auto f : {k_gemm1<64, 64>, k_gemm1<32, 64>, k_gemm1<16, 64>, k_gemm1<64, 32>, k_gemm1<32, 32>,
                 k_gemm1<16, 32>}) {
    e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, gemm1_smem_bytes());
    if (e != cudaSuccess) return e;
  }
  for (auto f : {k_gemm2_tma<kTile, false>, k_gemm2_tma<0, false>, k_gemm2_tma<kTile, true>, k_gemm2_tma<0, true>}) {
    e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, kFullSmem + 16);
    if (e != cudaSuccess) return e;
  }
  // the nonlocal-coefficient kernels stage O(nproj) vectors in dynamic shared memory (nproj <= 2048)
  for (auto f : {k_nlcarry<true>, k_nlcarry<false>}) {
    e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 40 * 2048);
    if (e != cudaSuccess) return e;
  }
  e = cudaFuncSetAttribute(k_nlmerge, cudaFuncAttributeMaxDynamicSharedMemorySize, 32 * 2048);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_nlnorm, cudaFuncAttributeMaxDynamicSharedMemorySize, 16 * 2048);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(k_gemm2<128, 32>, cudaFuncAttributeMaxDynamicSharedMemorySize, G2Shape<128, 32>::Smem);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(k_gemm2<64, 64>, cudaFuncAttributeMaxDynamicSharedMemorySize, G2Shape<64, 64>::Smem);
}

}  // namespace lfd
