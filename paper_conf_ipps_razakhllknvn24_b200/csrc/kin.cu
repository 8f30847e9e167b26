// kin.cu -- local propagator kernels for sm_100a.
//
// Paper: Eq. 6 local factor exp(-i Delta h_loc) by the O(N) space-splitting stencil (P:68,
// P:76-80). Alg. 3-5 stream each line along the stencil axis with one thread team per
// (other two coordinates, orbital block) and carry the pre-update neighbour (psi_old) so the update is
// in place. Here the same streaming structure keeps the pre-update values still needed in registers
// (the psi_old carry of Alg. 3 l.6), so each pass reads and writes Psi exactly once, and lanes
// run over consecutive orbitals (the paper's orbital-innermost SoA) so every access is coalesced.
//
// K_d = E_d(Delta/2) O_d(Delta) E_d(Delta/2) (readings R4/R5): E links (2m,2m+1), O links (2m+1,2m+2)
// plus the periodic wrap (n-1,0); zero BC turns missing links into the on-site factor e^{-i tau t_d}.
//
// Two passes per step:  (1) Psi <- K_x (Phi . Psi)   (k_kin, axis x, pre-phase)
//                       (2) Psi <- Phi . K_y K_z Psi (k_kin_yz; K_y and K_z commute exactly, R6)
// (k_kin also runs the y and z passes separately where k_kin_yz does not apply, nz > 80.)
//
// Scaled pair form (kS). Every pair block is  e^{-i tau t} [[c, i s e^{i theta}], [i s e^{-i theta}, c]]
// with c = cos(tau t), s = sin(tau t) (real). Pulling e^{-i tau t} c out of every block leaves
//     psi'_i = psi_i + w psi_j,   w = i tan(tau t) e^{+-i theta}      (4 DFMA per output instead of 8)
// and a factor that is the SAME for every grid point: each point sits in exactly one link per sweep,
// so K_d = e^{-2 i Delta t_d} c1_d^2 c2_d K~_d (c1 = cos(Delta t_d / 2), c2 = cos(Delta t_d)); zero-BC
// singletons keep their relative factor 1/c. The product over d of those scalars, g, is folded into
// Phi as sqrt(g) (Phi is applied once before and once after the kinetic sweeps). Exactly the same
// operator; used when every c >= 1/2 (else the general 2x2 form runs). The FP64 pipe (not tensor) is
// what bounds these sweeps next to HBM on B200 (DFMA 34 TF/s), so halving the FP64 work matters.
#include <cmath>
#include <type_traits>

#include "lfd_coef.cuh"
#include "lfd_complex.cuh"
#include "lfd_internal.h"
#include "lfd_march.cuh"
#include "lfd_tma.cuh"

namespace lfd {

__global__ void k_coef(CoefParams p, int dom0, int count, double hx, double hy, double hz, double dt,
                       DomCoef* __restrict__ coef) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= count) return;
  coef[dom0 + i] = make_coef(p.A[i], hx, hy, hz, dt);
}

// The same table from A in DEVICE memory ([ndom][3]): step-invariant kernel parameters, so a captured CUDA
// graph of several steps replays with new A values (lfd_step_graph).
__global__ void k_coef_dev(const double* __restrict__ A, int ndom, double hx, double hy, double hz, double dt,
                           DomCoef* __restrict__ coef) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= ndom) return;
  const double a[3] = {A[3 * i], A[3 * i + 1], A[3 * i + 2]};
  coef[i] = make_coef(a, hx, hy, hz, dt);
}

cudaError_t launch_coef_dev(const Geometry& g, const double* A, DomCoef* coef, cudaStream_t st) {
  launch_k(k_coef_dev, (g.ndom + 127) / 128, 128, 0, st, A, g.ndom, g.hx, g.hy, g.hz, g.dt, coef);
  return cudaGetLastError();
}

cudaError_t launch_coef(const Geometry& g, const CoefParams& p, int dom0, int count, DomCoef* coef,
                        cudaStream_t st) {
  launch_k(k_coef, (count + 127) / 128, 128, 0, st, p, dom0, count, g.hx, g.hy, g.hz, g.dt, coef);
  return cudaGetLastError();
}

// Phi(r) = e^{-i (Delta/2) v_loc(r)} (Strang placement of the potential, reading R7), times the
// constant sqrt(g) of the scaled pair form (1 for the general form).
// The kernel also keeps a copy of v_loc for lfd_energy (vcopy may alias v: then it is not written).
// With cf.count > 0 the first block also writes the coefficient tables of a pending lfd_set_vector_potential.
// (__launch_bounds__(256, 4): 64 registers instead of 126 -- the coefficient write of block 0 and sincos's
// never-taken large-argument path spill instead; 4 CTAs per SM: ncu 7.7 -> 6.6 us at C2)
template <class C>
__global__ void __launch_bounds__(256, 4) k_phase(const double* __restrict__ v, C* __restrict__ phi, double* vcopy, long long n,
                        double half_dt, double2 sg, CoefFuse cf, double hx, double hy, double hz) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  if (blockIdx.x == 0 && threadIdx.x < cf.count) cf.coef[threadIdx.x] = make_coef(cf.A[threadIdx.x], hx, hy, hz, 2.0 * half_dt);
  long long i = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= n) return;
  const double vi = v[i];
  double s, c;
  sincos(half_dt * vi, &s, &c);
  phi[i] = from_d2<C>(cmul(make_double2(c, -s), sg));  // FP64, rounded once for the SP variant
  if (vcopy != v) vcopy[i] = vi;
}

bool kin_scaled_ok(const Geometry& g) {
  const double h[3] = {g.hx, g.hy, g.hz};
  for (int d = 0; d < 3; ++d) {
    const double t = 1.0 / (2.0 * h[d] * h[d]);
    if (!(std::cos(0.5 * g.dt * t) >= 0.5) || !(std::cos(g.dt * t) >= 0.5)) return false;
  }
  return true;
}

static double2 scaled_sqrt_g(const Geometry& g) {
  const double h[3] = {g.hx, g.hy, g.hz};
  double re = 1.0, im = 0.0;
  for (int d = 0; d < 3; ++d) {  // prod_d e^{-i Delta t_d} c1_d sqrt(c2_d)
    const double t = 1.0 / (2.0 * h[d] * h[d]);
    const double mag = std::cos(0.5 * g.dt * t) * std::sqrt(std::cos(g.dt * t));
    const double pr = mag * std::cos(g.dt * t), pi = -mag * std::sin(g.dt * t);
    const double nr = re * pr - im * pi, ni = re * pi + im * pr;
    re = nr;
    im = ni;
  }
  return make_double2(re, im);
}

cudaError_t launch_phase(const Geometry& g, const double* v, double2* phi, double* vcopy, bool scaled,
                         cudaStream_t st, const CoefFuse* cf) {
  long long n = g.ng * g.ndom;
  const double2 sg = scaled ? scaled_sqrt_g(g) : make_double2(1.0, 0.0);
  CoefFuse c{};
  if (cf) c = *cf;
  launch_k(k_phase<double2>, (unsigned)((n + 255) / 256), 256, 0, st, v, phi, vcopy, n, 0.5 * g.dt, sg, c, g.hx, g.hy,
           g.hz);
  return cudaGetLastError();
}

cudaError_t launch_phase_sp(const Geometry& g, const double* v, float2* phi, double* vcopy, bool scaled,
                            cudaStream_t st, const CoefFuse* cf) {
  long long n = g.ng * g.ndom;
  const double2 sg = scaled ? scaled_sqrt_g(g) : make_double2(1.0, 0.0);
  CoefFuse c{};
  if (cf) c = *cf;
  launch_k(k_phase<float2>, (unsigned)((n + 255) / 256), 256, 0, st, v, phi, vcopy, n, 0.5 * g.dt, sg, c, g.hx, g.hy,
           g.hz);
  return cudaGetLastError();
}

// One K_axis pass. Column c of domain blockIdx.y: outer = c / inner_len, inner = c % inner_len,
// element offset = outer*outer_stride + inner; successive points of the line are pt_stride apart.
// Loads run two pairs ahead of the pair being combined (memory-level parallelism for the HBM stream).
// C: complex type of the coefficients and Phi; V: the value a lane moves per grid point (C, or cf2 = two
// complex64 orbitals); strides and norb are in units of V.
// src: the input (== psi for the usual in-place pass; another buffer for the out-of-place first pass of the
// self-consistent sweeps). In place is safe: each line belongs to one lane, whose reads of a point precede
// its write of that point.
// FP64 biased exponent bound of a complex64 value's components (0 for zero): |re|, |im| < 2^(E - 1022)
__device__ __forceinline__ int exp64_of(float2 v) {
  const uint32_t m = max(__float_as_uint(v.x) & 0x7fffffffu, __float_as_uint(v.y) & 0x7fffffffu);
  const int e8 = (int)(m >> 23);
  return m == 0 ? 0 : (e8 == 0 ? 897 : e8 + 896);
}

// colE (SP z pass with the int8-digit GEMMs only): the largest exponent of each orbital over the domain, for
// the next GEMM-1's digit scales (as k_kin_yz records it for FP64; a shared-memory max per CTA, then one global
// atomicMax per orbital).
template <bool kPeriodic, int kPhase, bool kS, class C = double2, class V = C>
__global__ void __launch_bounds__(256, 3) k_kin(V* psi, const V* src, const DomCoef* __restrict__ coef,
                                             const C* __restrict__ phi, int axis, int n, int pt_stride,
                                             int inner_len, int outer_stride, int ncols, int norb,
                                             long long dom_stride, long long ng, int* __restrict__ colE) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  int c = blockIdx.x * blockDim.x + threadIdx.x;
  if constexpr (std::is_same<C, float2>::value) {
    if (colE) {
      __shared__ int smax[128];
      for (int i = threadIdx.x; i < 128; i += blockDim.x) smax[i] = 0;
      __syncthreads();
      int ea = 0, eb = 0;
      if (c < ncols) {
        const int dom = blockIdx.y;
        const int outer = c / inner_len;
        const int inner = c - outer * inner_len;
        const int off = outer * outer_stride + inner;
        V* line = psi + dom * dom_stride + off;
        const V* sline = src + dom * dom_stride + off;
        const C* ph = phi + dom * ng + off / norb;
        const int ph_stride = pt_stride / norb;
        const PairCoefT<C> cf = pair_coef_t<kS, C>(coef + dom, axis);
        auto ld = [&](int i) -> V {
          V v = sline[(long long)i * pt_stride];
          if (kPhase == 1) v = cmul(ph[(long long)i * ph_stride], v);
          return v;
        };
        auto st = [&](int i, V v) {
          if (kPhase == 2) v = cmul(ph[(long long)i * ph_stride], v);
          line[(long long)i * pt_stride] = v;
          if constexpr (std::is_same<V, cf2>::value) {
            ea = max(ea, exp64_of(v.a));
            eb = max(eb, exp64_of(v.b));
          } else {
            ea = max(ea, exp64_of(v));
          }
        };
        march_line<kPeriodic, kS, C, V>(n, cf, ld, st);
        const int orb = std::is_same<V, cf2>::value ? 2 * inner : inner;  // (the z pass: inner = orbital unit)
        atomicMax(smax + orb, ea);
        if (std::is_same<V, cf2>::value) atomicMax(smax + orb + 1, eb);
      }
      __syncthreads();
      const int no = std::is_same<V, cf2>::value ? 2 * norb : norb;  // (norb is in units of V)
      for (int i = threadIdx.x; i < no; i += blockDim.x)
        if (smax[i] > 0) atomicMax(colE + (long long)blockIdx.y * no + i, smax[i]);
      return;
    }
  }
  if (c >= ncols) return;
  const int dom = blockIdx.y;
  const int outer = c / inner_len;
  const int inner = c - outer * inner_len;
  const int off = outer * outer_stride + inner;
  V* line = psi + dom * dom_stride + off;
  const V* sline = src + dom * dom_stride + off;
  const C* ph = phi + dom * ng + off / norb;
  const int ph_stride = pt_stride / norb;
  const PairCoefT<C> cf = pair_coef_t<kS, C>(coef + dom, axis);

  auto ld = [&](int i) -> V {
    V v = sline[(long long)i * pt_stride];
    if (kPhase == 1) v = cmul(ph[(long long)i * ph_stride], v);
    return v;
  };
  auto st = [&](int i, V v) {
    if (kPhase == 2) v = cmul(ph[(long long)i * ph_stride], v);
    line[(long long)i * pt_stride] = v;
  };

  march_line<kPeriodic, kS, C, V>(n, cf, ld, st);
}

// ------------------------------------------------------------------------------------------------
// Fused K_y K_z pass with the post-phase:  Psi <- Phi . K_y K_z Psi  (one HBM read + write of Psi).
// K_y and K_z act on different axes of the tensor grid and commute exactly (reading R6), so the pass
// applies K_z to each (x, y) z-line as it arrives and streams the K_z-transformed lines through the
// pair-aligned y-march of K_y.
// CTA = (x plane, chunk of kYZW = 8 orbitals, domain). A producer warp brings each (x, y) plane segment
// [nz rows][8 orbitals x 16 B] into an S-deep shared-memory ring with ONE tiled TMA tensor copy
// (cp.async.bulk.tensor, full/empty mbarriers); consumer thread (m, o) owns the z pair (2m, 2m+1) of
// orbital o0 + o and recomputes its neighbours' first-E outputs from the ring instead of exchanging
// them, so consumer warps never synchronise with each other.
// ------------------------------------------------------------------------------------------------
// a value of a loaded register, for mbar_release (lfd_tma.cuh)
__device__ __forceinline__ double dep_of(double2 v) { return v.x; }
__device__ __forceinline__ double dep_of(float2 v) { return (double)v.x; }
__device__ __forceinline__ double dep_of(cf2 v) { return (double)v.a.x; }

constexpr int kYZW = 8;
constexpr int kYZMaxThreads = 352;  // up to 40 z pairs x 8 orbitals + the producer warp
constexpr int kYZS = 16;            // ring depth (planes); even, so a y pair never straddles the wrap

// bytes of one ring slot: the Psi segment [nz][8 orbitals] + the Phi row [nz], 128-byte aligned
__host__ __device__ __forceinline__ int yz_slot_bytes(int nz) { return (nz * kYZW * 16 + nz * 16 + 127) & ~127; }

template <bool kPer, bool kS, class C = double2, class V = C>
__global__ void __launch_bounds__(kYZMaxThreads) k_kin_yz(const __grid_constant__ CUtensorMap tmap,
                                                          V* __restrict__ psi, const DomCoef* __restrict__ coef,
                                                          const C* __restrict__ phi, int nx, int ny, int nz,
                                                          int norb, int nchunks, long long ng, int* __restrict__ colE) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  // periodic => nz even (validated), so every thread owns a full pair and every link exists
  constexpr bool kFull = kPer;
  extern __shared__ __align__(128) unsigned char smem[];
  const int seg = nz * kYZW;                               // complex elements of the Psi segment
  const int slot_b = yz_slot_bytes(nz);                    // Psi segment + Phi row, 128-byte aligned
  auto slot_psi = [&](int s) { return reinterpret_cast<const V*>(smem + s * slot_b); };
  auto slot_phi = [&](int s) { return reinterpret_cast<const C*>(smem + s * slot_b + seg * 16); };
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + kYZS * slot_b);
  uint64_t* empty = full + kYZS;
  const int dom = blockIdx.y;
  const int x = blockIdx.x / nchunks, oc = blockIdx.x - (blockIdx.x / nchunks) * nchunks;
  const int o0 = oc * kYZW, wv = min(kYZW, norb - o0);
  const int npz = (nz + 1) >> 1;                 // z pairs (the last one a singleton for odd nz)
  const int nconsw = (npz * kYZW + 31) >> 5;     // consumer warps; the next warp is the producer
  // coefficients live in shared memory (broadcast LDS) to keep registers for the march state
  __shared__ PairCoefT<C> sc[2];
  const PairCoefT<C>& cz_ = sc[0];
  const PairCoefT<C>& cy = sc[1];
  const int tid = threadIdx.x;
  if (tid == 0) {
    sc[0] = pair_coef_t<kS, C>(coef + dom, 2);
    sc[1] = pair_coef_t<kS, C>(coef + dom, 1);
    for (int s = 0; s < kYZS; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], nconsw);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  const C* phx = phi + (long long)dom * ng + (long long)x * ny * nz;  // Phi(x, y = 0, z = 0)

  if (tid >= nconsw * 32) {  // producer warp: plane y -> slot y % kYZS (Psi: one tensor copy; Phi: one row)
    if (tid == nconsw * 32) {
      const int row0 = (dom * nx + x) * ny;
      int s = 0;
      uint32_t ph = 0;
      for (int y = 0; y < ny; ++y) {
        if (y >= kYZS) mbar_wait(&empty[s], ph ^ 1);
        mbar_expect_tx(&full[s], (uint32_t)(seg * 16 + nz * (int)sizeof(C)));
        tma_3d(smem + s * slot_b, &tmap, 2 * o0, 0, row0 + y, &full[s]);
        tma_row(smem + s * slot_b + seg * 16, phx + (long long)y * nz, (uint32_t)(nz * (int)sizeof(C)), &full[s]);
        if (++s == kYZS) { s = 0; ph ^= 1; }
      }
    }
    return;
  }

  const int o = tid % kYZW, m = tid / kYZW;
  const bool live = m < npz;
  const int z0 = 2 * m, z1 = 2 * m + 1;
  const bool has1 = kFull ? live : (live && z1 < nz);
  const bool act = live && o < wv;
  // ring offsets (complex elements within a slot) of the six points this thread's K_z reads
  const int zl = (m > 0) ? z0 - 2 : nz - 2;                    // pair m-1 (periodic wrap for m == 0)
  const int zr = (z1 + 1 < nz) ? z1 + 1 : 0;                   // pair m+1 (periodic wrap at the end)
  const bool has_l = kFull ? live : (live && m > 0);           // link (2m-1, 2m) exists
  const bool has_r = kFull ? live : (has1 && z1 + 1 < nz);     // link (2m+1, 2m+2) exists
  const bool r_single = kFull ? false : (zr + 1 >= nz);        // pair m+1 is a zero-BC singleton
  const int oz0 = live ? z0 * kYZW + o : o, oz1 = has1 ? z1 * kYZW + o : o;
  const int ozl = has_l ? zl * kYZW + o : o, ozl1 = has_l ? (zl + 1) * kYZW + o : o;
  const int ozr = has_r ? zr * kYZW + o : o, ozr1 = (has_r && !r_single) ? (zr + 1) * kYZW + o : o;
  const int pz0 = live ? z0 : 0, pz1 = has1 ? z1 : 0;          // Phi offsets in the slot's Phi row
  const int yst = nz * norb;  // element stride between y planes (< 2^31 per domain, validated)
  V* out0 = psi + (long long)dom * ng * norb + (long long)x * ny * yst + o0 + z0 * norb + o;
  V* out1 = out0 + norb;

  // K_z of plane y (slot s) for this thread's pair: the first E(Delta/2) on pairs m-1, m, m+1 (the
  // neighbours' outputs recomputed here), O(Delta) on the links (2m-1, 2m), (2m+1, 2m+2), then the
  // second E(Delta/2) on (2m, 2m+1).
  auto kz = [&](int s, V& w0, V& w1) {
    const V* r = slot_psi(s);
    const V a = r[oz0], b = r[oz1], vl = r[ozl], vl1 = r[ozl1], vr = r[ozr], vr1 = r[ozr1];
    V e0, e1 = V{};
    if (has1) {
      e0 = lk_L<kS>(cz_.a1, cz_.u1, a, b);
      e1 = lk_R<kS>(cz_.a1, cz_.d1, a, b);
    } else {
      e0 = lk_S<kS>(cz_.s1, a);
    }
    const V q0 = has_l ? lk_R<kS>(cz_.a2, cz_.d2, lk_R<kS>(cz_.a1, cz_.d1, vl, vl1), e0) : lk_S<kS>(cz_.s2, e0);
    if (has1) {
      V q1;
      if (has_r) {
        const V r0 = r_single ? lk_S<kS>(cz_.s1, vr) : lk_L<kS>(cz_.a1, cz_.u1, vr, vr1);
        q1 = lk_L<kS>(cz_.a2, cz_.u2, e1, r0);
      } else {
        q1 = lk_S<kS>(cz_.s2, e1);
      }
      w0 = lk_L<kS>(cz_.a1, cz_.u1, q0, q1);
      w1 = lk_R<kS>(cz_.a1, cz_.d1, q0, q1);
    } else {
      w0 = lk_S<kS>(cz_.s1, q0);
      w1 = V{};
    }
  };
  // dep: computed from this warp's last loads of the slot (they must have returned: lfd_tma.cuh)
  auto release = [&](int s, double dep) { mbar_release(&empty[s], dep, (tid & 31) == 0); };
  // colE != nullptr: the largest biased FP64 exponent of Re / Im of each orbital's output, for the int8-digit
  // GEMM-1 that follows (its per-orbital power-of-two scale; nl_i8.cu) -- integer max on the high words
  int me = 0, me2 = 0;  // (complex64 pairs: the exponents of the lane's two orbitals, FP64-biased)
  auto trk = [&](V w) {
    if constexpr (std::is_same<V, cf2>::value) {
      me = max(me, exp64_of(w.a));
      me2 = max(me2, exp64_of(w.b));
    } else {
      me = __vimax3_s32(me, __double2hiint(w.x) & 0x7ff00000, __double2hiint(w.y) & 0x7ff00000);
    }
    return w;
  };
  auto put0 = [&](int y, C f, V v) {
    if (act) out0[y * yst] = trk(cmul(f, v));
  };
  auto put1 = [&](int y, C f, V v) {
    if (act && has1) out1[y * yst] = trk(cmul(f, v));
  };

  LineMarch<kS, C, V> L0, L1;
  L0.init();
  L1.init();
  const int npairs = (ny + 1) >> 1;
  if (kFull && ny >= 4) {
    // periodic (even ny): pairs 0 and 1 peeled, then a steady loop without p / parity tests
    V wa0, wa1, wb0, wb1;
    mbar_wait(&full[0], 0);
    kz(0, wa0, wa1);
    mbar_wait(&full[1], 0);
    kz(1, wb0, wb1);
    release(0, dep_of(wa0) + dep_of(wa1));
    release(1, dep_of(wb0) + dep_of(wb1));
    L0.first(cy, wa0, wb0);
    L1.first(cy, wa1, wb1);
    mbar_wait(&full[2], 0);
    kz(2, wa0, wa1);
    mbar_wait(&full[3], 0);
    kz(3, wb0, wb1);
    L0.second(cy, wa0, wb0);
    L1.second(cy, wa1, wb1);
    int s_prev = 2, s_a = 4;  // slot of plane 2p-2 and of plane 2p (kYZS is even: pairs never straddle)
    uint32_t ph_a = 0;
    V* o0p = out0 + 2 * yst;  // plane 2p-2
#pragma unroll 2  // (C2 148.3 -> 145.6 us)
    for (int p = 2; p < npairs; ++p) {
      mbar_wait(&full[s_a], ph_a);
      kz(s_a, wa0, wa1);
      mbar_wait(&full[s_a + 1], ph_a);
      kz(s_a + 1, wb0, wb1);
      const C* pa = slot_phi(s_prev);
      const C* pb = slot_phi(s_prev + 1);
      const C fa0 = pa[pz0], fa1 = pa[pz1], fb0 = pb[pz0], fb1 = pb[pz1];
      L0.steady(cy, wa0, wb0, [&](int k, V v) {
        if (act) o0p[k * yst] = trk(cmul(k == 0 ? fa0 : fb0, v));
      });
      L1.steady(cy, wa1, wb1, [&](int k, V v) {
        if (act) o0p[k * yst + norb] = trk(cmul(k == 0 ? fa1 : fb1, v));
      });
      release(s_prev, dep_of(fa0) + dep_of(fa1));
      release(s_prev + 1, dep_of(fb0) + dep_of(fb1));
      o0p += 2 * yst;
      s_prev = s_a;
      s_a += 2;
      if (s_a == kYZS) { s_a = 0; ph_a ^= 1; }
    }
  } else {
    // ring bookkeeping: plane y sits in slot y % kYZS (phase (y / kYZS) & 1). Planes >= 2 are released
    // after their store (their Phi row is read then); planes 0 and 1 (stored last, by the wrap) right
    // after K_z -- their Phi comes from global memory at the end.
    int s_a = 0;
    uint32_t ph_a = 0;
    int s_prev = 0;  // slot of plane 2p-2
    for (int p = 0; p < npairs; ++p) {
      const int ya = 2 * p;
      const bool hb = ya + 1 < ny;
      int s_b = s_a + 1;
      uint32_t ph_b = ph_a;
      if (s_b == kYZS) { s_b = 0; ph_b ^= 1; }
      V wa0, wa1, wb0 = V{}, wb1 = V{};
      mbar_wait(&full[s_a], ph_a);
      kz(s_a, wa0, wa1);
      if (hb) {
        mbar_wait(&full[s_b], ph_b);
        kz(s_b, wb0, wb1);
      }
      if (p == 0) {
        release(s_a, dep_of(wa0) + dep_of(wa1));
        if (hb) release(s_b, dep_of(wb0) + dep_of(wb1));
      }
      // Phi of the planes this march step stores (2p-2 in slot s_prev, 2p-1 in the next slot)
      int s_pb = s_prev + 1;
      if (s_pb == kYZS) s_pb = 0;
      C fa0 = C{}, fa1 = C{}, fb0 = C{}, fb1 = C{};
      if (p >= 2) {
        const C* pa = slot_phi(s_prev);
        const C* pb = slot_phi(s_pb);
        fa0 = pa[pz0]; fa1 = pa[pz1];
        fb0 = pb[pz0]; fb1 = pb[pz1];
      }
      L0.push(cy, p, wa0, wb0, hb, [&](int y, V v) { put0(y, y == ya - 2 ? fa0 : fb0, v); });
      L1.push(cy, p, wa1, wb1, hb, [&](int y, V v) { put1(y, y == ya - 2 ? fa1 : fb1, v); });
      if (p >= 2) {
        release(s_prev, dep_of(fa0) + dep_of(fa1));
        release(s_pb, dep_of(fb0) + dep_of(fb1));
      }
      s_prev = s_a;
      s_a = s_b + 1;
      ph_a = ph_b;
      if (s_a == kYZS) { s_a = 0; ph_a ^= 1; }
    }
  }
  // wrap: planes ny-2, ny-1 (or ny-1 for odd ny; their slots are released at the end) and 0, 1
  const C* phb = phx + pz0;
  auto ph = [&](int y, int dz) { return (dz == 0 ? live : has1) ? __ldg(phb + y * nz + dz) : C{}; };
  const C f00 = ph(0, 0), f01 = ph(0, 1), f10 = ph(1, 0), f11 = ph(1, 1);
  const C fl0 = ph(ny - 1, 0), fl1 = ph(ny - 1, 1);
  const C fm0 = ph(ny - 2, 0), fm1 = ph(ny - 2, 1);
  auto pick0 = [&](int y) { return y == 0 ? f00 : y == 1 ? f10 : y == ny - 1 ? fl0 : fm0; };
  auto pick1 = [&](int y) { return y == 0 ? f01 : y == 1 ? f11 : y == ny - 1 ? fl1 : fm1; };
  L0.template finish<kPer>(cy, ny, [&](int y, V v) { put0(y, pick0(y), v); });
  L1.template finish<kPer>(cy, ny, [&](int y, V v) { put1(y, pick1(y), v); });
  if (colE) {  // max over this orbital's lanes (o = lane % 8), then one global atomicMax per (CTA, orbital)
    me = max(me, __shfl_xor_sync(0xffffffffu, me, 8));
    me = max(me, __shfl_xor_sync(0xffffffffu, me, 16));
    if constexpr (std::is_same<V, cf2>::value) {  // norb counts cf2 pairs here: orbitals 2 (o0 + o), + 1
      me2 = max(me2, __shfl_xor_sync(0xffffffffu, me2, 8));
      me2 = max(me2, __shfl_xor_sync(0xffffffffu, me2, 16));
      if ((tid & 31) < kYZW && act) {
        int* ce = colE + (long long)dom * 2 * norb + 2 * (o0 + o);
        if (me > 0) atomicMax(ce, me);
        if (me2 > 0) atomicMax(ce + 1, me2);
      }
    } else {
      if ((tid & 31) < kYZW && act) atomicMax(colE + (long long)dom * norb + o0 + o, me >> 20);
    }
  }
}

// (SP: two complex64 orbitals per lane (cf2), so norb must be even; the Phi row of nz complex64 must be a
// multiple of 16 bytes for its bulk copy: nz even)
bool kin_yz_supported(const Geometry& g) { return g.nz <= 80 && (!g.sp || (g.norb % 2 == 0 && g.nz % 2 == 0)); }

static size_t yz_smem(int nz) { return (size_t)kYZS * yz_slot_bytes(nz) + (size_t)kYZS * 16; }

// Tensor map of Psi for k_kin_yz: 3-D view [ndom*nx*ny planes][nz rows][2*norb doubles], box
// [1][nz][16 doubles] (one (x, y) plane segment of 8 orbitals), no swizzle (dense rows of 128 B).
// (SP: the same bytes, [planes][nz rows][norb 8-byte elements = complex64], box 16 elements = 8 cf2 pairs)
cudaError_t kin_yz_tensor_map(const Geometry& g, void* psi, CUtensorMap* out) {
  const uint64_t esz = g.sp ? 8 : 16;  // bytes per complex value
  const uint64_t dims[3] = {(uint64_t)g.norb * esz / 8, (uint64_t)g.nz, (uint64_t)g.ndom * g.nx * g.ny};
  const uint64_t strides[2] = {(uint64_t)g.norb * esz, (uint64_t)g.nz * g.norb * esz};
  const uint32_t box[3] = {2 * kYZW, (uint32_t)g.nz, 1};
  return encode_tmap_f64(out, 3, psi, dims, strides, box);
}

cudaError_t kin_yz_set_attributes() {
  const int sm = 220 * 1024;
  cudaError_t e = cudaFuncSetAttribute(k_kin_yz<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(k_kin_yz<true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(k_kin_yz<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(k_kin_yz<false, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(k_kin_yz<true, true, float2, cf2>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(k_kin_yz<true, false, float2, cf2>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(k_kin_yz<false, true, float2, cf2>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(k_kin_yz<false, false, float2, cf2>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm);
  return e;
}

cudaError_t launch_kin_yz(const Geometry& g, const CUtensorMap* tmap, double2* psi, const DomCoef* coef,
                          const double2* phi, bool scaled, cudaStream_t st, int* colE) {
  const int nchunks = (g.norb + kYZW - 1) / kYZW;
  const int threads = ((((g.nz + 1) / 2) * kYZW + 31) / 32 + 1) * 32;  // consumer warps + producer warp
  dim3 grid(g.nx * nchunks, g.ndom);
  const size_t sm = yz_smem(g.nz);
#define LFD_KYZ(P, K) \
  launch_k(k_kin_yz<P, K>, grid, threads, sm, st, *tmap, psi, coef, phi, g.nx, g.ny, g.nz, g.norb, nchunks, g.ng, colE)
  if (g.bc == 0) {
    if (scaled) LFD_KYZ(true, true); else LFD_KYZ(true, false);
  } else {
    if (scaled) LFD_KYZ(false, true); else LFD_KYZ(false, false);
  }
#undef LFD_KYZ
  return cudaGetLastError();
}

// SP: the same pass on complex64 Psi, two orbitals (16 bytes) per lane, FP32 arithmetic; colE gets the FP64-biased
// exponents of each complex64 orbital
cudaError_t launch_kin_yz_sp(const Geometry& g, const CUtensorMap* tmap, float2* psi, const DomCoef* coef,
                             const float2* phi, bool scaled, cudaStream_t st, int* colE) {
  const int nv = g.norb / 2;  // cf2 pairs per grid point
  const int nchunks = (nv + kYZW - 1) / kYZW;
  const int threads = ((((g.nz + 1) / 2) * kYZW + 31) / 32 + 1) * 32;
  dim3 grid(g.nx * nchunks, g.ndom);
  const size_t sm = yz_smem(g.nz);
  cf2* pv = reinterpret_cast<cf2*>(psi);
#define LFD_KYZ(P, K)                                                                                            \
  launch_k(k_kin_yz<P, K, float2, cf2>, grid, threads, sm, st, *tmap, pv, coef, phi, g.nx, g.ny, g.nz, nv, nchunks, \
           g.ng, colE)
  if (g.bc == 0) {
    if (scaled) LFD_KYZ(true, true); else LFD_KYZ(true, false);
  } else {
    if (scaled) LFD_KYZ(false, true); else LFD_KYZ(false, false);
  }
#undef LFD_KYZ
  return cudaGetLastError();
}

template <class C, class V>
static cudaError_t launch_kin_t(const Geometry& g, V* psi, const DomCoef* coef, const C* phi, int axis,
                                int phase_mode, bool scaled, cudaStream_t st, const V* src, int* colE = nullptr) {
  if (!src) src = psi;
  const int nd[3] = {g.nx, g.ny, g.nz};
  const int norb = g.norb / (int)(sizeof(V) / sizeof(C));  // values of type V per grid point
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
#define LFD_KIN(P, M, K)                                                                                       \
  launch_k(k_kin<P, M, K, C, V>, grid, 256, 0, st, psi, src, coef, phi, axis, n, pt_stride, inner_len, outer_stride, ncols, \
                                          norb, dom_stride, g.ng, colE)
#define LFD_KIN_M(P, K) \
  if (phase_mode == 1) LFD_KIN(P, 1, K); else if (phase_mode == 2) LFD_KIN(P, 2, K); else LFD_KIN(P, 0, K)
  if (g.bc == 0) {
    if (scaled) { LFD_KIN_M(true, true); } else { LFD_KIN_M(true, false); }
  } else {
    if (scaled) { LFD_KIN_M(false, true); } else { LFD_KIN_M(false, false); }
  }
#undef LFD_KIN_M
#undef LFD_KIN
  return cudaGetLastError();
}

cudaError_t launch_kin(const Geometry& g, double2* psi, const DomCoef* coef, const double2* phi, int axis,
                       int phase_mode, bool scaled, cudaStream_t st, const double2* src) {
  return launch_kin_t<double2, double2>(g, psi, coef, phi, axis, phase_mode, scaled, st, src);
}

cudaError_t launch_kin_sp(const Geometry& g, float2* psi, const DomCoef* coef, const float2* phi, int axis,
                          int phase_mode, bool scaled, cudaStream_t st, const float2* src, int* colE) {
  if (!src) src = psi;
  if (g.norb % 2 == 0 && ((reinterpret_cast<uintptr_t>(psi) | reinterpret_cast<uintptr_t>(src)) & 15) == 0)
    return launch_kin_t<float2, cf2>(g, reinterpret_cast<cf2*>(psi), coef, phi, axis, phase_mode, scaled, st,
                                     reinterpret_cast<const cf2*>(src), colE);  // two orbitals (16 bytes) per lane
  return launch_kin_t<float2, float2>(g, psi, coef, phi, axis, phase_mode, scaled, st, src, colE);
}

}  // namespace lfd
