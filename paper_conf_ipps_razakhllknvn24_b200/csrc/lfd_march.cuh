// lfd_march.cuh -- the pair-split line march of the local propagator (P:68, P:76-80,
// Alg. 3-5), shared by the stencil passes (kin.cu) and the fused nonlocal GEMM-2 + K_x kernel
// (nl_fx.cu): pair-block coefficients, the link outputs and the streaming K_d march of one line.
#pragma once
#include "lfd_complex.cuh"
#include "lfd_internal.h"

namespace lfd {

// ---- pair blocks -------------------------------------------------------------------------------
// Coefficients of one axis for tau = Delta/2 (1) and Delta (2). General form: a = alpha, u = up,
// d = dn, s = onsite. Scaled form: u = w_up, d = w_dn, s = (1/c, 0), a unused.
template <class C>
struct PairCoefT {
  C a1, u1, d1, s1, a2, u2, d2, s2;
};
using PairCoef = PairCoefT<double2>;

template <bool kS>
__device__ __forceinline__ PairCoef pair_coef(const DomCoef* cf, int axis) {
  PairCoef c;
  if (kS) {
    c.a1 = c.a2 = make_double2(1.0, 0.0);
    c.u1 = cf->wu[axis][0]; c.d1 = cf->wd[axis][0]; c.s1 = make_double2(cf->rc[axis][0], 0.0);
    c.u2 = cf->wu[axis][1]; c.d2 = cf->wd[axis][1]; c.s2 = make_double2(cf->rc[axis][1], 0.0);
  } else {
    c.a1 = cf->alpha[axis][0]; c.u1 = cf->up[axis][0]; c.d1 = cf->dn[axis][0]; c.s1 = cf->onsite[axis][0];
    c.a2 = cf->alpha[axis][1]; c.u2 = cf->up[axis][1]; c.d2 = cf->dn[axis][1]; c.s2 = cf->onsite[axis][1];
  }
  return c;
}

// The SP variant (complex64 Psi) runs the same sweeps in FP32 with the coefficients
// rounded once from the FP64 table.
template <bool kS, class C>
__device__ __forceinline__ PairCoefT<C> pair_coef_t(const DomCoef* cf, int axis) {
  const PairCoef d = pair_coef<kS>(cf, axis);
  PairCoefT<C> c;
  c.a1 = from_d2<C>(d.a1); c.u1 = from_d2<C>(d.u1); c.d1 = from_d2<C>(d.d1); c.s1 = from_d2<C>(d.s1);
  c.a2 = from_d2<C>(d.a2); c.u2 = from_d2<C>(d.u2); c.d2 = from_d2<C>(d.d2); c.s2 = from_d2<C>(d.s2);
  return c;
}

// x + w y
__device__ __forceinline__ double2 padd(double2 w, double2 x, double2 y) {
  return make_double2(fma(w.x, y.x, fma(-w.y, y.y, x.x)), fma(w.x, y.y, fma(w.y, y.x, x.y)));
}
__device__ __forceinline__ float2 padd(float2 w, float2 x, float2 y) {
  return make_float2(fmaf(w.x, y.x, fmaf(-w.y, y.y, x.x)), fmaf(w.x, y.y, fmaf(w.y, y.x, x.y)));
}
// Two adjacent orbitals of one grid point (the SP passes move 16 bytes per lane, like the FP64 ones).
struct __align__(16) cf2 {
  float2 a, b;
};
__device__ __forceinline__ cf2 padd(float2 w, cf2 x, cf2 y) { return {padd(w, x.a, y.a), padd(w, x.b, y.b)}; }
__device__ __forceinline__ cf2 cmul(float2 s, cf2 x) { return {cmul(s, x.a), cmul(s, x.b)}; }
__device__ __forceinline__ cf2 crow(float2 a, cf2 x, float2 b, cf2 y) {
  return {crow(a, x.a, b, y.a), crow(a, x.b, b, y.b)};
}
__device__ __forceinline__ double2 rscale(double r, double2 x) { return make_double2(r * x.x, r * x.y); }
__device__ __forceinline__ float2 rscale(float r, float2 x) { return make_float2(r * x.x, r * x.y); }
__device__ __forceinline__ cf2 rscale(float r, cf2 x) { return {rscale(r, x.a), rscale(r, x.b)}; }

// Left / right output of a link (x at the left point, y at the right point) and a singleton; coefficients
// of type C, values of type V (V = C, or two complex64 orbitals for the SP passes).
template <bool kS, class C, class V>
__device__ __forceinline__ V lk_L(C a, C u, V x, V y) {
  return kS ? padd(u, x, y) : crow(a, x, u, y);
}
template <bool kS, class C, class V>
__device__ __forceinline__ V lk_R(C a, C d, V x, V y) {
  return kS ? padd(d, y, x) : crow(d, x, a, y);
}
template <bool kS, class C, class V>
__device__ __forceinline__ V lk_S(C s, V x) {
  return kS ? rscale(s.x, x) : cmul(s, x);
}

// Streaming K_d along one line, fed one pair (2p, 2p+1) at a time: first E(Delta/2) on the new pair,
// O(Delta) on the link (2p-1, 2p), second E(Delta/2) on (2p-2, 2p-1) once both its O outputs exist;
// points 0, 1 wait for the wrap link (n-1, 0) at the end.
template <bool kS, class C = double2, class V = C>
struct LineMarch {
  V E10, O1, prev_e1, prev_oR;
  __device__ __forceinline__ void init() { E10 = O1 = prev_e1 = prev_oR = V{}; }
  template <class St>
  __device__ __forceinline__ void push(const PairCoefT<C>& c, int p, V a, V b, bool pair, St&& st) {
    V e0, e1 = V{};
    if (pair) {
      e0 = lk_L<kS>(c.a1, c.u1, a, b);
      e1 = lk_R<kS>(c.a1, c.d1, a, b);
    } else {
      e0 = lk_S<kS>(c.s1, a);  // zero-BC singleton (odd n)
    }
    if (p == 0) {
      E10 = e0;
    } else {
      const V oL = lk_L<kS>(c.a2, c.u2, prev_e1, e0);
      const V oR = lk_R<kS>(c.a2, c.d2, prev_e1, e0);
      if (p == 1) {
        O1 = oL;
      } else {
        st(2 * p - 2, lk_L<kS>(c.a1, c.u1, prev_oR, oL));
        st(2 * p - 1, lk_R<kS>(c.a1, c.d1, prev_oR, oL));
      }
      prev_oR = oR;
    }
    prev_e1 = e1;
  }
  // The three phases of push() without the p tests (p == 0, p == 1, p >= 2 with a full pair).
  __device__ __forceinline__ void first(const PairCoefT<C>& c, V a, V b) {
    E10 = lk_L<kS>(c.a1, c.u1, a, b);
    prev_e1 = lk_R<kS>(c.a1, c.d1, a, b);
  }
  __device__ __forceinline__ void second(const PairCoefT<C>& c, V a, V b) {
    const V e0 = lk_L<kS>(c.a1, c.u1, a, b);
    O1 = lk_L<kS>(c.a2, c.u2, prev_e1, e0);
    prev_oR = lk_R<kS>(c.a2, c.d2, prev_e1, e0);
    prev_e1 = lk_R<kS>(c.a1, c.d1, a, b);
  }
  template <class St>
  __device__ __forceinline__ void steady(const PairCoefT<C>& c, V a, V b, St&& st) {
    const V e0 = lk_L<kS>(c.a1, c.u1, a, b);
    const V oL = lk_L<kS>(c.a2, c.u2, prev_e1, e0);
    const V oR = lk_R<kS>(c.a2, c.d2, prev_e1, e0);
    st(0, lk_L<kS>(c.a1, c.u1, prev_oR, oL));
    st(1, lk_R<kS>(c.a1, c.d1, prev_oR, oL));
    prev_oR = oR;
    prev_e1 = lk_R<kS>(c.a1, c.d1, a, b);
  }
  template <bool kPer, class St>
  __device__ __forceinline__ void finish(const PairCoefT<C>& c, int n, St&& st) {
    if ((n & 1) == 0) {
      V Olast, O0;
      if (kPer) {  // wrap link (n-1, 0)
        Olast = lk_L<kS>(c.a2, c.u2, prev_e1, E10);
        O0 = lk_R<kS>(c.a2, c.d2, prev_e1, E10);
      } else {
        Olast = lk_S<kS>(c.s2, prev_e1);
        O0 = lk_S<kS>(c.s2, E10);
      }
      if (n == 2) {
        st(0, lk_L<kS>(c.a1, c.u1, O0, Olast));
        st(1, lk_R<kS>(c.a1, c.d1, O0, Olast));
      } else {
        st(n - 2, lk_L<kS>(c.a1, c.u1, prev_oR, Olast));
        st(n - 1, lk_R<kS>(c.a1, c.d1, prev_oR, Olast));
        st(0, lk_L<kS>(c.a1, c.u1, O0, O1));
        st(1, lk_R<kS>(c.a1, c.d1, O0, O1));
      }
    } else {  // odd n (zero BC): last point is an E singleton; point 0 an O singleton
      st(n - 1, lk_S<kS>(c.s1, prev_oR));
      const V O0 = lk_S<kS>(c.s2, E10);
      st(0, lk_L<kS>(c.a1, c.u1, O0, O1));
      st(1, lk_R<kS>(c.a1, c.d1, O0, O1));
    }
  }
};

// K_d along one line of n points: ld(i) returns point i (input), st(i, v) stores output point i. Pairs are
// fed two ahead of the pair being combined (memory-level parallelism when ld reads HBM). In place is safe:
// a line belongs to one thread, whose reads of a point precede its write of that point.
template <bool kPeriodic, bool kS, class C, class V, class LD, class ST>
__device__ __forceinline__ void march_line(int n, const PairCoefT<C>& cf, LD&& ld, ST&& st) {
  const int P = (n + 1) >> 1;
  LineMarch<kS, C, V> L;
  L.init();
  if (kPeriodic && n >= 6) {  // periodic (even n): first two pairs peeled, then a test-free steady loop
    V a0 = ld(0), b0 = ld(1), a1 = ld(2), b1 = ld(3), a2 = ld(4), b2 = ld(5);
    L.first(cf, a0, b0);
    a0 = a1; b0 = b1; a1 = a2; b1 = b2;
    if (3 < P) { a2 = ld(6); b2 = ld(7); }
    L.second(cf, a0, b0);
    for (int p = 2; p < P; ++p) {
      a0 = a1; b0 = b1; a1 = a2; b1 = b2;
      if (p + 2 < P) { a2 = ld(2 * p + 4); b2 = ld(2 * p + 5); }
      L.steady(cf, a0, b0, [&](int k, V v) { st(2 * p - 2 + k, v); });
    }
    L.template finish<kPeriodic>(cf, n, st);
    return;
  }
  V na = ld(0), nb = (n > 1) ? ld(1) : V{};
  V nc = V{}, nd = V{};
  if (P > 1) {
    nc = ld(2);
    nd = (3 < n) ? ld(3) : V{};
  }
  for (int p = 0; p < P; ++p) {
    const V a = na, b = nb;
    na = nc;
    nb = nd;
    if (p + 2 < P) {
      nc = ld(2 * p + 4);
      nd = (2 * p + 5 < n) ? ld(2 * p + 5) : V{};
    }
    L.push(cf, p, a, b, 2 * p + 1 < n, st);
  }
  L.template finish<kPeriodic>(cf, n, st);
}

// The same K_d on a periodic line (n even, n >= 8) as two segments A = [0, LA) and B = [LA, n), LA = 2 ceil(n/4),
// marched side by side by one thread (two independent dependency chains, half the chain length); the links
// across the segment ends -- (LA-1, LA) and the wrap (n-1, 0) -- are taken at the end from the segments' first
// and last E outputs, as finish() takes the wrap of a single line. Same outputs, same arithmetic per output.
template <bool kS, class C, class V, class LD, class ST>
__device__ __forceinline__ void march_line2(int n, const PairCoefT<C>& c, LD&& ld, ST&& st) {
  const int PA = (n / 2 + 1) / 2, PB = n / 2 - PA, LA = 2 * PA;
  LineMarch<kS, C, V> A, B;
  A.init();
  B.init();
  A.first(c, ld(0), ld(1));
  B.first(c, ld(LA), ld(LA + 1));
  A.second(c, ld(2), ld(3));
  B.second(c, ld(LA + 2), ld(LA + 3));
  for (int p = 2; p < PA; ++p) {
    A.steady(c, ld(2 * p), ld(2 * p + 1), [&](int k, V v) { st(2 * p - 2 + k, v); });
    if (p < PB) B.steady(c, ld(LA + 2 * p), ld(LA + 2 * p + 1), [&](int k, V v) { st(LA + 2 * p - 2 + k, v); });
  }
  const V OAl = lk_L<kS>(c.a2, c.u2, A.prev_e1, B.E10);  // O output at LA - 1
  const V OBf = lk_R<kS>(c.a2, c.d2, A.prev_e1, B.E10);  // O output at LA
  const V OBl = lk_L<kS>(c.a2, c.u2, B.prev_e1, A.E10);  // O output at n - 1 (wrap link)
  const V OAf = lk_R<kS>(c.a2, c.d2, B.prev_e1, A.E10);  // O output at 0
  st(LA - 2, lk_L<kS>(c.a1, c.u1, A.prev_oR, OAl));
  st(LA - 1, lk_R<kS>(c.a1, c.d1, A.prev_oR, OAl));
  st(n - 2, lk_L<kS>(c.a1, c.u1, B.prev_oR, OBl));
  st(n - 1, lk_R<kS>(c.a1, c.d1, B.prev_oR, OBl));
  st(0, lk_L<kS>(c.a1, c.u1, OAf, A.O1));
  st(1, lk_R<kS>(c.a1, c.d1, OAf, A.O1));
  st(LA, lk_L<kS>(c.a1, c.u1, OBf, B.O1));
  st(LA + 1, lk_R<kS>(c.a1, c.d1, OBf, B.O1));
}

}  // namespace lfd
