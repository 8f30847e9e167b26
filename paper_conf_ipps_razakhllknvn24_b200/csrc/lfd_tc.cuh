// lfd_tc.cuh -- tcgen05 / TMEM helpers (inline PTX) and the exact FP64 <-> int8-digit arithmetic of the
// int8-digit projector GEMMs (nl_i8.cu, nl_fx.cu). See nl_i8.cu for the digit scheme.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "lfd_tma.cuh"

namespace lfd {

constexpr int kI8S = 6;    // digits per operand
constexpr int kI8M = 128;  // MMA M: 2 norb padded to 128

// byte offset of (row, k) in a K-major SWIZZLE_128B image with 128-byte rows (8-row, 1024-byte atoms;
// the 16-byte chunk index is XOR-ed with the row within the atom)
__host__ __device__ __forceinline__ int sw128(int row, int k) {
  return ((row >> 3) << 10) + ((row & 7) << 7) + ((((k >> 4) ^ (row & 7))) << 4) + (k & 15);
}

// the S digits of 4 consecutive values of one row; the scale exponent e is shared by the row (x = v 2^-e)
template <int S = kI8S>
__device__ __forceinline__ void digits4(const double v[4], int e, bool zero, uint32_t out[S]) {
  double x[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) x[q] = zero ? 0.0 : ldexp(v[q], 6 - e);  // 64 x, exact
  // rint and the integer conversion in one full-rate DADD: x + 1.5 2^52 rounds x to the nearest integer
  // (ties to even, as rint) and holds it in the low word; no FRND / F2I (low-rate conversion pipe)
  constexpr double kM = 6755399441055744.0;
#pragma unroll
  for (int i = 0; i < S; ++i) {
    uint32_t w = 0;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const double t = x[q] + kM;
      const double d = t - kM;
      x[q] = (x[q] - d) * 128.0;  // exact: |x - d| <= 1/2
      w |= ((uint32_t)__double2loint(t) & 0xffu) << (8 * q);
    }
    out[i] = w;
  }
}

// bytewise two's-complement negation of 4 packed int8 digits
__device__ __forceinline__ uint32_t neg_bytes(uint32_t w) { return __vsub4(0u, w); }

// the 6 balanced base-128 digits of 4 values in integer arithmetic: X = rint(v sc) (one DFMA against
// 1.5 2^52; |X| < 2^41), X + C with C = 64 (128^6 - 1) / 127 has the unsigned 7-bit fields u_k, and
// d = u - 64 in [-64, 63] (the top field u_5 <= 128: d_1 in [-64, 64]). X = sum_i d_i 128^(6-i): the same
// digit weights as digits4 (digit i <-> field 6 - i), a different but exact decomposition.
__device__ __forceinline__ void digits_i64(const double v[4], double sc, uint32_t out[kI8S]) {
  constexpr double kM = 6755399441055744.0;
  constexpr long long kMb = 0x4338000000000000LL;
  constexpr long long kC = 64LL * ((1LL << 42) - 1) / 127;
  // per value: the 4 low fields spread into the bytes of one word, the 2 high fields into another, each
  // byte u -> u - 64 (mod 256); then 4 x 4 byte transposes (PRMT) give the digit words
  uint32_t sq[4], tq[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const long long Y = (__double_as_longlong(fma(v[q], sc, kM)) - kMb) + kC;
    const uint32_t lo = (uint32_t)Y, hi = (uint32_t)(Y >> 32);
    uint32_t s4 = (lo & 0x7fu) | ((lo << 1) & 0x7f00u) | ((lo << 2) & 0x7f0000u) | ((lo << 3) & 0x7f000000u);
    s4 = (s4 ^ 0x40404040u) | ((~s4 & 0x40404040u) << 1);  // bytewise u - 64 for u in [0, 127]
    uint32_t f4 = __funnelshift_r(lo, hi, 28) & 0x7fu;
    f4 = (f4 ^ 0x40u) | ((~f4 & 0x40u) << 1);
    const uint32_t f5 = ((hi >> 3) + 192u) & 0xffu;  // top field, may be 128
    sq[q] = s4;
    tq[q] = f4 | (f5 << 8);
  }
  const uint32_t a = __byte_perm(sq[0], sq[1], 0x5140), b = __byte_perm(sq[0], sq[1], 0x7362);
  const uint32_t c = __byte_perm(sq[2], sq[3], 0x5140), d = __byte_perm(sq[2], sq[3], 0x7362);
  const uint32_t e = __byte_perm(tq[0], tq[1], 0x5140), f = __byte_perm(tq[2], tq[3], 0x5140);
  out[0] = __byte_perm(e, f, 0x7632);  // digit 1 = field 5
  out[1] = __byte_perm(e, f, 0x5410);  // field 4
  out[2] = __byte_perm(b, d, 0x7632);  // field 3
  out[3] = __byte_perm(b, d, 0x5410);  // field 2
  out[4] = __byte_perm(a, c, 0x7632);  // field 1
  out[5] = __byte_perm(a, c, 0x5410);  // field 0
}

// The same with 4 digits (the SP variant: complex64 operands, products accurate to ~2^-27 of the scales, below
// FP32 rounding): X = rint(v sc), |X| < 2^27, X + C4 (C4 = 64 (128^4 - 1) / 127) fits one 32-bit word with the
// fields u_0 .. u_3 (u_3 <= 128), d = u - 64; digit i <-> field 4 - i.
__device__ __forceinline__ void digits_s4(const double v[4], double sc, uint32_t out[4]) {
  constexpr double kM = 6755399441055744.0;
  constexpr long long kMb = 0x4338000000000000LL;
  constexpr int kC4 = 64 * (((1 << 28) - 1) / 127);  // 64 (1 + 128 + 128^2 + 128^3): the fields' 64s
  uint32_t w[4];
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    const uint32_t lo = (uint32_t)((__double_as_longlong(fma(v[q], sc, kM)) - kMb) + kC4);
    uint32_t s3 = (lo & 0x7fu) | ((lo << 1) & 0x7f00u) | ((lo << 2) & 0x7f0000u);
    s3 = (s3 ^ 0x404040u) | ((~s3 & 0x404040u) << 1);  // bytewise u - 64 (fields 0..2, u in [0, 127])
    w[q] = s3 | ((((lo >> 21) + 192u) & 0xffu) << 24);  // top field, may be 128
  }
  const uint32_t a = __byte_perm(w[0], w[1], 0x5140), b = __byte_perm(w[0], w[1], 0x7362);
  const uint32_t c = __byte_perm(w[2], w[3], 0x5140), d = __byte_perm(w[2], w[3], 0x7362);
  out[0] = __byte_perm(b, d, 0x7632);  // digit 1 = field 3
  out[1] = __byte_perm(b, d, 0x5410);  // field 2
  out[2] = __byte_perm(a, c, 0x7632);  // field 1
  out[3] = __byte_perm(a, c, 0x5410);  // field 0
}
// S-digit dispatch (S = 6: FP64 contexts, 4: SP); sc = 2^(7 S - 1 - e) for |v| < 2^e
template <int S>
__device__ __forceinline__ void digits_x(const double v[4], double sc, uint32_t out[S]) {
  if constexpr (S == 6) digits_i64(v, sc, out);
  else digits_s4(v, sc, out);
}

// exact int32 -> FP64 without the (low-rate) I2F.F64 conversion: 2^52 + (x + 2^31) built from bits, minus
// 2^52 + 2^31 (one full-rate DADD)
constexpr double kI2dM = 4503601774854144.0;  // 2^52 + 2^31
__device__ __forceinline__ double i2d_raw(int32_t x) {  // 2^52 + 2^31 + x (exact), no subtraction
  return __hiloint2double(0x43300000, (int)((uint32_t)x ^ 0x80000000u));
}
__device__ __forceinline__ double i2d(int32_t x) {
  return __hiloint2double(0x43300000, (int)((uint32_t)x ^ 0x80000000u)) - 4503601774854144.0;
}

// exact int64 -> FP64 for |x| < 2^51: (1.5 2^52 + x) built from bits, minus 1.5 2^52 (one DADD)
__device__ __forceinline__ double l2d(long long x) {
  return __longlong_as_double(x + 0x4338000000000000LL) - 6755399441055744.0;
}

// product of two powers of two (or zeros) by exponent arithmetic on the bits: no FP64 multiply
__device__ __forceinline__ double pow2mul(double a, double b) {
  const int ea = (__double2hiint(a) >> 20) & 0x7ff, eb = (__double2hiint(b) >> 20) & 0x7ff;
  const int e = ea + eb - 1023;
  return (ea == 0 || eb == 0 || e <= 0) ? 0.0 : __hiloint2double(e << 20, 0);
}

// x * a * b for powers of two a, b (or zeros) and x = 0 or a normal number whose product stays normal: an
// integer add on the exponent field instead of FP64 multiplies (the epilogue is FP64-pipe bound)
__device__ __forceinline__ double scale_pow2(double x, double a, double b) {
  const int ea = (__double2hiint(a) >> 20) & 0x7ff, eb = (__double2hiint(b) >> 20) & 0x7ff;
  const int hx = __double2hiint(x);
  const bool zero = ea == 0 || eb == 0 || (hx & 0x7fffffff) == 0;  // (x = 0: low word 0 too, it is an exact sum)
  return zero ? 0.0 : __hiloint2double(hx + ((ea + eb - 2046) << 20), __double2loint(x));
}

// x sigma tau for power-of-two FP64 scales, on an FP32 x (the SP epilogues): exponent-field arithmetic; a result
// below the FP32 normal range flushes to 0 (an SP update that small is far below the SP rounding of Psi)
__device__ __forceinline__ float scale_pow2f(float x, double a, double b) {
  const int ea = (__double2hiint(a) >> 20) & 0x7ff, eb = (__double2hiint(b) >> 20) & 0x7ff;
  const int hx = __float_as_int(x), k = ea + eb - 2046;
  const int ex = (hx >> 23) & 0xff;
  return (ea == 0 || eb == 0 || ex == 0 || ex + k <= 0) ? 0.0f : __int_as_float(hx + (k << 23));
}
// exact int32 -> float for |x| < 2^22: 1.5 2^23 + x built from bits, minus 1.5 2^23
__device__ __forceinline__ float i2f(int32_t x) { return __int_as_float(0x4B400000 + x) - 12582912.0f; }

__device__ __forceinline__ int row_exponent(double mx) {
  int e = 0;
  frexp(mx, &e);  // mx = m 2^e, m in [0.5, 1): mx < 2^e
  return e;
}

// ---- tcgen05 helpers (inline PTX) ----------------------------------------------------------------------
__device__ __forceinline__ uint64_t umma_desc_sw128(uint32_t saddr) {
  // start address >> 4 [0,14), LBO (unused for swizzled K-major) = 1 [16,30), SBO = 1024 B >> 4 [32,46),
  // version 1 [46,48), base offset 0, layout SWIZZLE_128B = 2 [61,64)
  return (uint64_t)((saddr >> 4) & 0x3FFFu) | (1ull << 16) | (64ull << 32) | (1ull << 46) | (2ull << 61);
}
// kind::i8 instruction descriptor: D s32, A/B signed int8, both K-major, M = 128, N = n (n % 16 == 0, <= 256)
__host__ __device__ constexpr uint32_t i8_idesc(int n) {
  return (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(kI8M >> 4) << 24);
}

// A (W^T digits) from TMEM, B (digit tile) from shared memory
__device__ __forceinline__ void umma_i8_ts(uint32_t tmem_d, uint32_t tmem_a, uint64_t db, uint32_t accumulate,
                                           uint32_t idesc) {
  asm volatile(
      "{\n.reg .pred p, e;\nelect.sync _|e, 0xffffffff;\nsetp.ne.b32 p, %4, 0;\n"
      "@e tcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n}\n" ::"r"(tmem_d),
      "r"(tmem_a), "l"(db), "r"(idesc), "r"(accumulate));
}
__device__ __forceinline__ void tmem_st8(uint32_t taddr, const uint32_t v[8]) {
  asm volatile("tcgen05.st.sync.aligned.32x32b.x8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"r"(taddr), "r"(v[0]),
               "r"(v[1]), "r"(v[2]), "r"(v[3]), "r"(v[4]), "r"(v[5]), "r"(v[6]), "r"(v[7])
               : "memory");
}
// issued by one elected lane of the (converged) calling warp
__device__ __forceinline__ void umma_commit(uint64_t* bar) {
  asm volatile(
      "{\n.reg .pred e;\nelect.sync _|e, 0xffffffff;\n"
      "@e tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n}\n" ::"r"(smem_addr(bar))
      : "memory");
}
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, int32_t v[16]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
      : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
        "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
      : "r"(taddr));
}
__device__ __forceinline__ void tmem_ld8(uint32_t taddr, int32_t v[8]) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7])
               : "r"(taddr));
}
template <int W>
__device__ __forceinline__ void tmem_ld(uint32_t taddr, int32_t* v);
template <>
__device__ __forceinline__ void tmem_ld<16>(uint32_t taddr, int32_t* v) { tmem_ld16(taddr, v); }
template <>
__device__ __forceinline__ void tmem_ld<8>(uint32_t taddr, int32_t* v) { tmem_ld8(taddr, v); }
__device__ __forceinline__ void tmem_ld4(uint32_t taddr, int32_t v[4]) {
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0,%1,%2,%3}, [%4];"
               : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3])
               : "r"(taddr));
}
__device__ __forceinline__ void tmem_wait_ld() { asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory"); }

}  // namespace lfd
