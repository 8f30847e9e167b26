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
#include "lfd_tma.cuh"

#include <algorithm>
#include <cstdlib>
#include <new>
#include <type_traits>

namespace lfd {

// Tiling: a CTA owns a (kTY x kTZ) tile of (y, z) points and a chunk of kXC x-planes, which it walks in
// x order; each point is served by kSub consecutive lanes that split its orbitals (s = q, q+kSub, ...),
// so a warp load covers kSub*16 contiguous bytes per point. The x+1 / y+1 / z+1 neighbour rows are
// re-read through L1 (the x+1 row is the next iteration's own row; y+1 / z+1 rows mostly belong to the
// same tile), so HBM sees each row about once. Per-point sums are 3-level shuffle reductions over the
// kSub lanes; per-CTA partial J sums are reduced in a fixed order by k_jreduce.
constexpr int kSub = 8, kTY = 2, kTZ = 8, kXC = 10;
constexpr int kDensThreads = kSub * kTY * kTZ;  // 128

template <class C>
__global__ void __launch_bounds__(kDensThreads) k_density(Geometry g, DensArgs a, int ntz, int nty, int nxc) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  __shared__ double jsh[5][kDensThreads / kSub];
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
  // the SP variant (complex64 Psi) reads float2 and accumulates in FP64
  const C* P = reinterpret_cast<const C*>(sizeof(C) == 8 ? (const void*)a.psi_sp : (const void*)a.psi) +
               (long long)dom * g.ng * norb;
  const double* f = a.occ + (long long)dom * norb;
  const DomCoef* cf = a.coef + dom;
  const double2 ex = cf->eth[0], ey = cf->eth[1], ez = cf->eth[2];
  const double ihx = cf->inv_h[0], ihy = cf->inv_h[1], ihz = cf->inv_h[2];
  const int x0 = xc * nxc, x1 = min(g.nx, x0 + nxc);
  double jsx = 0.0, jsy = 0.0, jsz = 0.0, ekin = 0.0, eloc = 0.0;
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
        const double2 v = to_d2(__ldg(P + r * norb + s));
        rho = fma(fs, fma(v.x, v.x, v.y * v.y), rho);
        if (has_x) {
          const double2 w = cconjmul(v, to_d2(__ldg(P + rx * norb + s)));
          pxr = fma(fs, w.x, pxr);
          pxi = fma(fs, w.y, pxi);
        }
        if (has_y) {
          const double2 w = cconjmul(v, to_d2(__ldg(P + ry * norb + s)));
          pyr = fma(fs, w.x, pyr);
          pyi = fma(fs, w.y, pyi);
        }
        if (has_z) {
          const double2 w = cconjmul(v, to_d2(__ldg(P + rz * norb + s)));
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
    if (a.epart && valid) {  // kinetic / local energy densities (lfd_energy), FD Peierls form
      const double w2x = ihx * ihx, w2y = ihy * ihy, w2z = ihz * ihz;
      double ek = (w2x + w2y + w2z) * rho;
      if (has_x) ek -= w2x * (ex.x * pxr - ex.y * pxi);  // Re(e^{i theta} P)
      if (has_y) ek -= w2y * (ey.x * pyr - ey.y * pyi);
      if (has_z) ek -= w2z * (ez.x * pzr - ez.y * pzi);
      ekin += ek;
      eloc += a.v[(long long)dom * g.ng + ((long long)x * g.ny + y) * g.nz + z] * rho;
    }
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
    jsh[3][pt] = ekin; jsh[4][pt] = eloc;
  }
  __syncthreads();
  if (a.epart && threadIdx.x >= 32 && threadIdx.x < 34) {
    double t = 0.0;
    for (int k = 0; k < kDensThreads / kSub; ++k) t += jsh[3 + threadIdx.x - 32][k];
    a.epart[((long long)dom * gridDim.x + blockIdx.x) * 2 + threadIdx.x - 32] = t;
  }
  if (threadIdx.x < 3) {
    double t = 0.0;
    for (int i = 0; i < kDensThreads / kSub; ++i) t += jsh[threadIdx.x][i];
    a.jline[((long long)dom * gridDim.x + blockIdx.x) * 3 + threadIdx.x] = t;
  }
}

// ------------------------------------------------------------------------------------------------
// TMA-staged variant (norb <= 64): the CTA walks its x-chunk plane by plane through a 3-slot ring of
// shared-memory planes. A plane slot holds rows y0..y0+kTY (the last one is the y+1 halo row) x points
// z0..z0+kTZ (the last is the z+1 halo point), all orbitals; each row segment is contiguous in HBM and
// arrives by one cp.async.bulk. Iteration x reads slot(x) and slot(x+1) and then recycles slot(x) for
// plane x+3, so each row is fetched from HBM about once and every neighbour access is an LDS.
// ------------------------------------------------------------------------------------------------
constexpr int kRingSlots = 3;
constexpr int kMaxNorbTma = 64;
constexpr int kPlanePts = (kTY + 1) * (kTZ + 1);

__global__ void __launch_bounds__(kDensThreads) k_density_tma(Geometry g, DensArgs a, int ntz, int nty, int nxc) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  extern __shared__ __align__(128) unsigned char dsm[];
  __shared__ __align__(8) uint64_t bars[kRingSlots];
  __shared__ double jsh[5][kDensThreads / kSub];
  const int norb = g.norb;
  const int slot_elems = kPlanePts * norb;  // complex elements per slot
  double2* ring = reinterpret_cast<double2*>(dsm);
  const int dom = blockIdx.y;
  int b = blockIdx.x;
  const int tz = b % ntz; b /= ntz;
  const int ty = b % nty; b /= nty;
  const int xc = b;
  const int q = threadIdx.x % kSub, pt = threadIdx.x / kSub;
  const int py = pt / kTZ, pz = pt % kTZ;
  const int y0 = ty * kTY, z0 = tz * kTZ;
  const int y = y0 + py, z = z0 + pz;
  const bool valid = (y < g.ny) && (z < g.nz);
  const bool per = (g.bc == 0);
  const bool has_y = valid && (per || y + 1 < g.ny);
  const bool has_z = valid && (per || z + 1 < g.nz);
  const double2* P = a.psi + (long long)dom * g.ng * norb;
  const double* f = a.occ + (long long)dom * norb;
  const DomCoef* cf = a.coef + dom;
  const double2 ex = cf->eth[0], ey = cf->eth[1], ez = cf->eth[2];
  const double ihx = cf->inv_h[0], ihy = cf->inv_h[1], ihz = cf->inv_h[2];
  const int x0 = xc * nxc, x1 = min(g.nx, x0 + nxc);
  const int nplanes = x1 - x0 + 1;  // planes x0 .. x1 (x1 is the x+1 neighbour of the last)

  if (threadIdx.x == 0) {
    for (int s = 0; s < kRingSlots; ++s) mbar_init(&bars[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  // plane x0 + i -> slot i % 3; rows r = 0..kTY are y0 + r (periodic wrap), each kTZ+1 points from z0
  // (the periodic z halo past nz wraps to z = 0 and needs a second copy). Issued by warp 0.
  auto issue = [&](int i) {
    const int xg = x0 + i;
    const int slot = i % kRingSlots;
    const bool have_plane = (xg < g.nx) || per;
    const int xs = (xg < g.nx) ? xg : xg - g.nx;
    double2* dst = ring + (long long)slot * slot_elems;
    const int nz_in = min(kTZ + 1, g.nz - z0);       // contiguous part
    const int nz_wrap = per ? (kTZ + 1 - nz_in) : 0;  // wrapped halo points (z = 0 ..)
    int nrow = 0;
    if (have_plane)
      for (int r = 0; r <= kTY; ++r)
        if (y0 + r < g.ny || per) ++nrow;
    const uint32_t bytes = (uint32_t)(nrow * (nz_in + nz_wrap) * norb * 16);
    if (threadIdx.x == 0) mbar_expect_tx(&bars[slot], bytes);
    __syncwarp();
    if (!have_plane) return;
    const int lane = threadIdx.x & 31;
    if (lane <= kTY) {
      const int yy = y0 + lane;
      if (yy < g.ny || per) {
        const int ys = yy < g.ny ? yy : yy - g.ny;
        const long long row0 = ((long long)xs * g.ny + ys) * g.nz;
        double2* d = dst + (long long)lane * (kTZ + 1) * norb;
        tma_row(d, P + (row0 + z0) * norb, (uint32_t)(nz_in * norb * 16), &bars[slot]);
        if (nz_wrap > 0)
          tma_row(d + (long long)nz_in * norb, P + row0 * norb, (uint32_t)(nz_wrap * norb * 16), &bars[slot]);
      }
    }
  };

  if (threadIdx.x < 32)
    for (int i = 0; i < kRingSlots && i < nplanes; ++i) issue(i);

  double jsx = 0.0, jsy = 0.0, jsz = 0.0, ekin = 0.0, eloc = 0.0;
  for (int i = 0; i + 1 < nplanes; ++i) {
    const int x = x0 + i;
    mbar_wait(&bars[i % kRingSlots], (uint32_t)((i / kRingSlots) & 1));
    mbar_wait(&bars[(i + 1) % kRingSlots], (uint32_t)(((i + 1) / kRingSlots) & 1));
    const double2* S0 = ring + (long long)(i % kRingSlots) * slot_elems;
    const double2* S1 = ring + (long long)((i + 1) % kRingSlots) * slot_elems;
    const bool has_x = valid && (per || x + 1 < g.nx);
    double rho = 0.0, pxr = 0.0, pxi = 0.0, pyr = 0.0, pyi = 0.0, pzr = 0.0, pzi = 0.0;
    if (valid) {
      const double2* own = S0 + (py * (kTZ + 1) + pz) * norb;
      const double2* nx_ = S1 + (py * (kTZ + 1) + pz) * norb;
      const double2* ny_ = S0 + ((py + 1) * (kTZ + 1) + pz) * norb;
      const double2* nz_ = S0 + (py * (kTZ + 1) + pz + 1) * norb;
#pragma unroll 4
      for (int s = q; s < norb; s += kSub) {
        const double fs = __ldg(f + s);
        const double2 v = own[s];
        rho = fma(fs, fma(v.x, v.x, v.y * v.y), rho);
        if (has_x) {
          const double2 w = cconjmul(v, nx_[s]);
          pxr = fma(fs, w.x, pxr);
          pxi = fma(fs, w.y, pxi);
        }
        if (has_y) {
          const double2 w = cconjmul(v, ny_[s]);
          pyr = fma(fs, w.x, pyr);
          pyi = fma(fs, w.y, pyi);
        }
        if (has_z) {
          const double2 w = cconjmul(v, nz_[s]);
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
    const double jx = has_x ? (ex.x * pxi + ex.y * pxr) * ihx : 0.0;
    const double jy = has_y ? (ey.x * pyi + ey.y * pyr) * ihy : 0.0;
    const double jz = has_z ? (ez.x * pzi + ez.y * pzr) * ihz : 0.0;
    jsx += jx; jsy += jy; jsz += jz;
    if (a.epart && valid) {  // kinetic / local energy densities (lfd_energy), FD Peierls form
      const double w2x = ihx * ihx, w2y = ihy * ihy, w2z = ihz * ihz;
      double ek = (w2x + w2y + w2z) * rho;
      if (has_x) ek -= w2x * (ex.x * pxr - ex.y * pxi);  // Re(e^{i theta} P)
      if (has_y) ek -= w2y * (ey.x * pyr - ey.y * pyi);
      if (has_z) ek -= w2z * (ez.x * pzr - ez.y * pzi);
      ekin += ek;
      eloc += a.v[(long long)dom * g.ng + ((long long)x * g.ny + y) * g.nz + z] * rho;
    }
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
    __syncthreads();  // slot i % 3 is free
    if (threadIdx.x < 32 && i + kRingSlots < nplanes) issue(i + kRingSlots);
  }
  if (q == 0) {
    jsh[0][pt] = jsx; jsh[1][pt] = jsy; jsh[2][pt] = jsz;
    jsh[3][pt] = ekin; jsh[4][pt] = eloc;
  }
  __syncthreads();
  if (a.epart && threadIdx.x >= 32 && threadIdx.x < 34) {
    double t = 0.0;
    for (int k = 0; k < kDensThreads / kSub; ++k) t += jsh[3 + threadIdx.x - 32][k];
    a.epart[((long long)dom * gridDim.x + blockIdx.x) * 2 + threadIdx.x - 32] = t;
  }
  if (threadIdx.x < 3) {
    double t = 0.0;
    for (int k = 0; k < kDensThreads / kSub; ++k) t += jsh[threadIdx.x][k];
    a.jline[((long long)dom * gridDim.x + blockIdx.x) * 3 + threadIdx.x] = t;
  }
}

// ------------------------------------------------------------------------------------------------
// y-marching kernel (the bench shape; nact <= kQMaxAct). CTA = (px consecutive x planes, z chunk of zc
// points, y chunk, domain): it walks y and needs, at step y, the z-line segments of its own points
// (x0..x0+px-1, y, z0..z0+zc-1) plus their z+1 halo points, the next lines (y+1) for the y links and, for the
// x links, the lines of its own next plane -- or, for the last plane, of plane x0+px (the next CTA's first
// plane, read about when that CTA reads it: an L2 hit, so HBM sees each line about once). A producer warp
// brings each segment with one tiled TMA tensor copy (the halo point is a second, 1-point copy) into two rings
// (own lines: nso slots of px segments, x+px lines: nsx slots) with full/empty mbarriers; the own line y+1 stays
// resident as the next step's own line.
//
// Lanes: 4 per point (lane = 8 q + p: point p of the warp's 8, orbital quarter q owning s = q, q+4, q+8, ...),
// so a lane does 8 orbitals per step at nact = 32 and the per-point sums need a 2-level shuffle reduce-scatter.
// Bank conflicts: the 8 lanes of an LDS.128 phase read the same orbital of 8 consecutive points, so each smem row
// (one point, the active orbitals) is padded to an odd number of 16-byte units (a multiple of 16 bytes + 16 for
// complex64, whose 16-lane phases take q = 0, 1): the TMA box starts `pad` orbitals BEFORE orbital 0, where the
// tensor is out of bounds and the copy zero-fills -- padding without HBM traffic. Every LDS then has a
// compile-time offset from a per-step row pointer.
// ------------------------------------------------------------------------------------------------
constexpr int kQMaxWarps = 8;                        // consumer warps per CTA (8 points each; <= 168 registers)
constexpr int kQMaxThreads = (kQMaxWarps + 1) * 32;  // + the producer warp
constexpr int kQMaxAct = 120;                        // box inner dim <= 256 elements (FP64: 2 (nact + pad))

struct DensMaps {
  CUtensorMap seg;   // box [1][zc][E (nact + pad)] at orbital -pad: a z-line segment, each row padded in front
  CUtensorMap one;   // box [1][1][E (nact + pad)]: the z+1 halo point
  int zc;            // points per CTA and plane (divides nz)
  int px;            // x planes per CTA (divides nx)
  int nyc;           // y chunks per (plane group, z chunk)
  int nact;          // active orbitals: 1 + the last index with f != 0 (f = 0 contributes exactly 0)
  int pad;           // zero-filled orbitals in front of each shared-memory row (odd row length in 16-byte units)
  int esz;           // bytes per complex value: 16 (complex128) or 8 (complex64, the SP variant)
  int nso, nsx;      // ring depths: own lines, x+px lines
  int blocks;        // CTAs per domain
};

__host__ __device__ inline uint32_t q_al128(uint32_t b) { return (b + 127u) & ~127u; }

// shared-memory layout (every TMA destination 128-byte aligned): an own slot holds px (segment, halo point) pairs
struct QLayout {
  uint32_t rs, seg_b, halo_b, pl_b, own_b, xp_b, fsh_off, bar_off, total;
  __host__ __device__ QLayout(int zc, int px, int nact, int pad, int esz, int nso, int nsx) {
    rs = (uint32_t)((nact + pad) * esz);
    seg_b = q_al128((uint32_t)zc * rs);
    halo_b = q_al128(rs);
    pl_b = seg_b + halo_b;
    own_b = (uint32_t)px * pl_b;
    xp_b = seg_b;
    fsh_off = (uint32_t)nso * own_b + (uint32_t)nsx * xp_b;
    if (fsh_off < 3u * (kQMaxWarps * 32u) * 8u) fsh_off = 3u * (kQMaxWarps * 32u) * 8u;  // the end-of-kernel sums reuse it
    bar_off = fsh_off + (((uint32_t)nact * 8u + 15u) & ~15u);
    total = bar_off + (uint32_t)(2 * nso + 2 * nsx) * 8u;
  }
};

// pad: FP64 rows of an odd number of 16-byte units; complex64 rows of 2 (mod 4) 8-byte units (a 16-byte multiple).
// The box must start 16-byte aligned (the TMA faults otherwise): an even pad for complex64, whose active count is
// rounded up to even first (density_maps_shape; the extra orbital has f = 0).
static int q_pad(int nact, int esz) {
  if (esz == 16) return (nact & 1) ? 2 : 1;
  return (nact % 4 == 0) ? 2 : 0;
}

struct QShape {
  int zc, px, nyc, nso, nsx, pad;
};

static int q_num_sms() {
  int dev = 0, n = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess ||
      n <= 0) {
    cudaGetLastError();
    n = 148;
  }
  return n;
}

// Shape search: lanes used (px zc of 8 W), CTA balance over the resident slots (SMs x CTAs per SM by shared
// memory, threads and 168 registers per thread), the y+1 line each y chunk re-reads, warps straddling two planes
// and consumer warps per SM (>= 8); among equals, more ring bytes per SM. (L2 tensor prefetches of lines ahead
// of the ring loads measured slower in the step: C2 48.8 -> 55.9 us at 4 lines ahead.)
static QShape q_shape(const Geometry& g, int nact, int nsm) {
  QShape best{0, 1, 1, 3, 2, 1};
  const int esz = g.sp ? 8 : 16;
  if (nact > kQMaxAct) return best;
  if (g.sp && (g.norb & 1)) return best;  // TMA global strides must be multiples of 16 bytes
  const int pad = q_pad(nact, esz);
  best.pad = pad;
  double bscore = -1.0, binfl = 0.0;
  int fzc = 0, fpx = 0, fyc = 0, fso = 0, fsx = 0;
#ifdef LFD_TUNING_KNOBS
  if (const char* v = std::getenv("LFD_DENS_ZC")) fzc = std::atoi(v);
  if (const char* v = std::getenv("LFD_DENS_PX")) fpx = std::atoi(v);
  if (const char* v = std::getenv("LFD_DENS_YC")) fyc = std::atoi(v);
  if (const char* v = std::getenv("LFD_DENS_OWN")) fso = std::atoi(v);
  if (const char* v = std::getenv("LFD_DENS_XP")) fsx = std::atoi(v);
#endif
  for (int px = 1; px <= std::min(8, g.nx); ++px) {
    if (g.nx % px || (fpx && px != fpx)) continue;
    for (int zc = 1; zc <= g.nz; ++zc) {
      if (g.nz % zc || (fzc && zc != fzc)) continue;
      const int pts = px * zc, W = (pts + 7) / 8;
      if (W > kQMaxWarps) continue;
      const double util = (double)pts / (8.0 * W);
      if (util < 0.7) continue;
      for (int nso = 3; nso <= 6; ++nso) {
        if (fso && nso != fso) continue;
        for (int nsx = 2; nsx <= 3; ++nsx) {
          if (fsx && nsx != fsx) continue;
          const QLayout L(zc, px, nact, pad, esz, nso, nsx);
          if (L.total > 200u * 1024u) continue;
          const int cps = std::min({(int)((228u * 1024u) / (L.total + 1024u)), 2048 / ((W + 1) * 32),
                                    65536 / (168 * 32 * (W + 1)), 32});
          if (cps < 1) continue;
          const double R = (double)nsm * cps;
          const int base = (g.nx / px) * (g.nz / zc) * g.ndom;
          for (int nyc = 1; nyc <= std::min(8, std::max(1, g.ny / 2)); ++nyc) {
            if (fyc && nyc != fyc) continue;
            const double T = (double)base * nyc;
            const double bal = T / (std::ceil(T / R) * R);
            const double yeff = (double)g.ny / (double)(g.ny + nyc - 1);
            const double infl = (double)cps * ((nso - 2) * (double)L.own_b + (nsx - 1) * (double)L.xp_b);
            const double warps = (double)cps * W;
            const double straddle = (px > 1 && zc % 8) ? 0.9 : 1.0;  // warps across two planes: bank conflicts
            const double sc = util * bal * yeff * straddle * std::min(1.0, warps / 8.0);
            if (sc > bscore + 1e-9 || (sc > bscore - 1e-9 && infl > binfl)) {
              bscore = sc;
              binfl = infl;
              best = QShape{zc, px, nyc, nso, nsx, pad};
            }
          }
        }
      }
    }
  }
  return best;
}

template <bool kPer, int kIt, class C = double2>
__global__ void __launch_bounds__(kQMaxThreads, 1) k_density_q(const __grid_constant__ DensMaps mp, Geometry g,
                                                            DensArgs a) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
  extern __shared__ __align__(128) unsigned char dsm[];
  const int nact = mp.nact, zc = mp.zc, px = mp.px, nso = mp.nso, nsx = mp.nsx;
  const QLayout Ly(zc, px, nact, mp.pad, (int)sizeof(C), nso, nsx);
  const uint32_t rs = Ly.rs;
  auto own_seg = [&](int s, int p) { return dsm + s * Ly.own_b + p * Ly.pl_b; };
  auto halo_of = [&](int s, int p) { return dsm + s * Ly.own_b + p * Ly.pl_b + Ly.seg_b; };
  auto xp_slot = [&](int s) { return dsm + nso * Ly.own_b + s * Ly.xp_b; };
  double* fsh = reinterpret_cast<double*>(dsm + Ly.fsh_off);
  uint64_t* bars = reinterpret_cast<uint64_t*>(dsm + Ly.bar_off);
  uint64_t *ofull = bars, *oempty = bars + nso, *xfull = bars + 2 * nso, *xempty = xfull + nsx;
  const int dom = blockIdx.y;
  const int nzc = g.nz / zc, nyc = mp.nyc;
  const int yci = blockIdx.x % nyc, xz = blockIdx.x / nyc;
  const int xg = xz / nzc, z0 = (xz - xg * nzc) * zc;
  const int xb = xg * px;  // first plane of the CTA
  const int y0 = (int)(((long long)yci * g.ny) / nyc), ycnt = (int)(((long long)(yci + 1) * g.ny) / nyc) - y0;
  const bool has_xn = kPer || xb + px < g.nx;  // plane xb + px exists (the x+1 of the last plane)
  const bool xring = has_xn;
  const int xnext = (xb + px == g.nx) ? 0 : xb + px;
  const bool last_chunk = z0 + zc == g.nz;
  const int nconsw = (zc * px + 7) >> 3;
  const int tid = threadIdx.x;
  // own lines y0 .. y0+ycnt-1 plus the y+1 halo line (y = 0 again past the periodic wrap)
  const int nown = (kPer || y0 + ycnt < g.ny) ? ycnt + 1 : ycnt;
  const int E = (int)sizeof(C) / 8;  // 8-byte tensor elements per complex value
  if (tid == 0) {
    for (int s = 0; s < nso; ++s) { mbar_init(&ofull[s], 1); mbar_init(&oempty[s], nconsw); }
    for (int s = 0; s < nsx; ++s) { mbar_init(&xfull[s], 1); mbar_init(&xempty[s], nconsw); }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  for (int s = tid; s < nact; s += blockDim.x) fsh[s] = a.occ[(long long)dom * g.norb + s];
  __syncthreads();

  if (tid >= nconsw * 32) {  // producer warp
    if (tid == nconsw * 32) {
      const int rowxn = (dom * g.nx + xnext) * g.ny;
      const int c0 = -E * mp.pad;  // the row's zero-filled front padding (out of bounds: no HBM traffic)
      const bool halo = !last_chunk || kPer;  // z+1 halo point: z0 + zc, or z = 0 (periodic wrap)
      const uint32_t own_tx = (uint32_t)(px * (zc + (halo ? 1 : 0))) * rs, xp_tx = (uint32_t)zc * rs;
      int so = 0, sx = 0;
      uint32_t pho = 0, phx = 0;
      auto issue_own = [&](int k) {  // own lines y0 + k (== ny: plane 0 again) of the px planes
        if (k >= nso) mbar_wait(&oempty[so], pho ^ 1u);
        const int yy = (y0 + k == g.ny) ? 0 : y0 + k;
        mbar_expect_tx(&ofull[so], own_tx);
        for (int p = 0; p < px; ++p) {
          const int row = (dom * g.nx + xb + p) * g.ny + yy;
          tma_3d(own_seg(so, p), &mp.seg, c0, z0, row, &ofull[so]);
          if (halo) tma_3d(halo_of(so, p), &mp.one, c0, last_chunk ? 0 : z0 + zc, row, &ofull[so]);
        }
        if (++so == nso) { so = 0; pho ^= 1u; }
      };
      auto issue_xp = [&](int k) {
        if (k >= nsx) mbar_wait(&xempty[sx], phx ^ 1u);
        mbar_expect_tx(&xfull[sx], xp_tx);
        tma_3d(xp_slot(sx), &mp.seg, c0, z0, rowxn + y0 + k, &xfull[sx]);
        if (++sx == nsx) { sx = 0; phx ^= 1u; }
      };
      // keep the rings full: line k + depth reuses the slot the consumers release after step k
      for (int k = 0; k < nso && k < nown; ++k) issue_own(k);
      if (xring)
        for (int k = 0; k < nsx && k < ycnt; ++k) issue_xp(k);
      for (int k = 0; k < ycnt; ++k) {
        if (k + nso < nown) issue_own(k + nso);
        if (xring && k + nsx < ycnt) issue_xp(k + nsx);
      }
    }
    return;
  }

  const int lane = tid & 31, q = lane >> 3;
  const int pa = (tid >> 5) * 8 + (lane & 7);
  const int pl = pa / zc, pt = pa - pl * zc;  // plane within the CTA, point within the z chunk
  const bool valid = pl < px;
  const int plr = valid ? pl : 0, ptr = valid ? pt : 0;
  const int x = xb + plr, z = z0 + ptr;
  const bool has_x = valid && (kPer || x + 1 < g.nx);
  const bool has_z = valid && (kPer || z + 1 < g.nz);
  const DomCoef* cf = a.coef + dom;
  const double2 ex = cf->eth[0], ey = cf->eth[1], ez = cf->eth[2];
  const double ihx = cf->inv_h[0], ihy = cf->inv_h[1], ihz = cf->inv_h[2];
  const double w2x = ihx * ihx, w2y = ihy * ihy, w2z = ihz * ihz;
  // the per-point combination (rho, the link products, j, the lane reduce-scatter) in the accumulators' type:
  // FP32 for the SP variant (no FP64 pipe work per point but the final store conversion), FP64 otherwise
  using PA = typename std::conditional<sizeof(C) == 8, float, double>::type;
  const PA exx = (PA)ex.x, exy = (PA)ex.y, eyx = (PA)ey.x, eyy = (PA)ey.y, ezx = (PA)ez.x, ezy = (PA)ez.y;
  const PA ihxa = (PA)ihx, ihya = (PA)ihy, ihza = (PA)ihz;
  const uint32_t lo = (uint32_t)(mp.pad + q) * (uint32_t)sizeof(C);  // this lane's first orbital (s = q) in a row
  const uint32_t orow = (uint32_t)ptr * rs + lo;
  const bool zin = ptr + 1 < zc;  // z+1 in the segment (else the halo point)
  // occupations of this lane's orbitals s = q + 4 i in registers (kIt > 0: nact == 4 kIt exactly)
  double fr[kIt > 0 ? kIt : 1];
#pragma unroll
  for (int i = 0; i < (kIt > 0 ? kIt : 1); ++i) fr[i] = kIt > 0 ? fsh[q + 4 * i] : 0.0;
  const int nit = (nact - q + 3) >> 2;  // this lane's orbital count (kIt == 0)
  double jacc = 0.0, ekin = 0.0, eloc = 0.0;
  const long long rbase = a.base[dom], jb = a.j ? a.jbase[dom] : 0;  // hoisted global loads
  int so = 0, sn = nso > 1 ? 1 : 0, sx = 0;
  uint32_t pho = 0, phn = 0, phx = 0;
  C ocur[kIt > 0 ? kIt : 1];  // this lane's own values of the current line (kIt > 0)
  for (int k = 0; k < ycnt; ++k) {
    const int y = y0 + k;
    const bool has_y = valid && (kPer || y + 1 < g.ny);
    if (k == 0) mbar_wait(&ofull[so], pho);  // (later own lines were waited for as the previous step's y+1 line)
    if (k + 1 < nown) mbar_wait(&ofull[sn], phn);
    if (xring) mbar_wait(&xfull[sx], phx);
    const unsigned char* O = own_seg(so, plr) + orow;
    const unsigned char* Oz = zin ? O + rs : halo_of(so, plr) + lo;  // point z+1
    const unsigned char* N = own_seg(sn, plr) + orow;
    const unsigned char* X = (plr + 1 < px ? own_seg(so, plr + 1) : xp_slot(sx)) + orow;  // plane x+1
    // per-lane partial sums over this lane's orbitals: rho and the three link products P_d = sum f
    // conj(psi_r) psi_{r+e_d} (f folded into fv = f psi_r)
    // (two accumulator sets over alternate orbitals halve the FP64 dependency chains; summed in a fixed order)
    // (complex64 Psi, the SP variant: FP32 products and partial sums over the lane's orbitals -- <= 16 terms, a
    // relative error ~2^-20, far below the SP contract n 30 2^-24 -- then FP64 for the reduction over lanes)
    using A = typename std::conditional<sizeof(C) == 8, float, double>::type;
    A acc[2][7] = {};
    if (valid) {
      auto orb = [&](int i, A f, A* r, const C v, C& nv) {
        const uint32_t off = (uint32_t)i * 4u * (uint32_t)sizeof(C);
        const A fx = f * v.x, fy = f * v.y;
        r[0] = fma(fx, v.x, fma(fy, v.y, r[0]));
        if (kPer || has_x) {
          const C w = *reinterpret_cast<const C*>(X + off);
          r[1] = fma(fx, w.x, fma(fy, w.y, r[1]));
          r[2] = fma(fx, w.y, fma(-fy, w.x, r[2]));
        }
        if (kPer || has_y) {
          const C w = *reinterpret_cast<const C*>(N + off);
          nv = w;
          r[3] = fma(fx, w.x, fma(fy, w.y, r[3]));
          r[4] = fma(fx, w.y, fma(-fy, w.x, r[4]));
        }
        if (kPer || has_z) {
          const C w = *reinterpret_cast<const C*>(Oz + off);
          r[5] = fma(fx, w.x, fma(fy, w.y, r[5]));
          r[6] = fma(fx, w.y, fma(-fy, w.x, r[6]));
        }
      };
      if (kIt > 0) {  // the own values come from registers: the y+1 values of the previous step
        if (k == 0) {
#pragma unroll
          for (int i = 0; i < (kIt > 0 ? kIt : 1); ++i) ocur[i] = *reinterpret_cast<const C*>(O + i * 4 * (int)sizeof(C));
        }
        C nn[kIt > 0 ? kIt : 1];
#pragma unroll
        for (int i = 0; i < (kIt > 0 ? kIt : 1); ++i) orb(i, (A)fr[i], acc[i & 1], ocur[i], nn[i]);
#pragma unroll
        for (int i = 0; i < (kIt > 0 ? kIt : 1); ++i) ocur[i] = nn[i];
      } else {
        C nn;
#pragma unroll 4
        for (int i = 0; i < nit; ++i)
          orb(i, (A)fsh[q + 4 * i], acc[0], *reinterpret_cast<const C*>(O + i * 4 * (int)sizeof(C)), nn);
      }
    }
    const PA rho = (PA)acc[0][0] + acc[1][0], pxr = (PA)acc[0][1] + acc[1][1];
    const PA pxi = (PA)acc[0][2] + acc[1][2], pyr = (PA)acc[0][3] + acc[1][3];
    const PA pyi = (PA)acc[0][4] + acc[1][4], pzr = (PA)acc[0][5] + acc[1][5];
    const PA pzi = (PA)acc[0][6] + acc[1][6];
    // this warp is done with own line y and x+1 line y (once its loads have returned: lfd_tma.cuh)
    mbar_release2(&oempty[so], &xempty[sx], xring, ((rho + pxr) + (pyr + pzr)) + (pxi + pyi + pzi), lane == 0);
    if (++so == nso) { so = 0; pho ^= 1u; }
    if (++sn == nso) { sn = 0; phn ^= 1u; }
    if (xring && ++sx == nsx) { sx = 0; phx ^= 1u; }
    // the currents and the kinetic energy density are linear in the P_d: form them per lane first
    // (Im(e^{i theta} P) = cos Im P + sin Re P, Re(e^{i theta} P) = cos Re P - sin Im P)
    const PA jx = (kPer || has_x) ? (exx * pxi + exy * pxr) * ihxa : PA(0);
    const PA jy = (kPer || has_y) ? (eyx * pyi + eyy * pyr) * ihya : PA(0);
    const PA jz = (kPer || has_z) ? (ezx * pzi + ezy * pzr) * ihza : PA(0);
    if (a.epart) {  // kinetic energy density (FD Peierls form) summed per lane; reduced per CTA at the end
      double ek = (w2x + w2y + w2z) * (double)rho;
      if (kPer || has_x) ek -= w2x * (ex.x * (double)pxr - ex.y * (double)pxi);
      if (kPer || has_y) ek -= w2y * (ey.x * (double)pyr - ey.y * (double)pyi);
      if (kPer || has_z) ek -= w2z * (ez.x * (double)pzr - ez.y * (double)pzi);
      ekin += ek;
    }
    // reduce-scatter of (rho, jx, jy, jz) over the 4 lanes of the point (lanes xor 16, then xor 8; fixed order)
    PA u0, u1;
    {
      const bool hi = (q & 2) != 0;  // q = 2, 3 keep (jy, jz); q = 0, 1 keep (rho, jx)
      const PA s0 = hi ? rho : jy, s1 = hi ? jx : jz;
      const PA k0 = hi ? jy : rho, k1 = hi ? jz : jx;
      u0 = k0 + __shfl_xor_sync(0xffffffffu, s0, 16);
      u1 = k1 + __shfl_xor_sync(0xffffffffu, s1, 16);
    }
    const bool odd = (q & 1) != 0;  // keep the second of the two
    const double val = (double)((odd ? u1 : u0) + __shfl_xor_sync(0xffffffffu, odd ? u0 : u1, 8));
    // lane q now holds value q of its point: 0 rho, 1 jx, 2 jy, 3 jz
    if (valid) {
      const long long o = (long long)x * a.sx + (long long)y * a.sy + z;
      if (q == 0) {
        a.rho[rbase + o] = val;
        if (a.epart) eloc += a.v[(long long)dom * g.ng + ((long long)x * g.ny + y) * g.nz + z] * val;
      } else {
        jacc += val;
        if (a.j) a.j[jb + o + (q - 1) * a.jstride] = val;
      }
    }
  }
  // per-CTA sums in a fixed order: J components from lanes q = 1, 2, 3 of every point, energies from all; the
  // partials go to the (consumed) ring space once every consumer warp is done with it
  const int pts = nconsw * 8;
  double(*jsh)[kQMaxWarps * 8] = reinterpret_cast<double(*)[kQMaxWarps * 8]>(dsm);
  asm volatile("bar.sync 1, %0;" ::"r"(nconsw * 32) : "memory");
  if (q > 0) jsh[q - 1][pa] = jacc;
  double ekp = ekin;  // sum the kinetic partials over the 4 lanes of the point (fixed tree)
  ekp += __shfl_xor_sync(0xffffffffu, ekp, 16);
  ekp += __shfl_xor_sync(0xffffffffu, ekp, 8);
  if (q == 0) {
    jsh[3][pa] = ekp;
    jsh[4][pa] = eloc;
  }
  asm volatile("bar.sync 1, %0;" ::"r"(nconsw * 32) : "memory");  // consumer warps only
  if (a.epart && tid >= 3 && tid < 5) {  // (warp 0: there may be a single consumer warp)
    double t = 0.0;
    for (int k = 0; k < pts; ++k) t += jsh[tid][k];
    a.epart[((long long)dom * gridDim.x + blockIdx.x) * 2 + tid - 3] = t;
  }
  if (tid < 3) {
    double t = 0.0;
    for (int k = 0; k < pts; ++k) t += jsh[tid][k];
    a.jline[((long long)dom * gridDim.x + blockIdx.x) * 3 + tid] = t;
    __threadfence();  // (before the CTA's completion count below)
  }
  if (!a.Jmac) return;
  // the domain's last CTA to finish reduces the per-CTA partials into J_d = (1/Ngrid) sum (fixed order: by CTA
  // index, whatever the arrival order) and re-arms the counter -- the k_jreduce launch folded in
  __shared__ int last;
  asm volatile("bar.sync 1, %0;" ::"r"(nconsw * 32) : "memory");
  if (tid == 0) last = atomicAdd(a.dcount + dom, 1) == (int)gridDim.x - 1;
  asm volatile("bar.sync 1, %0;" ::"r"(nconsw * 32) : "memory");
  if (!last) return;
  __threadfence();
  const int nt = nconsw * 32;
  double sj[3] = {0.0, 0.0, 0.0};
  const volatile double* jl = a.jline + (long long)dom * gridDim.x * 3;
  for (int l = tid; l < (int)gridDim.x; l += nt)
    for (int d = 0; d < 3; ++d) sj[d] += jl[l * 3 + d];
  double* red = reinterpret_cast<double*>(dsm);  // (the ring is consumed)
  for (int d = 0; d < 3; ++d) red[d * nt + tid] = sj[d];
  asm volatile("bar.sync 1, %0;" ::"r"(nt) : "memory");
  if (tid < 3) {
    double t = 0.0;
    for (int k = 0; k < nt; ++k) t += red[tid * nt + k];
    a.Jmac[dom * 3 + tid] = t / (double)g.ng;
  }
  if (tid == 0) a.dcount[dom] = 0;
}

bool density_reduces_J(const DensMaps* m) { return m != nullptr; }

static size_t q_smem(const DensMaps& m) { return QLayout(m.zc, m.px, m.nact, m.pad, m.esz, m.nso, m.nsx).total; }

// Psi as a 3-D tensor of 8-byte elements [rows][nz][norb * esz / 8] (the TMA only moves bytes: a complex64 value
// is one 8-byte element, a complex128 value two); the box spans nact + pad values from value -pad.
static cudaError_t density_maps_encode(DensMaps* m, const Geometry& g, const double2* psi) {
  const uint64_t w = (uint64_t)m->esz / 8;
  const uint64_t dims[3] = {w * g.norb, (uint64_t)g.nz, (uint64_t)g.ndom * g.nx * g.ny};
  const uint64_t str[2] = {(uint64_t)g.norb * m->esz, (uint64_t)g.nz * g.norb * m->esz};
  const uint32_t b2[3] = {(uint32_t)(w * (m->nact + m->pad)), (uint32_t)m->zc, 1};
  const uint32_t b3[3] = {(uint32_t)(w * (m->nact + m->pad)), 1, 1};
  cudaError_t e = encode_tmap_f64(&m->seg, 3, psi, dims, str, b2);
  if (e == cudaSuccess) e = encode_tmap_f64(&m->one, 3, psi, dims, str, b3);
  return e;
}

static bool density_maps_shape(DensMaps* m, const Geometry& g, int nact) {
  if (g.sp && (nact & 1) && nact < g.norb) ++nact;  // complex64: an even active count (q_pad)
  const QShape sh = q_shape(g, nact, q_num_sms());
  if (sh.zc == 0) return false;
  m->zc = sh.zc; m->px = sh.px; m->nyc = sh.nyc; m->nso = sh.nso; m->nsx = sh.nsx; m->pad = sh.pad;
  m->nact = nact;
  m->esz = g.sp ? 8 : 16;
  m->blocks = (g.nx / sh.px) * (g.nz / sh.zc) * sh.nyc;
  return true;
}

DensMaps* density_maps_create(const Geometry& g, const double2* psi, int nact) {
  nact = std::min(std::max(nact, 1), g.norb);
  DensMaps* m = new (std::nothrow) DensMaps;
  if (!m) return nullptr;
  if (!density_maps_shape(m, g, nact) || density_maps_encode(m, g, psi) != cudaSuccess) {
    delete m;
    return nullptr;
  }
  return m;
}

// The active-orbital count changed (lfd_set_occupations): new shape and descriptors. A count past kQMaxAct keeps the
// old shape and its (larger) active set -- the extra orbitals have f = 0 and add exactly zero.
cudaError_t density_maps_set_active(DensMaps* m, const Geometry& g, const double2* psi, int nact) {
  nact = std::min(std::max(nact, 1), g.norb);
  if (!m || m->nact == nact) return cudaSuccess;
  DensMaps t = *m;
  if (!density_maps_shape(&t, g, nact)) {
    if (nact < m->nact) return cudaSuccess;
    return cudaErrorNotSupported;
  }
  const cudaError_t e = density_maps_encode(&t, g, psi);
  if (e == cudaSuccess) *m = t;
  return e;
}

void density_maps_destroy(DensMaps* m) { delete m; }

int density_smem_bytes(int norb) { return kRingSlots * kPlanePts * norb * 16; }

static int fallback_blocks(const Geometry& g) {
  const int ntz = (g.nz + kTZ - 1) / kTZ, nty = (g.ny + kTY - 1) / kTY, nxc = (g.nx + kXC - 1) / kXC;
  return ntz * nty * nxc;
}

// workspace bound on the CTAs per domain (per-CTA partial sums): any y-marching shape has at most nx nz 8 CTAs
int density_blocks(const Geometry& g) {
  return std::max(fallback_blocks(g), g.nx * g.nz * std::min(8, std::max(1, g.ny / 2)));
}

int density_blocks_used(const Geometry& g, const DensMaps* m) { return m ? m->blocks : fallback_blocks(g); }

cudaError_t launch_density(const Geometry& g, const DensArgs& a_in, const DensMaps* maps, cudaStream_t st) {
  DensArgs a = a_in;
  if (!maps) a.Jmac = nullptr;  // (the generic kernels leave J to k_jreduce)
  if (maps) {
    dim3 grid(maps->blocks, g.ndom);
    const int threads = ((maps->zc * maps->px + 7) / 8 + 1) * 32;
    const size_t sm = q_smem(*maps);
    const int n = maps->nact;
    if (maps->esz == 8) {  // SP variant (complex64 Psi)
      if (g.bc == 0 && n == 32) launch_k(k_density_q<true, 8, float2>, grid, threads, sm, st, *maps, g, a);
      else if (g.bc == 0 && n == 64) launch_k(k_density_q<true, 16, float2>, grid, threads, sm, st, *maps, g, a);
      else if (g.bc == 0) launch_k(k_density_q<true, 0, float2>, grid, threads, sm, st, *maps, g, a);
      else launch_k(k_density_q<false, 0, float2>, grid, threads, sm, st, *maps, g, a);
      return cudaGetLastError();
    }
    if (g.bc == 0 && n == 32) launch_k(k_density_q<true, 8>, grid, threads, sm, st, *maps, g, a);
    else if (g.bc == 0 && n == 64) launch_k(k_density_q<true, 16>, grid, threads, sm, st, *maps, g, a);
    else if (g.bc == 0) launch_k(k_density_q<true, 0>, grid, threads, sm, st, *maps, g, a);
    else launch_k(k_density_q<false, 0>, grid, threads, sm, st, *maps, g, a);
    return cudaGetLastError();
  }
  dim3 grid(fallback_blocks(g), g.ndom);
  const int ntz = (g.nz + kTZ - 1) / kTZ, nty = (g.ny + kTY - 1) / kTY;
  if (a.psi_sp)
    launch_k(k_density<float2>, grid, kDensThreads, 0, st, g, a, ntz, nty, kXC);
  else if (g.norb <= kMaxNorbTma)
    launch_k(k_density_tma, grid, kDensThreads, density_smem_bytes(g.norb), st, g, a, ntz, nty, kXC);
  else
    launch_k(k_density<double2>, grid, kDensThreads, 0, st, g, a, ntz, nty, kXC);
  return cudaGetLastError();
}

cudaError_t density_set_attributes() {
  cudaError_t e = cudaFuncSetAttribute(k_density_tma, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                       density_smem_bytes(kMaxNorbTma));
  if (e != cudaSuccess) return e;
  for (auto f : {k_density_q<true, 8>, k_density_q<true, 16>, k_density_q<true, 0>, k_density_q<false, 0>,
                 k_density_q<true, 8, float2>, k_density_q<true, 16, float2>, k_density_q<true, 0, float2>,
                 k_density_q<false, 0, float2>}) {
    e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, 210 * 1024);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

// J_d = (1/Ngrid) sum_lines jline (one block per domain, fixed-order tree over a fixed partition).
__global__ void __launch_bounds__(256) k_jreduce(const double* __restrict__ jline, int lines, double inv_ng,
                                                 double* __restrict__ Jmac) {
  pdl_wait();     // programmatic dependent launch: the previous kernel's writes are visible
  pdl_trigger();  // let the next kernel launch (its CTAs wait in pdl_wait)
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

cudaError_t launch_jreduce(const Geometry& g, const double* jline, int blocks, double* Jmac, cudaStream_t st) {
  launch_k(k_jreduce, g.ndom, 256, 0, st, jline, blocks, 1.0 / (double)g.ng, Jmac);
  return cudaGetLastError();
}

}  // namespace lfd
