// lfd_tma.cuh -- mbarrier + TMA bulk-copy helpers (inline PTX) for the sm_100a kernels.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

namespace lfd {

__device__ __forceinline__ uint32_t smem_addr(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(bar)) : "memory");
}
// Warp-collective release of a shared-memory stage that TMA refills. An mbarrier.arrive is not held back for the
// warp's shared loads still in flight (measured: one 8-lane phase of a k_gemm2_tma LDS.128 returned the bytes of
// the next refill -- two rows of a DMMA tile wrong, a few times per 10^5 tiles), and the TMA write does not queue
// behind them. So the arrive waits for a value computed from the warp's last loads of the stage (`dep`): every
// lane turns it into an always-zero integer (+-0 or NaN times 0 is never > 1), a warp-wide OR (redux) needs every
// lane's value, and the arrive's count is 1 + that zero. Lane `leader` arrives on each of the n barriers.
__device__ __forceinline__ uint32_t lds_done_count(double dep) {
  uint32_t cnt;
  asm volatile(
      "{\n.reg .f64 t;\n.reg .pred p;\n.reg .b32 z;\n"
      "mul.f64 t, %1, 0d0000000000000000;\n"
      "setp.gt.f64 p, t, 0d3FF0000000000000;\n"
      "selp.b32 z, 1, 0, p;\n"
      "redux.sync.or.b32 z, z, 0xffffffff;\n"
      "add.u32 %0, z, 1;\n}\n"
      : "=r"(cnt)
      : "d"(dep)
      : "memory");
  return cnt;
}
__device__ __forceinline__ void mbar_release(uint64_t* bar, double dep, bool leader) {
  const uint32_t cnt = lds_done_count(dep);
  if (leader) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(cnt) : "memory");
}
__device__ __forceinline__ void mbar_release2(uint64_t* bar0, uint64_t* bar1, bool two, double dep, bool leader) {
  const uint32_t cnt = lds_done_count(dep);
  if (leader) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar0)), "r"(cnt) : "memory");
    if (two) asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar1)), "r"(cnt) : "memory");
  }
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "LAB_WAIT:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra LAB_WAIT;\n"
      "}\n" ::"r"(smem_addr(bar)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void tma_row(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_addr(dst)),
      "l"(src), "r"(bytes), "r"(smem_addr(bar))
      : "memory");
}

// Row copy of any multiple of 8 bytes (complex64 rows of odd length): cp.async.bulk takes multiples of 16, so an
// 8-byte tail goes by a plain load / shared store, made visible to the async proxy and ordered before the
// arrive (release) that the consumers acquire; the barrier expects the bulk bytes plus `extra` (other copies
// completing on it). One thread.
__device__ __forceinline__ void tma_row8(void* dst, const void* src, uint32_t bytes, uint64_t* bar, uint32_t extra) {
  const uint32_t bulk = bytes & ~15u;
  if (bulk != bytes) {
    *reinterpret_cast<uint2*>(static_cast<char*>(dst) + bulk) =
        *reinterpret_cast<const uint2*>(static_cast<const char*>(src) + bulk);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  mbar_expect_tx(bar, bulk + extra);
  if (bulk) tma_row(dst, src, bulk, bar);
}

// Tiled tensor copy (3-D tensor map, coordinates innermost first) into shared memory.
__device__ __forceinline__ void tma_3d(void* dst, const void* tmap, int c0, int c1, int c2, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::
          "r"(smem_addr(dst)),
      "l"(reinterpret_cast<uint64_t>(tmap)), "r"(c0), "r"(c1), "r"(c2), "r"(smem_addr(bar))
      : "memory");
}

// Tiled tensor copy (4-D tensor map, coordinates innermost first) into shared memory.
__device__ __forceinline__ void tma_4d(void* dst, const void* tmap, int c0, int c1, int c2, int c3, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.4d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5}], [%6];" ::
          "r"(smem_addr(dst)),
      "l"(reinterpret_cast<uint64_t>(tmap)), "r"(c0), "r"(c1), "r"(c2), "r"(c3), "r"(smem_addr(bar))
      : "memory");
}

__device__ __forceinline__ void l2_prefetch(const void* src, uint32_t bytes) {
  asm volatile("cp.async.bulk.prefetch.L2.global [%0], %1;" ::"l"(src), "r"(bytes) : "memory");
}

}  // namespace lfd
