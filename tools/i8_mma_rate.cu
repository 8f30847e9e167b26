// Micro-benchmark: tcgen05.mma kind::i8 issue rate for M=128 and several N, A from smem (SS) or TMEM (TS).
// One CTA per SM, one thread issues R MMAs back to back into one accumulator; cycles via clock64 around
// issue + commit wait. nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/i8_mma_rate tools/i8_mma_rate.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t saddr(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc(uint32_t a) {
  return (uint64_t)((a >> 4) & 0x3FFFu) | (1ull << 16) | (64ull << 32) | (1ull << 46) | (2ull << 61);
}
template <int N, bool TS>
__global__ void k(int R, long long* out) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint32_t tbase;
  __shared__ __align__(8) uint64_t bar;
  unsigned char* s = sm + ((1024u - (saddr(sm) & 1023u)) & 1023u);
  for (int i = threadIdx.x; i < 64 * 1024; i += blockDim.x) s[i] = (unsigned char)(i * 7);
  asm volatile("fence.proxy.async.shared::cta;");
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(saddr(&tbase)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(saddr(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t idesc = (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(N >> 3) << 17) | (8u << 24);
  if (threadIdx.x == 0) {
    const uint32_t a = saddr(s), b = saddr(s + 32768);
    const uint32_t tacc = tbase + 256;  // accumulator columns 256.. (N <= 256)
    long long t0 = clock64();
    for (int r = 0; r < R; ++r) {
      const uint32_t kk = (r & 3) * 32;
      if (TS) {
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n}\n"
                     ::"r"(tacc), "r"(tbase + (r & 3) * 8), "l"(desc(b + kk)), "r"(idesc), "r"(1));
      } else {
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n}\n"
                     ::"r"(tacc), "l"(desc(a + kk)), "l"(desc(b + kk)), "r"(idesc), "r"(1));
      }
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(saddr(&bar)));
    asm volatile("{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W;\n}\n" ::"r"(saddr(&bar)));
    long long t1 = clock64();
    out[blockIdx.x] = t1 - t0;
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tbase));
}
template <int N, bool TS>
void run(int sms, long long* d) {
  cudaFuncSetAttribute(k<N, TS>, cudaFuncAttributeMaxDynamicSharedMemorySize, 66 * 1024);
  const int R = 4096;
  k<N, TS><<<sms, 128, 66 * 1024>>>(R, d);
  k<N, TS><<<sms, 128, 66 * 1024>>>(R, d);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[256];
  cudaMemcpy(h, d, sizeof(long long) * sms, cudaMemcpyDeviceToHost);
  double avg = 0; for (int i = 0; i < sms; ++i) avg += h[i]; avg /= sms;
  const double macs = 128.0 * N * 32;
  printf("%s N=%3d: %.1f cycles/MMA  (%.0f MAC/clk/SM; peak 8192)  %s\n", TS ? "TS" : "SS", N, avg / R,
         macs * R / avg, cudaGetErrorString(e));
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  long long* d; cudaMalloc(&d, sizeof(long long) * 256);
  run<16, false>(sms, d); run<32, false>(sms, d); run<64, false>(sms, d); run<128, false>(sms, d); run<256, false>(sms, d);
  run<16, true>(sms, d); run<32, true>(sms, d); run<64, true>(sms, d); run<128, true>(sms, d); run<256, true>(sms, d);
  return 0;
}
