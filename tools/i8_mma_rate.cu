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
// the k_gemm2_i8 issue pattern: per tile 6 diagonals x (pairs) x 4 K-steps, TS, N = 64, accumulators in 4
// slots; readers > 0: that many extra warps loop tcgen05.ld 32x32b.x16 over the accumulator columns meanwhile
__global__ void kpat(int tiles, int readers, long long* out) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ uint32_t tbase;
  __shared__ __align__(8) uint64_t bar;
  __shared__ volatile int done;
  unsigned char* s = sm + ((1024u - (saddr(sm) & 1023u)) & 1023u);
  for (int i = threadIdx.x; i < 48 * 1024; i += blockDim.x) s[i] = (unsigned char)(i * 7);
  asm volatile("fence.proxy.async.shared::cta;");
  if (threadIdx.x < 32) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(saddr(&tbase)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    done = 0;
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(saddr(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t idesc = (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(64 >> 3) << 17) | (8u << 24);
  const int warp = threadIdx.x >> 5;
  if (threadIdx.x == 0) {
    const uint32_t b = saddr(s);
    long long t0 = clock64();
    int cnt = 0;
    for (int t = 0; t < tiles; ++t)
      for (int d = 2; d <= 7; ++d) {
        const uint32_t acc = tbase + 192 + ((t * 6 + d - 2) % 4) * 64;
        uint32_t first = 1;
        for (int i = 1; i <= 6; ++i) {
          const int j = d - i;
          if (j < 1 || j > 6) continue;
          for (int kk = 0; kk < 4; ++kk) {
            asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::i8 [%0], [%1], %2, %3, p;\n}\n"
                         ::"r"(acc), "r"(tbase + (j - 1) * 32 + kk * 8), "l"(desc(b + (i - 1) * 8192 + kk * 32)), "r"(idesc),
                         "r"(first ? 0u : 1u));
            first = 0;
            ++cnt;
          }
        }
      }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(saddr(&bar)));
    asm volatile("{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared::cta.b64 p, [%0], 0;\n@!p bra W;\n}\n" ::"r"(saddr(&bar)));
    long long t1 = clock64();
    out[blockIdx.x] = (t1 - t0) / cnt;
    done = 1;
  } else if (warp >= 1 && warp <= readers) {
    const uint32_t la = tbase + ((uint32_t)(32 * (warp & 3)) << 16) + 192;
    uint32_t v[16];
    int k = 0;
    while (!done) {
      asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];"
                   : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                     "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
                   : "r"(la + (k & 15) * 16));
      asm volatile("tcgen05.wait::ld.sync.aligned;");
      ++k;
    }
    if (v[0] == 12345 && v[15] == 7) out[1000] = k;
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (threadIdx.x < 32) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tbase));
}
void runpat(int sms, long long* d, int readers) {
  cudaFuncSetAttribute(kpat, cudaFuncAttributeMaxDynamicSharedMemorySize, 50 * 1024);
  kpat<<<sms, 32 * 17, 50 * 1024>>>(40, readers, d);
  cudaError_t e = cudaDeviceSynchronize();
  long long h[256];
  cudaMemcpy(h, d, sizeof(long long) * sms, cudaMemcpyDeviceToHost);
  double avg = 0; for (int i = 0; i < sms; ++i) avg += h[i]; avg /= sms;
  printf("gemm2 pattern TS N=64, %2d TMEM reader warps: %.1f cycles/MMA  %s\n", readers, avg, cudaGetErrorString(e));
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
  run<16, true>(sms, d); run<32, true>(sms, d); run<64, true>(sms, d); run<80, true>(sms, d); run<96, true>(sms, d);
  run<128, true>(sms, d); run<160, true>(sms, d); run<256, true>(sms, d); run<80, false>(sms, d);
  cudaMalloc(&d, sizeof(long long) * 2048);
  runpat(sms, d, 0); runpat(sms, d, 4); runpat(sms, d, 16);
  return 0;
}
