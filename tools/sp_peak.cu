// FP32 pipe microbenchmark for B200 (sm_100a): legacy warp-level HMMA (mma.sync m16n8k8 tf32) and FFMA
// issue-rate peaks -- the candidates for the SP (complex64) projector GEMMs.
#include <cstdio>
#include <cuda_runtime.h>
template <int CH>
__global__ void tf32_loop(float* out, int iters) {
  float c[CH][4];
  unsigned a[4], b[2];
  for (int i = 0; i < 4; ++i) a[i] = __float_as_uint(1.0f + threadIdx.x * 1e-6f + i);
  for (int i = 0; i < 2; ++i) b[i] = __float_as_uint(1.0f - threadIdx.x * 1e-6f + i);
#pragma unroll
  for (int j = 0; j < CH; ++j) c[j][0] = c[j][1] = c[j][2] = c[j][3] = 0.f;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < CH; ++j)
      asm volatile("mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                   : "+f"(c[j][0]), "+f"(c[j][1]), "+f"(c[j][2]), "+f"(c[j][3])
                   : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b[0]), "r"(b[1]));
  }
  float s = 0;
#pragma unroll
  for (int j = 0; j < CH; ++j) s += c[j][0] + c[j][1] + c[j][2] + c[j][3];
  if (s == 12345.0f) out[threadIdx.x] = s;
}
template <int CH>
__global__ void ffma_loop(float* out, int iters) {
  float c[CH];
  float a = 1.0f + threadIdx.x * 1e-9f, b = 1.0f - threadIdx.x * 1e-9f;
#pragma unroll
  for (int j = 0; j < CH; ++j) c[j] = j;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < CH; ++j) c[j] = fmaf(c[j], a, b);
  }
  float s = 0;
#pragma unroll
  for (int j = 0; j < CH; ++j) s += c[j];
  if (s == 12345.0f) out[threadIdx.x] = s;
}
int main() {
  float* out; cudaMalloc(&out, 4096 * sizeof(float));
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int threads : {128, 256, 512}) for (int blocksPerSM : {1, 2, 4}) {
    int grid = sms * blocksPerSM, iters = 20000;
    tf32_loop<8><<<grid, threads>>>(out, 100);
    cudaEventRecord(e0);
    tf32_loop<8><<<grid, threads>>>(out, iters);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double flops = 2.0 * 16 * 8 * 8 * 8.0 * iters * (double)grid * (threads / 32);
    printf("{\"kind\":\"hmma_tf32_m16n8k8\",\"threads\":%d,\"grid\":%d,\"tflops\":%.3f}\n", threads, grid, flops / ms / 1e9);
  }
  for (int threads : {256, 512, 1024}) for (int blocksPerSM : {1, 2}) {
    int grid = sms * blocksPerSM, iters = 20000;
    ffma_loop<8><<<grid, threads>>>(out, 100);
    cudaEventRecord(e0);
    ffma_loop<8><<<grid, threads>>>(out, iters);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double flops = 2.0 * 8.0 * iters * (double)grid * threads;
    printf("{\"kind\":\"ffma\",\"threads\":%d,\"grid\":%d,\"tflops\":%.3f}\n", threads, grid, flops / ms / 1e9);
  }
  cudaError_t err = cudaGetLastError();
  printf("{\"err\":\"%s\",\"sms\":%d}\n", cudaGetErrorString(err), sms);
  return 0;
}
