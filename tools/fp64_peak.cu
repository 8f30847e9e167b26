// FP64 pipe microbenchmark for B200 (sm_100a): DMMA.8x8x4 and DFMA issue-rate peaks.
// Used once to fix the FP64 roofline denominator ("FP64 peak must be measured").
#include <cstdio>
#include <cuda_runtime.h>
template <int CH>
__global__ void dmma_loop(double* out, int iters) {
  double c[CH][2];
  double a = 1.0 + threadIdx.x * 1e-9, b = 1.0 - threadIdx.x * 1e-9;
#pragma unroll
  for (int j = 0; j < CH; ++j) { c[j][0] = 0; c[j][1] = 0; }
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < CH; ++j)
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                   : "+d"(c[j][0]), "+d"(c[j][1]) : "d"(a), "d"(b));
  }
  double s = 0;
#pragma unroll
  for (int j = 0; j < CH; ++j) s += c[j][0] + c[j][1];
  if (s == 12345.0) out[threadIdx.x] = s;
}
template <int CH>
__global__ void dfma_loop(double* out, int iters) {
  double c[CH];
  double a = 1.0 + threadIdx.x * 1e-9, b = 1.0 - threadIdx.x * 1e-9;
#pragma unroll
  for (int j = 0; j < CH; ++j) c[j] = j;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < CH; ++j) c[j] = fma(c[j], a, b);
  }
  double s = 0;
#pragma unroll
  for (int j = 0; j < CH; ++j) s += c[j];
  if (s == 12345.0) out[threadIdx.x] = s;
}
int main() {
  double* out; cudaMalloc(&out, 4096 * sizeof(double));
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int threads : {128, 256, 512}) for (int blocksPerSM : {1, 2, 4}) {
    int grid = sms * blocksPerSM, iters = 20000;
    dmma_loop<8><<<grid, threads>>>(out, 100);
    cudaEventRecord(e0);
    dmma_loop<8><<<grid, threads>>>(out, iters);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double flops = 2.0 * 8 * 8 * 4 * 8.0 * iters * (double)grid * (threads / 32);
    printf("{\"kind\":\"dmma884\",\"threads\":%d,\"grid\":%d,\"tflops\":%.3f}\n", threads, grid, flops / ms / 1e9);
  }
  for (int threads : {256, 512, 1024}) for (int blocksPerSM : {1, 2}) {
    int grid = sms * blocksPerSM, iters = 20000;
    dfma_loop<8><<<grid, threads>>>(out, 100);
    cudaEventRecord(e0);
    dfma_loop<8><<<grid, threads>>>(out, iters);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    double flops = 2.0 * 8.0 * iters * (double)grid * threads;
    printf("{\"kind\":\"dfma\",\"threads\":%d,\"grid\":%d,\"tflops\":%.3f}\n", threads, grid, flops / ms / 1e9);
  }
  cudaError_t err = cudaGetLastError();
  printf("{\"err\":\"%s\",\"sms\":%d}\n", cudaGetErrorString(err), sms);
  return 0;
}
