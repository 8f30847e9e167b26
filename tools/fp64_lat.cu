// Micro-benchmark: DFMA dependent-chain latency and per-SMSP throughput on this GPU (A/B reference for the FP64
// march kernels).  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/fp64_lat tools/fp64_lat.cu
#include <cstdio>
#include <cuda_runtime.h>
template <int CH>
__global__ void k(int n, double a, double b, double* out, long long* cyc) {
  double x[CH];
#pragma unroll
  for (int c = 0; c < CH; ++c) x[c] = threadIdx.x + c;
  __syncthreads();
  long long t0 = clock64();
  for (int i = 0; i < n; ++i) {
#pragma unroll
    for (int c = 0; c < CH; ++c) x[c] = fma(x[c], a, b);
  }
  long long t1 = clock64();
  double s = 0;
#pragma unroll
  for (int c = 0; c < CH; ++c) s += x[c];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
}
int main() {
  double* o; long long* c; cudaMalloc(&o, 1 << 24); cudaMalloc(&c, 8 * 4096);
  const int n = 4096;
  for (int warps : {1, 2, 4, 8, 16}) {
    long long h;
    k<1><<<1, 32 * warps>>>(n, 0.999, 1e-3, o, c); cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost);
    printf("warps %2d chains 1: %.2f cyc per DFMA per warp-chain\n", warps, (double)h / n);
    k<8><<<1, 32 * warps>>>(n, 0.999, 1e-3, o, c); cudaMemcpy(&h, c, 8, cudaMemcpyDeviceToHost);
    printf("warps %2d chains 8: %.2f cyc per 8 DFMA per warp -> %.1f DFMA lanes/clk/SM\n", warps, (double)h / n,
           8.0 * 32 * warps * n / (double)h);
  }
  return 0;
}
