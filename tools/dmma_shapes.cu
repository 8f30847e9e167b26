#include <cstdio>
__global__ void k16(double* out, int iters) {
  double c[8][4];
  double a[8], b[4];
  for (int i = 0; i < 8; ++i) a[i] = 1.0 + threadIdx.x * 1e-9 + i;
  for (int i = 0; i < 4; ++i) b[i] = 1.0 - threadIdx.x * 1e-9 + i;
  for (int j = 0; j < 8; ++j) for (int i = 0; i < 4; ++i) c[j][i] = 0;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 8; ++j)
      asm volatile("mma.sync.aligned.m16n8k16.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7,%8,%9,%10,%11}, {%12,%13,%14,%15}, {%0,%1,%2,%3};"
                   : "+d"(c[j][0]), "+d"(c[j][1]), "+d"(c[j][2]), "+d"(c[j][3])
                   : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(a[4]), "d"(a[5]), "d"(a[6]), "d"(a[7]),
                     "d"(b[0]), "d"(b[1]), "d"(b[2]), "d"(b[3]));
  }
  double s = 0;
  for (int j = 0; j < 8; ++j) for (int i = 0; i < 4; ++i) s += c[j][i];
  if (s == 12345.0) out[threadIdx.x] = s;
}
__global__ void k8(double* out, int iters) {
  double c[8][4];
  double a[4], b[2];
  for (int i = 0; i < 4; ++i) a[i] = 1.0 + threadIdx.x * 1e-9 + i;
  for (int i = 0; i < 2; ++i) b[i] = 1.0 - threadIdx.x * 1e-9 + i;
  for (int j = 0; j < 8; ++j) for (int i = 0; i < 4; ++i) c[j][i] = 0;
  for (int it = 0; it < iters; ++it) {
#pragma unroll
    for (int j = 0; j < 8; ++j)
      asm volatile("mma.sync.aligned.m16n8k8.row.col.f64.f64.f64.f64 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, {%0,%1,%2,%3};"
                   : "+d"(c[j][0]), "+d"(c[j][1]), "+d"(c[j][2]), "+d"(c[j][3])
                   : "d"(a[0]), "d"(a[1]), "d"(a[2]), "d"(a[3]), "d"(b[0]), "d"(b[1]));
  }
  double s = 0;
  for (int j = 0; j < 8; ++j) for (int i = 0; i < 4; ++i) s += c[j][i];
  if (s == 12345.0) out[threadIdx.x] = s;
}
int main() {
  double* out; cudaMalloc(&out, 4096 * sizeof(double));
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  for (int threads : {128, 256}) for (int bps : {1, 2}) {
    int grid = sms * bps, iters = 5000; float ms;
    k16<<<grid, threads>>>(out, 10); cudaEventRecord(e0); k16<<<grid, threads>>>(out, iters); cudaEventRecord(e1); cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    printf("{\"kind\":\"dmma16x8x16\",\"threads\":%d,\"grid\":%d,\"tflops\":%.3f}\n", threads, grid, 2.0*16*8*16*8.0*iters*grid*(threads/32)/ms/1e9);
    k8<<<grid, threads>>>(out, 10); cudaEventRecord(e0); k8<<<grid, threads>>>(out, iters); cudaEventRecord(e1); cudaEventSynchronize(e1);
    cudaEventElapsedTime(&ms, e0, e1);
    printf("{\"kind\":\"dmma16x8x8\",\"threads\":%d,\"grid\":%d,\"tflops\":%.3f}\n", threads, grid, 2.0*16*8*8*8.0*iters*grid*(threads/32)/ms/1e9);
  }
  printf("{\"err\":\"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
}
