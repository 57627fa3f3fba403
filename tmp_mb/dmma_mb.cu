#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ void dmma(double (&d)[2], double a, double b) {
  asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
               : "+d"(d[0]), "+d"(d[1]) : "d"(a), "d"(b));
}
template <int CH>
__global__ void k(double* out, int iters, long long* cyc) {
  double acc[CH][2];
  for (int c = 0; c < CH; ++c) acc[c][0] = acc[c][1] = 0;
  double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-4;
  long long t0 = clock64();
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int c = 0; c < CH; ++c) dmma(acc[c], a, b);
  }
  long long t1 = clock64();
  double s = 0;
  for (int c = 0; c < CH; ++c) s += acc[c][0] + acc[c][1];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
  if (threadIdx.x == 0 && blockIdx.x == 0) *cyc = t1 - t0;
}
template <int CH>
void run(int blocks, int threads, int iters) {
  double* out; long long* cyc; cudaMalloc(&out, blocks * threads * 8); cudaMalloc(&cyc, 8);
  k<CH><<<blocks, threads>>>(out, iters, cyc);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  cudaEventRecord(e0);
  k<CH><<<blocks, threads>>>(out, iters, cyc);
  cudaEventRecord(e1); cudaEventSynchronize(e1);
  float ms; cudaEventElapsedTime(&ms, e0, e1);
  long long c; cudaMemcpy(&c, cyc, 8, cudaMemcpyDeviceToHost);
  double dm = (double)blocks * (threads / 32) * iters * CH;
  printf("CH=%d blocks=%d threads=%d: %.3f ms, %.2f TF/s, cycles/iter(warp0)=%.1f -> %.1f cyc per dmma per warp\n", CH, blocks,
         threads, ms, dm * 512 / ms / 1e9, (double)c / iters, (double)c / iters / CH);
}
int main() {
  run<1>(1, 32, 10000);
  run<4>(1, 32, 10000);
  run<8>(1, 32, 10000);
  run<16>(1, 32, 10000);
  run<8>(148, 128, 4000);
  run<8>(148, 256, 4000);
  run<8>(148, 512, 2000);
  run<16>(148, 512, 2000);
  run<4>(148, 1024, 2000);
  return 0;
}
