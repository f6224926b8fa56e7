// Microbenchmark: FP64 DMMA (mma.sync m8n8k4 f64) vs DFMA issue throughput on sm_100a.
#include <cstdio>
#include <cuda_runtime.h>
__global__ void dmma_loop(double* out, int iters) {
  double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-4;
  double c[8][2];
  for (int i = 0; i < 8; i++) { c[i][0] = i; c[i][1] = threadIdx.x+i; }
  for (int it = 0; it < iters; it++) {
#pragma unroll
    for (int i = 0; i < 8; i++) {
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                   : "+d"(c[i][0]), "+d"(c[i][1]) : "d"(a), "d"(b));
    }
  }
  double s = 0; for (int i = 0; i < 8; i++) s += c[i][0] + c[i][1];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void dfma_loop(double* out, int iters) {
  double a = threadIdx.x * 1e-3, b = 1.0 + threadIdx.x * 1e-4;
  double c[16];
  for (int i = 0; i < 16; i++) c[i] = i;
  for (int it = 0; it < iters; it++) {
#pragma unroll
    for (int i = 0; i < 16; i++) c[i] = fma(a, c[i], b);
  }
  double s = 0; for (int i = 0; i < 16; i++) s += c[i];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
__global__ void dmma_lat(double* out, long long* cyc, int iters) {
  double a = threadIdx.x * 1e-3, b = 1.0; double c0 = 0, c1 = 0;
  long long t0 = clock64();
  for (int it = 0; it < iters; it++)
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                 : "+d"(c0), "+d"(c1) : "d"(a), "d"(b));
  long long t1 = clock64();
  out[threadIdx.x] = c0 + c1; if (threadIdx.x == 0) *cyc = t1 - t0;
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  printf("SMs %d clock %d kHz\n", sms, clk);
  double* out; cudaMalloc(&out, 1 << 26); long long* cyc; cudaMalloc(&cyc, 8);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int iters = 20000;
  for (int warps : {4, 8, 16, 32}) {
    for (int rep = 0; rep < 2; rep++) {
      int grid = sms * 2; int threads = warps * 32 / 2;
      dmma_loop<<<grid, threads>>>(out, 100);
      cudaEventRecord(e0); dmma_loop<<<grid, threads>>>(out, iters); cudaEventRecord(e1);
      cudaEventSynchronize(e1); float ms; cudaEventElapsedTime(&ms, e0, e1);
      double flops = (double)grid * (threads / 32) * iters * 8 * 512.0;
      if (rep) printf("DMMA warps/SM %2d : %.2f TFLOP/s\n", warps, flops / ms / 1e9);
    }
  }
  for (int warps : {4, 8, 16, 32}) {
    int grid = sms * 2; int threads = warps * 32 / 2;
    dfma_loop<<<grid, threads>>>(out, 100);
    cudaEventRecord(e0); dfma_loop<<<grid, threads>>>(out, iters); cudaEventRecord(e1);
    cudaEventSynchronize(e1); float ms; cudaEventElapsedTime(&ms, e0, e1);
    double flops = (double)grid * threads * iters * 16 * 2.0;
    printf("DFMA warps/SM %2d : %.2f TFLOP/s\n", warps, flops / ms / 1e9);
  }
  dmma_lat<<<1, 32>>>(out, cyc, 1000); long long hc; cudaMemcpy(&hc, cyc, 8, cudaMemcpyDeviceToHost);
  printf("DMMA dependent latency: %.1f cyc\n", hc / 1000.0);
  return 0;
}
