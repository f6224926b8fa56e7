// Latency / issue rate of mma.sync.m8n8k4.f64 (DMMA) in one warp: a chain of
// dependent DMMAs on one accumulator pair vs 2 / 4 / 8 independent chains.
//   nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/ubench/dmma_lat.cu -o tools/ubench/dmma_lat
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ void dmma(double &c0, double &c1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                 : "+d"(c0), "+d"(c1) : "d"(a), "d"(b));
}
template <int NC>
__global__ void chains(double *out, long long *cyc, int n) {
    double c[NC][2];
    for (int i = 0; i < NC; i++) c[i][0] = c[i][1] = threadIdx.x;
    const double a = 1e-9 * threadIdx.x, b = 1e-9;
    long long t0 = clock64();
    for (int it = 0; it < n; it++)
#pragma unroll
        for (int i = 0; i < NC; i++) dmma(c[i][0], c[i][1], a, b);
    long long t1 = clock64();
    double s = 0;
    for (int i = 0; i < NC; i++) s += c[i][0] + c[i][1];
    out[threadIdx.x] = s;
    if (threadIdx.x == 0) *cyc = t1 - t0;
}
template <int NC>
void run(double *out, long long *cyc) {
    const int n = 2048;
    chains<NC><<<1, 32>>>(out, cyc, n);
    chains<NC><<<1, 32>>>(out, cyc, n);
    long long h;
    cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("%d independent chain(s): %.1f cycles per DMMA (%.1f per chain step)\n", NC, (double)h / (n * NC), (double)h / n);
}
int main() {
    double *out; long long *cyc;
    cudaMalloc(&out, 256); cudaMalloc(&cyc, 8);
    run<1>(out, cyc); run<2>(out, cyc); run<4>(out, cyc); run<8>(out, cyc); run<16>(out, cyc);
    return 0;
}
