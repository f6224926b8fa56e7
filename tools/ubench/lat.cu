// Dependent-latency microbenchmark of the fp64 operations on the pivot chain.
#include <cstdio>
#include <cuda_runtime.h>
__device__ __forceinline__ double fast_rsqrt(double x) {
    double y = (double)rsqrtf((float)x);
    double h = x * y; double r = fma(-h, y, 1.0); y = fma(0.5 * y, r, y);
    h = x * y; r = fma(-h, y, 1.0); return fma(0.5 * y, r, y);
}
template <int OP>
__global__ void chain(double *out, long long *cyc, double x0, int n) {
    double x = x0 + threadIdx.x * 1e-9;
    long long t0 = clock64();
    for (int i = 0; i < n; i++) {
        if (OP == 0) x = fma(x, 0.999999, 1e-7);
        if (OP == 1) x = rsqrt(x) + 1.0;
        if (OP == 2) x = fast_rsqrt(x) + 1.0;
        if (OP == 3) x = __drcp_rn(x) + 1.0;
        if (OP == 4) x = sqrt(x) + 1.0;
        if (OP == 5) x = __shfl_sync(0xffffffffu, x, (threadIdx.x + 1) & 31) * 0.9999999;
        if (OP == 6) x = 1.0 / x + 1.0;
    }
    long long t1 = clock64();
    out[threadIdx.x] = x;
    if (threadIdx.x == 0) *cyc = t1 - t0;
}
template <int OP>
void run(const char *name, double *out, long long *cyc) {
    const int n = 4096;
    chain<OP><<<1, 32>>>(out, cyc, 1.5, n);
    chain<OP><<<1, 32>>>(out, cyc, 1.5, n);
    long long h; cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("%-28s %.1f cycles/op\n", name, (double)h / n);
}
int main1() {
    double *out; long long *cyc; cudaMalloc(&out, 256); cudaMalloc(&cyc, 8);
    run<0>("DFMA dependent", out, cyc);
    run<1>("rsqrt(double) + add", out, cyc);
    run<2>("float-seed 2-Newton + add", out, cyc);
    run<3>("__drcp_rn + add", out, cyc);
    run<4>("sqrt(double) + add", out, cyc);
    run<5>("shfl + DMUL", out, cyc);
    run<6>("1.0/x + add", out, cyc);
    return 0;
}
// (appended) latency of a register-resident 8x8 Cholesky in one thread
__global__ void chol8(double *out, long long *cyc, int n) {
    double a[8][8];
    for (int r = 0; r < 8; r++) for (int c = 0; c < 8; c++) a[r][c] = (r == c) ? 10.0 + threadIdx.x : 0.5;
    long long t0 = clock64();
    for (int it = 0; it < n; it++) {
#pragma unroll
        for (int q = 0; q < 8; q++) {
            const double inv = rsqrt(a[q][q]);
            a[q][q] *= inv;
#pragma unroll
            for (int r = q + 1; r < 8; r++) a[r][q] *= inv;
#pragma unroll
            for (int c = q + 1; c < 8; c++)
#pragma unroll
                for (int r = c; r < 8; r++) a[r][c] = fma(-a[r][q], a[c][q], a[r][c]);
        }
        // restore a SPD matrix that depends on the result (keeps the chain)
#pragma unroll
        for (int r = 0; r < 8; r++)
#pragma unroll
            for (int c = 0; c <= r; c++) a[r][c] = (r == c) ? 10.0 + a[r][c] * 1e-3 : 0.5 + a[r][c] * 1e-6;
    }
    long long t1 = clock64();
    double sacc = 0; for (int r = 0; r < 8; r++) for (int c = 0; c <= r; c++) sacc += a[r][c];
    out[threadIdx.x] = sacc;
    if (threadIdx.x == 0) *cyc = t1 - t0;
}
int main2() {
    double *out; long long *cyc; cudaMalloc(&out, 256); cudaMalloc(&cyc, 8);
    chol8<<<1, 1>>>(out, cyc, 100);
    chol8<<<1, 1>>>(out, cyc, 1000);
    long long h; cudaMemcpy(&h, cyc, 8, cudaMemcpyDeviceToHost);
    printf("register 8x8 cholesky: %.1f cycles per factorization (%.1f per pivot)\n", h / 1000.0, h / 8000.0);
    return 0;
}
int main() { main1(); main2(); return 0; }
