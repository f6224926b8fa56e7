// Latency microbenchmark of the 64x64 diagonal-block potrf (one CTA), with
// phases switched off one at a time to see where the time goes.
#include <cstdio>
#include <cuda_runtime.h>
#include <cmath>
#include <vector>
constexpr int kWmax = 64;
__device__ __forceinline__ double fast_rsqrt(double x) {
    // float MUFU seed (~22 bits) + two Newton steps in fp64 (exact for powers of 4)
    double y = (double)rsqrtf((float)x);
    double h = x * y;
    double r = fma(-h, y, 1.0);
    y = fma(0.5 * y, r, y);
    h = x * y;
    r = fma(-h, y, 1.0);
    y = fma(0.5 * y, r, y);
    return y;
}
template <int PHASES, bool USE_RSQRT>
__global__ void __launch_bounds__(256) potrf64(double *P, int ld, int we, long long *clk) {
    constexpr int LDA = kWmax;
    __shared__ double A[kWmax * LDA];
    __shared__ double sinv[kWmax];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    long long t0 = clock64();
    {
        const int i = tid & 63, h = tid >> 6;
        double v[kWmax / 4];
#pragma unroll
        for (int t = 0; t < kWmax / 4; t++) {
            const int c = h + 4 * t;
            v[t] = (i < we && c < we) ? P[i + (int64_t)c * ld] : 0.0;
        }
#pragma unroll
        for (int t = 0; t < kWmax / 4; t++) A[(h + 4 * t) * LDA + i] = v[t];
    }
    __syncthreads();
    long long ta = 0, tb = 0, tc = 0;
#pragma unroll 1
    for (int s0 = 0; s0 < we; s0 += 16) {
        const int nb = min(16, we - s0);
        long long x0 = clock64();
        if ((PHASES & 8) && warp == 0) {
            // column broadcast through shared memory (LDS.128 pairs) instead of 15 shuffles per pivot
            __shared__ __align__(16) double colbuf[16];
            const int l = lane & 15;
            double a[16];
#pragma unroll
            for (int q = 0; q < 16; q++) a[q] = (q <= l && l < nb) ? A[(s0 + q) * LDA + s0 + l] : 0.0;
#pragma unroll
            for (int q = 0; q < 16; q++) {
                if (q < nb) {
                    const double dq = __shfl_sync(0xffffffffu, a[q], q);
                    const double inv = rsqrt(dq);
                    const double lq = (l == q) ? dq * inv : a[q] * inv;
                    if (l >= q) a[q] = lq;
                    if (l == q) sinv[s0 + q] = inv;
                    if (lane >= q && lane < 16) colbuf[lane] = lq;
                    __syncwarp();
#pragma unroll
                    for (int c = (q + 1) & ~1; c < 16; c += 2) {
                        const double2 lc = *reinterpret_cast<const double2 *>(colbuf + c);
                        if (c > q && l >= c) a[c] = fma(-lq, lc.x, a[c]);
                        if (l >= c + 1) a[c + 1] = fma(-lq, lc.y, a[c + 1]);
                    }
                    __syncwarp();
                }
            }
            if (lane < nb) {
#pragma unroll
                for (int q = 0; q < 16; q++)
                    if (q <= lane) {
                        A[(s0 + q) * LDA + s0 + lane] = a[q];
                        P[(s0 + lane) + (int64_t)(s0 + q) * ld] = a[q];
                    }
            }
        }
        if ((PHASES & 1) && warp == 0) {
            const int l = lane & 15;
            double a[16];
#pragma unroll
            for (int q = 0; q < 16; q++) a[q] = (q <= l && l < nb) ? A[(s0 + q) * LDA + s0 + l] : 0.0;
#pragma unroll
            for (int q = 0; q < 16; q++) {
                if (q < nb) {
                    const double dq = __shfl_sync(0xffffffffu, a[q], q);
                    const double inv = USE_RSQRT ? fast_rsqrt(dq) : rsqrt(dq);
                    const double piv = dq * inv;
                    if (lane == q) {
                        sinv[s0 + q] = inv;
                        a[q] = piv;
                    } else if (l > q) {
                        a[q] *= inv;
                    }
#pragma unroll
                    for (int c = q + 1; c < 16; c++) {
                        const double lc = __shfl_sync(0xffffffffu, a[q], c);
                        if (l >= c) a[c] -= a[q] * lc;
                    }
                }
            }
            if (lane < nb) {
#pragma unroll
                for (int q = 0; q < 16; q++)
                    if (q <= lane) {
                        A[(s0 + q) * LDA + s0 + lane] = a[q];
                        P[(s0 + lane) + (int64_t)(s0 + q) * ld] = a[q];
                    }
            }
        }
        __syncthreads();
        long long x1 = clock64();
        const int r0 = s0 + 16;
        if (r0 >= we) { ta += x1 - x0; break; }
        if ((PHASES & 2) && tid < we - r0) {
            const int r = r0 + tid;
            double x[16];
#pragma unroll
            for (int q = 0; q < 16; q++) x[q] = A[(s0 + q) * LDA + r];
#pragma unroll
            for (int q = 0; q < 16; q++) {
                x[q] *= sinv[s0 + q];
#pragma unroll
                for (int q2 = q + 1; q2 < 16; q2++) x[q2] -= x[q] * A[(s0 + q) * LDA + s0 + q2];
            }
#pragma unroll
            for (int q = 0; q < 16; q++) {
                A[(s0 + q) * LDA + r] = x[q];
                P[r + (int64_t)(s0 + q) * ld] = x[q];
            }
        }
        __syncthreads();
        long long x2 = clock64();
        if (PHASES & 4) {
            const int i = tid & 63, h = tid >> 6;
            if (i >= r0 && i < we) {
                double li[16];
#pragma unroll
                for (int q = 0; q < 16; q++) li[q] = A[(s0 + q) * LDA + i];
                for (int c = r0 + h; c <= i; c += 4) {
                    double acc = A[c * LDA + i];
#pragma unroll
                    for (int q = 0; q < 16; q++) acc -= li[q] * A[(s0 + q) * LDA + c];
                    A[c * LDA + i] = acc;
                }
            }
        }
        __syncthreads();
        long long x3 = clock64();
        ta += x1 - x0; tb += x2 - x1; tc += x3 - x2;
    }
    if (tid == 0) { clk[0] = clock64() - t0; clk[1] = ta; clk[2] = tb; clk[3] = tc; }
}

// 8-wide sub-blocks: the 8x8 diagonal block is factored by ONE thread in registers
// (independent FMAs pipeline; no shuffles, no barriers on the pivot chain)
__global__ void __launch_bounds__(256) potrf64_b8(double *P, int ld, int we, long long *clk) {
    constexpr int LDA = kWmax;
    __shared__ double A[kWmax * LDA];
    __shared__ double sinv[kWmax];
    const int tid = threadIdx.x;
    long long t0 = clock64();
    {
        const int i = tid & 63, h = tid >> 6;
        double v[kWmax / 4];
#pragma unroll
        for (int t = 0; t < kWmax / 4; t++) {
            const int c = h + 4 * t;
            v[t] = (i < we && c < we) ? P[i + (int64_t)c * ld] : 0.0;
        }
#pragma unroll
        for (int t = 0; t < kWmax / 4; t++) A[(h + 4 * t) * LDA + i] = v[t];
    }
    __syncthreads();
    long long ta = 0, tb = 0, tc = 0;
#pragma unroll 1
    for (int s0 = 0; s0 < we; s0 += 8) {
        const int nb = min(8, we - s0);
        long long x0 = clock64();
        if (tid == 0) {
            double a[8][8];
#pragma unroll
            for (int c = 0; c < 8; c++)
#pragma unroll
                for (int r = c; r < 8; r++) a[r][c] = (r < nb) ? A[(s0 + c) * LDA + s0 + r] : (r == c ? 1.0 : 0.0);
#pragma unroll
            for (int q = 0; q < 8; q++) {
                const double inv = rsqrt(a[q][q]);
                a[q][q] *= inv;
                sinv[s0 + q] = inv;
#pragma unroll
                for (int r = q + 1; r < 8; r++) a[r][q] *= inv;
#pragma unroll
                for (int c = q + 1; c < 8; c++)
#pragma unroll
                    for (int r = c; r < 8; r++) a[r][c] = fma(-a[r][q], a[c][q], a[r][c]);
            }
#pragma unroll
            for (int c = 0; c < 8; c++)
#pragma unroll
                for (int r = c; r < 8; r++)
                    if (r < nb) A[(s0 + c) * LDA + s0 + r] = a[r][c];
        }
        __syncthreads();
        long long x1 = clock64();
        const int r0 = s0 + 8;
        if (r0 >= we) { ta += x1 - x0; break; }
        if (tid < we - r0) {
            const int r = r0 + tid;
            double x[8];
#pragma unroll
            for (int q = 0; q < 8; q++) x[q] = A[(s0 + q) * LDA + r];
#pragma unroll
            for (int q = 0; q < 8; q++) {
                x[q] *= sinv[s0 + q];
#pragma unroll
                for (int q2 = q + 1; q2 < 8; q2++) x[q2] -= x[q] * A[(s0 + q) * LDA + s0 + q2];
            }
#pragma unroll
            for (int q = 0; q < 8; q++) A[(s0 + q) * LDA + r] = x[q];
        }
        __syncthreads();
        long long x2 = clock64();
        {
            const int i = tid & 63, h = tid >> 6;
            if (i >= r0 && i < we) {
                double li[8];
#pragma unroll
                for (int q = 0; q < 8; q++) li[q] = A[(s0 + q) * LDA + i];
                for (int c = r0 + h; c <= i; c += 4) {
                    double acc = A[c * LDA + i];
#pragma unroll
                    for (int q = 0; q < 8; q++) acc -= li[q] * A[(s0 + q) * LDA + c];
                    A[c * LDA + i] = acc;
                }
            }
        }
        __syncthreads();
        long long x3 = clock64();
        ta += x1 - x0; tb += x2 - x1; tc += x3 - x2;
    }
    __syncthreads();
    for (int c = tid >> 6; c < we; c += 4) {   // coalesced write-back of the lower triangle
        const int i = tid & 63;
        if (i < we && i >= c) P[i + (int64_t)c * ld] = A[c * LDA + i];
    }
    if (tid == 0) { clk[0] = clock64() - t0; clk[1] = ta; clk[2] = tb; clk[3] = tc; }
}

template <int PH, bool R>
void run(const char *name, double *P, long long *clk) {
    potrf64<PH, R><<<1, 256>>>(P, 64, 64, clk);
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    cudaEventRecord(e0);
    for (int i = 0; i < 20; i++) potrf64<PH, R><<<1, 256>>>(P, 64, 64, clk);
    cudaEventRecord(e1); cudaEventSynchronize(e1);
    float ms; cudaEventElapsedTime(&ms, e0, e1);
    long long h[4]; cudaMemcpy(h, clk, sizeof(h), cudaMemcpyDeviceToHost);
    printf("%-28s %7.2f us/launch  clk total %lld  a %lld  b %lld  c %lld\n", name, ms * 1000 / 20, h[0], h[1], h[2], h[3]);
}
int main() {
    std::vector<double> A(64 * 64, 0.0);
    for (int i = 0; i < 64; i++) for (int j = 0; j <= i; j++) A[i + j * 64] = (i == j) ? 100.0 : -0.5;
    double *P; cudaMalloc(&P, A.size() * 8); long long *clk; cudaMalloc(&clk, 64);
    cudaMemcpy(P, A.data(), A.size() * 8, cudaMemcpyHostToDevice);
    run<7, false>("all phases rsqrt", P, clk);
    run<14, false>("all phases, pipelined (a)", P, clk);
    run<1, false>("a only", P, clk);
    run<8, false>("a pipelined only", P, clk);
    run<2, true>("b only", P, clk);
    run<4, true>("c only", P, clk);
    run<0, true>("none (load+barriers)", P, clk);
    {
        potrf64_b8<<<1, 256>>>(P, 64, 64, clk);
        cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
        cudaEventRecord(e0);
        for (int i = 0; i < 20; i++) potrf64_b8<<<1, 256>>>(P, 64, 64, clk);
        cudaEventRecord(e1); cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        long long h[4]; cudaMemcpy(h, clk, sizeof(h), cudaMemcpyDeviceToHost);
        printf("%-28s %7.2f us/launch  clk total %lld  a %lld  b %lld  c %lld\n", "8-wide single-thread", ms * 1000 / 20, h[0], h[1], h[2], h[3]);
    }
    return 0;
}
