// Cycle counts of the pieces of one 8-column step of the dataflow panel's potrf
// (kernels.cu: factor_diag8, potrf_rows8, upd_block8), each timed alone in one
// warp on a 64 x 64 SPD tile in shared memory (clock64, 100 repetitions).
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I include \
//        -I paper_conf_ipps_georgesgsc11_b200/csrc tools/ubench/potrf_parts.cu -o tools/ubench/potrf_parts
#include "../../paper_conf_ipps_georgesgsc11_b200/csrc/kernels.cu"

#include <cstdio>

using namespace mf;

// variant of factor_diag8 (kernels.cu) with a one-step, second-order rsqrt refinement
__device__ __forceinline__ double rsqrt_h2(double x) {
    double y;
    asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
    const double r = fma(-x * y, y, 1.0);      // 1 - x y^2
    const double p = fma(0.375, r, 0.5);       // 1/2 + 3 r / 8
    return fma(y * r, p, y);                   // y (1 + r/2 + 3 r^2/8)
}
__device__ __forceinline__ void factor_diag8_h2(double *A, double *sinv, int s0, int nb) {
    constexpr int SB = 8;
    double a[SB][SB];
#pragma unroll
    for (int c = 0; c < SB; c++)
#pragma unroll
        for (int r = c; r < SB; r++) a[r][c] = (r < nb) ? A[(s0 + c) * kPLD + s0 + r] : (r == c ? 1.0 : 0.0);
#pragma unroll
    for (int q = 0; q < SB; q++) {
        const double dq = a[q][q];
        const double inv = rsqrt_h2(dq);
        if (q + 1 < SB) {
            a[q + 1][q] *= inv;
            a[q + 1][q + 1] = fma(-a[q + 1][q], a[q + 1][q], a[q + 1][q + 1]);
        }
        a[q][q] = dq * inv;
        sinv[s0 + q] = inv;
#pragma unroll
        for (int r = q + 2; r < SB; r++) a[r][q] *= inv;
#pragma unroll
        for (int c = q + 1; c < SB; c++)
#pragma unroll
            for (int r = c; r < SB; r++)
                if (r != q + 1) a[r][c] = fma(-a[r][q], a[c][q], a[r][c]);
    }
#pragma unroll
    for (int c = 0; c < SB; c++)
#pragma unroll
        for (int r = c; r < SB; r++)
            if (r < nb) A[(s0 + c) * kPLD + s0 + r] = a[r][c];
}

__device__ __forceinline__ void nbar_arrive(int id, int n) { asm volatile("bar.arrive %0, %1;" ::"r"(id), "r"(n) : "memory"); }
// one row of the row solve of panel_potrf_dmma (kernels.cu), as a function
__device__ __forceinline__ void potrf_rows8(double *A, const double *sinv, int s0, int nb, int r) {
    double x[8];
#pragma unroll
    for (int q = 0; q < 8; q++) x[q] = (q < nb) ? A[(s0 + q) * kPLD + r] : 0.0;
#pragma unroll
    for (int q = 0; q < 8; q++)
        if (q < nb) {
            x[q] *= sinv[s0 + q];
#pragma unroll
            for (int q2 = q + 1; q2 < 8; q2++)
                if (q2 < nb) x[q2] = fma(-x[q], A[(s0 + q) * kPLD + s0 + q2], x[q2]);
        }
#pragma unroll
    for (int q = 0; q < 8; q++)
        if (q < nb) A[(s0 + q) * kPLD + r] = x[q];
}

__global__ void parts(DevPlan d, long long *out) {
    __shared__ double A[64 * kPLD];
    __shared__ double sinv[64];
    const int tid = threadIdx.x, lane = tid & 31;
    for (int q = tid; q < 64 * kPLD; q += blockDim.x) {
        const int r = q % kPLD, c = q / kPLD;
        A[q] = (r == c) ? 64.0 : 1.0 / (1 + r + c);
    }
    __syncthreads();
    long long t0, t1, acc[4] = {0, 0, 0, 0};
    for (int it = 0; it < 100; it++) {
        __syncwarp();
        t0 = clock64();
        if (lane == 0) factor_diag8(d, A, sinv, 0, 8, 0);
        __syncwarp();
        t1 = clock64();
        acc[0] += t1 - t0;
        t0 = clock64();
        if (lane < 8) potrf_rows8(A, sinv, 0, 8, 8 + lane);
        __syncwarp();
        t1 = clock64();
        acc[1] += t1 - t0;
        t0 = clock64();
        upd_block8(A, 1, 1, 0);
        __syncwarp();
        t1 = clock64();
        acc[2] += t1 - t0;
        t0 = clock64();
        if (lane == 0) factor_diag8_h2(A, sinv, 0, 8);
        __syncwarp();
        t1 = clock64();
        acc[3] += t1 - t0;
        // restore
        for (int q = lane; q < 16 * kPLD; q += 32) {
            const int r = q % kPLD, c = q / kPLD;
            A[q] = (r == c) ? 64.0 : 1.0 / (1 + r + c);
        }
        __syncwarp();
    }
    if (tid == 0)
        for (int i = 0; i < 4; i++) out[i] = acc[i] / 100;
}

template <int V>
__global__ void whole(DevPlan d, long long *out) {
    __shared__ double A[64 * kPLD];
    __shared__ double sinv[64];
    const int tid = threadIdx.x;
    long long acc = 0, g0 = 0, g1 = 0;
    for (int it = 0; it < 20; it++) {
        for (int q = tid; q < 64 * kPLD; q += blockDim.x) {
            const int r = q % kPLD, c = q / kPLD;
            A[q] = (r == c) ? 64.0 : 1.0 / (1 + r + c);
        }
        __syncthreads();
        const long long t0 = clock64();
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g0));
        if (V == 0) panel_potrf_dmma(d, A, sinv, 64, 64, 0);
        else panel_potrf_dmma(d, A, sinv, 64, 64, 0);
        const long long t1 = clock64();
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g1));
        acc += t1 - t0;
        __syncthreads();
    }
    if (tid == 0) { out[0] = acc / 20; out[1] = g1 - g0; }
}

// warp 0: factor_diag8 x 100 (cycles); warps 1-3 meanwhile: 0 idle, 1 DMMA loop, 2 DFMA loop, 3 LDS/STS loop
template <int BG>
__global__ void interfere(DevPlan d, long long *out) {
    __shared__ double A[64 * kPLD];
    __shared__ double sinv[64];
    __shared__ volatile int stop;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    for (int q = tid; q < 64 * kPLD; q += blockDim.x) {
        const int r = q % kPLD, c = q / kPLD;
        A[q] = (r == c) ? 64.0 : 1.0 / (1 + r + c);
    }
    if (tid == 0) stop = 0;
    __syncthreads();
    if (warp == 0) {
        long long acc = 0;
        for (int it = 0; it < 100; it++) {
            __syncwarp();
            const long long t0 = clock64();
            if (lane == 0) factor_diag8(d, A, sinv, 0, 8, 0);
            __syncwarp();
            acc += clock64() - t0;
            for (int q = lane; q < 8 * kPLD; q += 32) {
                const int r = q % kPLD, c = q / kPLD;
                A[q] = (r == c) ? 64.0 : 1.0 / (1 + r + c);
            }
            __syncwarp();
        }
        if (lane == 0) { out[0] = acc / 100; stop = 1; }
    } else if (BG > 0) {
        double c0 = lane, c1 = 1.0, a = 1e-3 * lane, b = 1e-3;
        double *B = A + 16 * kPLD + 8 * warp;
        while (!stop) {
#pragma unroll 4
            for (int i = 0; i < 64; i++) {
                if (BG == 1) dmma(c0, c1, a, b);
                else if (BG == 2) { c0 = fma(c0, a, b); c1 = fma(c1, a, b); }
                else { B[lane] = B[lane + 1] + 1.0; }
            }
        }
        if (c0 == 12345.0) out[1] = (long long)c1;
    }
}

int main() {
    DevPlan d{};
    int *failed;
    cudaMalloc(&failed, 16);
    int hf[4] = {INT_MAX, 1, 0, 0};
    cudaMemcpy(failed, hf, 16, cudaMemcpyHostToDevice);
    d.failed = failed;
    long long *out;
    cudaMalloc(&out, 32);
    parts<<<1, 32>>>(d, out);
    parts<<<1, 32>>>(d, out);
    long long h[4];
    cudaMemcpy(h, out, 32, cudaMemcpyDeviceToHost);
    printf("factor_diag8 %lld cycles, potrf_rows8 %lld, upd_block8 %lld, factor_diag8 with 1-step rsqrt %lld (%s)\n", h[0], h[1], h[2],
           h[3], cudaGetErrorString(cudaGetLastError()));
    const char *bgn[4] = {"idle", "DMMA", "DFMA", "LDS/STS"};
    for (int bg = 0; bg < 4; bg++) {
        for (int rep = 0; rep < 2; rep++) {
            if (bg == 0) interfere<0><<<1, 128>>>(d, out);
            if (bg == 1) interfere<1><<<1, 128>>>(d, out);
            if (bg == 2) interfere<2><<<1, 128>>>(d, out);
            if (bg == 3) interfere<3><<<1, 128>>>(d, out);
        }
        cudaMemcpy(h, out, 8, cudaMemcpyDeviceToHost);
        printf("factor_diag8 with warps 1-3 %s: %lld cycles (%s)\n", bgn[bg], h[0], cudaGetErrorString(cudaGetLastError()));
    }
    for (int v = 0; v < 1; v++) {
        for (int rep = 0; rep < 2; rep++) whole<0><<<1, 128>>>(d, out);
        cudaMemcpy(h, out, 16, cudaMemcpyDeviceToHost);
        printf("%s 64x64: %lld cycles, last call %lld ns (%s)\n", v == 0 ? "panel_potrf_dmma" : "panel_potrf_la", h[0], h[1],
               cudaGetErrorString(cudaGetLastError()));
    }
    return 0;
}
