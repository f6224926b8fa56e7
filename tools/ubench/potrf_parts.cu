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


// instrumented copy of panel_potrf_dmma (kernels.cu): clock64 per phase, step 0..7
__device__ long long g_ph[8][6];
template <bool PAIR>
__device__ __forceinline__ void potrf_inst(const DevPlan &d, double *A, double *sinv, int R, int we) {
    constexpr int SB = 8;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int nrb = (R + 7) / 8, ncb = (we + 7) / 8;
    long long t0 = clock64();
    if (tid == 0) factor_diag8(d, A, sinv, 0, min(SB, we), 0);
    __syncthreads();
#pragma unroll 1
    for (int st = 0; st < ncb; st++) {
        const int s0 = st * SB, nb = min(SB, we - s0);
        const int rb = s0 + nb;
        if (rb >= R) break;
        long long ta = clock64();
        if (tid < R - rb) {
            const int r = rb + tid;
            double x[SB];
#pragma unroll
            for (int q = 0; q < SB; q++) x[q] = (q < nb) ? A[(s0 + q) * kPLD + r] : 0.0;
#pragma unroll
            for (int q = 0; q < SB; q++) {
                if (q < nb) {
                    x[q] *= sinv[s0 + q];
#pragma unroll
                    for (int q2 = q + 1; q2 < SB; q2++)
                        if (q2 < nb) x[q2] = fma(-x[q], A[(s0 + q) * kPLD + s0 + q2], x[q2]);
                }
            }
#pragma unroll
            for (int q = 0; q < SB; q++)
                if (q < nb) A[(s0 + q) * kPLD + r] = x[q];
        }
        long long tb = clock64();
        __syncthreads();
        long long tc = clock64();
        long long td = tc, te = tc;
        if (st + 1 < ncb) {
            const int J1 = st + 1;
            if (warp == 0) {
                upd_block8(A, J1, J1, s0);
                __syncwarp();
                td = clock64();
                if (lane == 0) factor_diag8(d, A, sinv, J1 * SB, min(SB, we - J1 * SB), 0);
                __syncwarp();
                te = clock64();
            } else {
                if (PAIR) {   // by block column: B fragments of column J loaded once, rows I in the column
                    const int gq = lane >> 2, tq = lane & 3;
                    for (int J = J1 + warp - 1; J < ncb; J += 3) {
                        double b0 = A[J * 8 + gq + (s0 + tq) * kPLD], b1 = A[J * 8 + gq + (s0 + 4 + tq) * kPLD];
                        for (int I = (J == J1 ? J + 1 : J); I < nrb; I++) {
                            double *Ci = A + I * 8 + gq;
                            double c0 = Ci[(J * 8 + 2 * tq) * kPLD], c1 = Ci[(J * 8 + 2 * tq + 1) * kPLD];
                            const double a0 = -Ci[(s0 + tq) * kPLD], a1 = -Ci[(s0 + 4 + tq) * kPLD];
                            dmma(c0, c1, a0, b0);
                            dmma(c0, c1, a1, b1);
                            Ci[(J * 8 + 2 * tq) * kPLD] = c0;
                            Ci[(J * 8 + 2 * tq + 1) * kPLD] = c1;
                        }
                    }
                } else {
                    int t = 0;
                    for (int J = J1; J < ncb; J++)
                        for (int I = (J == J1 ? J + 1 : J); I < nrb; I++, t++)
                            if (t % 3 == warp - 1) upd_block8(A, I, J, s0);
                }
                te = clock64();
            }
        }
        __shared__ long long wend[4];
        if (lane == 0) wend[warp] = te;
        __syncthreads();
        long long tf = clock64();
        if (tid == 0 && st < 8) {
            g_ph[st][0] = tb - ta;           // thread 0's row solve
            g_ph[st][1] = tc - ta;           // row solve + barrier
            g_ph[st][2] = td - tc;           // warp 0: upd_block8 (J1, J1)
            g_ph[st][3] = te - td;           // warp 0: factor_diag8
            g_ph[st][4] = max(max(wend[1], wend[2]), wend[3]) - tc;   // warps 1-3: trailing updates
            g_ph[st][5] = tf - tc;           // whole second half incl. barrier
        }
    }
    __syncthreads();
}
template <bool PAIR>
__global__ void inst_kernel(DevPlan d) {
    __shared__ double A[64 * kPLD];
    __shared__ double sinv[64];
    const int tid = threadIdx.x;
    for (int it = 0; it < 3; it++) {
        for (int q = tid; q < 64 * kPLD; q += blockDim.x) {
            const int r = q % kPLD, c = q / kPLD;
            A[q] = (r == c) ? 64.0 : 1.0 / (1 + r + c);
        }
        __syncthreads();
        potrf_inst<PAIR>(d, A, sinv, 64, 64);
    }
}

// trailing-update contention: NW warps (1..3) each run upd_block8 on 9 distinct blocks
template <int NW, bool W0>
__global__ void upd_contend(DevPlan d, long long *out) {
    __shared__ double A[64 * kPLD];
    __shared__ double B[16 * kPLD];
    __shared__ double sinv[64];
    const int tid = threadIdx.x, warp = tid >> 5;
    for (int q = tid; q < 64 * kPLD; q += blockDim.x) A[q] = 1.0 / (1 + q);
    for (int q = tid; q < 16 * kPLD; q += blockDim.x) { const int r = q % kPLD, c = q / kPLD; B[q] = (r == c) ? 64.0 : 1.0 / (1 + r + c); }
    __syncthreads();
    long long t0 = clock64();
    if (W0 && warp == 0 && (tid & 31) == 0)   // warp 0: the single-thread pivot block, as in the potrf
        for (int rep = 0; rep < 4; rep++) factor_diag8(d, B, sinv, 0, 8, 0);
    if (warp >= 1 && warp <= NW) {
        int t = 0;
        for (int J = 1; J < 8; J++)
            for (int I = J; I < 8; I++, t++)
                if (t % 3 == warp - 1) upd_block8(A, I, J, 0);
    }
    long long t1 = clock64();
    __syncthreads();
    if ((tid & 31) == 0 && warp >= 1 && warp <= NW) out[warp] = t1 - t0;
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
    {
        long long *o2; cudaMalloc(&o2, 64); cudaMemset(o2, 0, 64);
        long long hh[8];
        upd_contend<1, false><<<1, 128>>>(d, o2); upd_contend<1, false><<<1, 128>>>(d, o2); cudaMemcpy(hh, o2, 64, cudaMemcpyDeviceToHost);
        printf("trailing update, warp 1 alone (its ~9 blocks): %lld cycles\n", hh[1]);
        upd_contend<3, false><<<1, 128>>>(d, o2); upd_contend<3, false><<<1, 128>>>(d, o2); cudaMemcpy(hh, o2, 64, cudaMemcpyDeviceToHost);
        printf("trailing update, warps 1-3 together: %lld %lld %lld cycles\n", hh[1], hh[2], hh[3]);
        upd_contend<3, true><<<1, 128>>>(d, o2); upd_contend<3, true><<<1, 128>>>(d, o2); cudaMemcpy(hh, o2, 64, cudaMemcpyDeviceToHost);
        printf("trailing update, warps 1-3 while warp 0 lane 0 factors pivot blocks: %lld %lld %lld cycles\n", hh[1], hh[2], hh[3]);
    }
    for (int pair = 0; pair < 2; pair++) {
        if (pair) inst_kernel<true><<<1, 128>>>(d); else inst_kernel<false><<<1, 128>>>(d);
        cudaDeviceSynchronize();
        long long ph[8][6];
        cudaMemcpyFromSymbol(ph, g_ph, sizeof(ph));
        printf("potrf phases per step (cycles, %s): rows | rows+bar | w0 upd | w0 factor | w1-3 upd | 2nd half+bar\n",
               pair ? "by block column" : "one block at a time");
        for (int st = 0; st < 8; st++)
            printf("  step %d: %5lld %5lld %5lld %5lld %5lld %5lld\n", st, ph[st][0], ph[st][1], ph[st][2], ph[st][3], ph[st][4], ph[st][5]);
    }
    return 0;
}
