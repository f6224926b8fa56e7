// Cycle counts of the pieces of one 8-column step of the dataflow panel's potrf
// (kernels.cu: factor_diag8, potrf_rows8, upd_block8), each timed alone in one
// warp on a 64 x 64 SPD tile in shared memory (clock64, 100 repetitions).
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -I include \
//        -I paper_conf_ipps_georgesgsc11_b200/csrc tools/ubench/potrf_parts.cu -o tools/ubench/potrf_parts
#include "../../paper_conf_ipps_georgesgsc11_b200/csrc/kernels.cu"

#include <cstdio>

using namespace mf;

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
        nbar_arrive(1, 32);
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
        else panel_potrf_la(d, A, sinv, 64, 64, 0);
        const long long t1 = clock64();
        asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(g1));
        acc += t1 - t0;
        __syncthreads();
    }
    if (tid == 0) { out[0] = acc / 20; out[1] = g1 - g0; }
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
    printf("factor_diag8 %lld cycles, potrf_rows8 %lld, upd_block8 %lld, bar.arrive %lld (%s)\n", h[0], h[1], h[2],
           h[3], cudaGetErrorString(cudaGetLastError()));
    for (int v = 0; v < 2; v++) {
        for (int rep = 0; rep < 2; rep++) {
            if (v == 0) whole<0><<<1, 128>>>(d, out); else whole<1><<<1, 128>>>(d, out);
        }
        cudaMemcpy(h, out, 16, cudaMemcpyDeviceToHost);
        printf("%s 64x64: %lld cycles, last call %lld ns (%s)\n", v == 0 ? "panel_potrf_dmma" : "panel_potrf_la", h[0], h[1],
               cudaGetErrorString(cudaGetLastError()));
    }
    return 0;
}
