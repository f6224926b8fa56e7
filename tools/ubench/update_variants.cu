// Microbenchmark of DMMA Schur-update tile/pipeline variants on one large
// lower-trapezoid SYRK (M = N = 8192, K = 4096), the shape class that carries
// most of c5's flops.  Reports algorithmic TFLOP/s (lower trapezoid only) and
// checks that every variant produces bitwise the same C (the per-element
// summation order does not depend on the tile shape).
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>
#include "dmma_update.cuh"

using namespace mf;

template <class Cfg, bool BULK = false>
double run(const char *name, double *L, double *U, int M, int N, int K, int ld, std::vector<double> &out,
           int aoff = 0, int reps = 5) {
    std::vector<TileTask> tiles;
    const int tm = (M + Cfg::BM - 1) / Cfg::BM, tn = (N + Cfg::BN - 1) / Cfg::BN;
    for (int tj = 0; tj < tn; tj++)
        for (int ti = 0; ti < tm; ti++) {
            if ((int64_t)(ti + 1) * Cfg::BM - 1 < (int64_t)tj * Cfg::BN) continue;
            tiles.push_back({0, (ti << 16) | tj});
        }
    GemmProb g{aoff, 0, ld, M, M, N, K, 1};
    GemmProb *dp;
    TileTask *dt;
    cudaMalloc(&dp, sizeof(g));
    cudaMalloc(&dt, tiles.size() * sizeof(TileTask));
    cudaMemcpy(dp, &g, sizeof(g), cudaMemcpyHostToDevice);
    cudaMemcpy(dt, tiles.data(), tiles.size() * sizeof(TileTask), cudaMemcpyHostToDevice);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float best = 1e30f;
    for (int r = 0; r < reps + 1; r++) {
        cudaMemset(U, 0, (size_t)M * M * sizeof(double));
        cudaEventRecord(e0);
        launch_update_t<Cfg, BULK>(L, U, dp, dt, (int64_t)tiles.size(), 0);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms;
        cudaEventElapsedTime(&ms, e0, e1);
        if (r) best = ms < best ? ms : best;
    }
    cudaError_t err = cudaGetLastError();
    const double flops = 2.0 * K * ((double)N * (N + 1) / 2 + (double)(M - N) * N);
    const double tf = flops / (best * 1e-3) / 1e12;
    std::vector<double> h((size_t)M * M);
    cudaMemcpy(h.data(), U, h.size() * sizeof(double), cudaMemcpyDeviceToHost);
    bool same = true;
    if (out.empty()) out = h;
    else
        for (int j = 0; j < N && same; j++)
            for (int i = j; i < M; i++)
                if (h[i + (size_t)j * M] != out[i + (size_t)j * M]) { same = false; break; }
    printf("a_off=%d %-34s tiles=%7zu  %8.3f ms  %6.2f TF/s  regs/smem=%zuKB  %s %s\n", aoff, name, tiles.size(), best, tf,
           Cfg::SMEM / 1024, same ? "bitwise-equal" : "MISMATCH", err == cudaSuccess ? "" : cudaGetErrorString(err));
    cudaFree(dp);
    cudaFree(dt);
    return tf;
}

int main(int argc, char **argv) {
    setvbuf(stdout, nullptr, _IONBF, 0);
    int M = 8192, K = 4096;
    if (argc > 1) M = atoi(argv[1]);
    if (argc > 2) K = atoi(argv[2]);
    const int N = M, ld = M + 2;   // odd shift exercised by a_off = 1
    double *L, *U;
    cudaMalloc(&L, ((size_t)ld * K + 256) * sizeof(double));
    cudaMalloc(&U, (size_t)M * M * sizeof(double));
    std::vector<double> hA((size_t)ld * K + 16);
    srand(1);
    for (auto &x : hA) x = (double)(rand() % 17 - 8);   // small integers: exact sums, any order
    cudaMemcpy(L, hA.data(), hA.size() * sizeof(double), cudaMemcpyHostToDevice);
    double *Lshift = L;   // a_off = 0 here: the kernel requires even first rows (the planner shifts odd ones)
    std::vector<double> ref;
    printf("lower-trapezoid SYRK M=N=%d K=%d\n", M, K);
    std::vector<double> ref1;
    run<UpdCfg<64, 64, 16, 3, 2, 2, 4>>("64x64 bk16 s3 w2x2 m4", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<64, 64, 16, 3, 2, 2, 4>, true>("BULK 64x64 bk16 s3 w2x2 m4", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<128, 64, 16, 3, 4, 2, 2>, true>("BULK 128x64 bk16 s3 w4x2 m2", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<128, 64, 16, 4, 4, 2, 2>, true>("BULK 128x64 bk16 s4 w4x2 m2", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<64, 128, 16, 4, 2, 4, 2>, true>("BULK 64x128 bk16 s4 w2x4 m2", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<128, 128, 16, 3, 4, 4, 1>, true>("BULK 128x128 bk16 s3 w4x4 m1", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<64, 64, 32, 2, 2, 2, 3>, true>("BULK 64x64 bk32 s2 w2x2 m3", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<64, 64, 16, 4, 2, 2, 3>, true>("BULK 64x64 bk16 s4 w2x2 m3", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<128, 64, 16, 3, 2, 2, 2>, true>("BULK 128x64 bk16 s3 w2x2 (64x32) m2", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<64, 64, 16, 4, 2, 2, 3>>("64x64 bk16 s4 w2x2 m3", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<64, 64, 32, 2, 2, 2, 3>>("64x64 bk32 s2 w2x2 m3", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<64, 64, 32, 3, 2, 2, 2>>("64x64 bk32 s3 w2x2 m2", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<128, 64, 16, 4, 4, 2, 2>>("128x64 bk16 s4 w4x2 m2", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<128, 64, 16, 3, 2, 2, 2>>("128x64 bk16 s3 w2x2 (64x32) m2", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<64, 128, 16, 3, 2, 2, 2>>("64x128 bk16 s3 w2x2 (32x64) m2", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<128, 128, 16, 4, 4, 4, 1>>("128x128 bk16 s4 w4x4 m1", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<64, 128, 16, 3, 2, 4, 2>>("64x128 bk16 s3 w2x4 m2", Lshift, U, M, N, K, ld, ref);
    run<UpdCfg<128, 128, 16, 3, 2, 2, 1>>("128x128 bk16 s3 w2x2 (64x64) m1", Lshift, U, M, N, K, ld, ref);
    return 0;
}
