// Microbenchmark + check of the Ozaki-scheme Schur update (csrc/ozaki_update.cuh)
// against the FP64 DMMA update (csrc/dmma_update.cuh) on one lower-trapezoid SYRK
// C -= A A[0:N]^T (M x K, column-major): accuracy of sampled entries against a
// long-double reference (error in units of u * sum_p |A_ip A_jp|), and time.
//   ozaki_gemm [M N K]
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <random>
#include <vector>
#include <cuda_runtime.h>

#include "dmma_update.cuh"
#include "ozaki_update.cuh"

using namespace mf;
using Big = UpdCfg<64, 64, 16, 3, 2, 2, 4>;

#define CK(x)                                                                              \
    do {                                                                                   \
        cudaError_t e_ = (x);                                                              \
        if (e_ != cudaSuccess) {                                                           \
            printf("CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); \
            exit(1);                                                                       \
        }                                                                                  \
    } while (0)

template <int S>
float run_oz(double *dL, double *dU, GemmProb *dprob, int M, int N, int K, int reps, const double *C0, size_t cbytes,
             int wide = 0) {
    const int BN = wide ? 128 : kOzBN;
    OzProb op{0, (M + kOzBM - 1) / kOzBM * kOzBM, (K + kOzBK - 1) / kOzBK * kOzBK, 0, 0, 0};
    std::vector<int32_t> tasks;
    for (int rb = 0; rb < op.Mpad / kOzBM; rb++)
        for (int sg = 0; sg < (op.Kpad + kOzSeg - 1) / kOzSeg; sg++) tasks.insert(tasks.end(), {0, rb, sg});
    std::vector<OzTile> tiles;
    for (int tj = 0; tj < (N + BN - 1) / BN; tj++)
        for (int ti = 0; ti < op.Mpad / kOzBM; ti++)
            if ((ti + 1) * kOzBM > tj * BN) tiles.push_back({0, (ti << 16) | tj});
    OzProb *dop;
    int32_t *dt, *dex;
    OzTile *dtl;
    int8_t *dsl;
    CK(cudaMalloc(&dop, sizeof op));
    CK(cudaMalloc(&dt, tasks.size() * 4));
    CK(cudaMalloc(&dtl, tiles.size() * sizeof(OzTile)));
    CK(cudaMalloc(&dsl, (size_t)S * op.Mpad * op.Kpad));
    CK(cudaMalloc(&dex, (size_t)op.Mpad * 4));
    CK(cudaMemcpy(dop, &op, sizeof op, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dt, tasks.data(), tasks.size() * 4, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dtl, tiles.data(), tiles.size() * sizeof(OzTile), cudaMemcpyHostToDevice));
    cudaEvent_t e0, e1, e2;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaEventCreate(&e2);
    float best = 1e30f, bsplit = 0;
    for (int r = 0; r < reps; r++) {
        CK(cudaMemcpy(dU, C0, cbytes, cudaMemcpyDeviceToDevice));
        cudaEventRecord(e0);
        launch_oz<S>(dL, dU, dprob, dop, dt, (int64_t)tasks.size() / 3, nullptr, 0, dsl, dex, op.Mpad, 0);
        cudaEventRecord(e1);
        launch_oz<S>(dL, dU, dprob, dop, nullptr, 0, dtl, (int64_t)tiles.size(), dsl, dex, 0, 0, UpdGather{}, wide);
        cudaEventRecord(e2);
        CK(cudaEventSynchronize(e2));
        CK(cudaGetLastError());
        float t1, t2;
        cudaEventElapsedTime(&t1, e0, e1);
        cudaEventElapsedTime(&t2, e0, e2);
        if (t2 < best) best = t2, bsplit = t1;
    }
    printf("  ozaki S=%d %s: %zu tiles, split %.3f ms, total %.3f ms\n", S, wide ? "128x128" : "128x64", tiles.size(),
           bsplit, best);
    cudaFree(dop); cudaFree(dt); cudaFree(dtl); cudaFree(dsl); cudaFree(dex);
    return best;
}

int main(int argc, char **argv) {
    int M = argc > 1 ? atoi(argv[1]) : 8192, N = argc > 2 ? atoi(argv[2]) : 8192, K = argc > 3 ? atoi(argv[3]) : 4096;
    const int lda = M + (M & 1);
    std::mt19937_64 rng(7);
    std::normal_distribution<double> nd(0.0, 1.0);
    std::uniform_int_distribution<int> ex(-30, 0);
    std::vector<double> A((size_t)lda * K), C((size_t)M * M, 0.0);
    // rows of mixed magnitudes (like factor panels): per-entry exponents down to 2^-30
    for (int p = 0; p < K; p++)
        for (int i = 0; i < M; i++) A[i + (size_t)p * lda] = std::ldexp(nd(rng), ex(rng));
    for (int j = 0; j < N; j++)
        for (int i = j; i < M; i++) C[i + (size_t)j * M] = nd(rng);
    double *dL, *dU, *dC0;
    const size_t cbytes = (size_t)M * M * 8;
    CK(cudaMalloc(&dL, ((size_t)lda * K + 64) * 8));
    CK(cudaMalloc(&dU, cbytes));
    CK(cudaMalloc(&dC0, cbytes));
    CK(cudaMemcpy(dL, A.data(), (size_t)lda * K * 8, cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dC0, C.data(), cbytes, cudaMemcpyHostToDevice));
    GemmProb g{0, 0, lda, M, M, N, K, 1};
    GemmProb *dprob;
    CK(cudaMalloc(&dprob, sizeof g));
    CK(cudaMemcpy(dprob, &g, sizeof g, cudaMemcpyHostToDevice));
    const double flops = 2.0 * K * ((double)N * (N + 1) / 2 + (double)(M - N) * N);
    printf("SYRK M=%d N=%d K=%d (%.3e flops)\n", M, N, K, flops);

    // sampled reference entries (long double)
    std::uniform_int_distribution<int> ri(0, M - 1);
    std::vector<int> si, sj;
    for (int q = 0; q < 3000; q++) {
        int i = ri(rng), j = ri(rng) % N;
        if (i < j) std::swap(i, j);
        if (j >= N) continue;
        si.push_back(i);
        sj.push_back(j);
    }
    std::vector<long double> ref(si.size());
    std::vector<double> mag(si.size());
    for (size_t q = 0; q < si.size(); q++) {
        long double s = C[si[q] + (size_t)sj[q] * M];
        double m = 0;
        for (int p = 0; p < K; p++) {
            const double a = A[si[q] + (size_t)p * lda], b = A[sj[q] + (size_t)p * lda];
            s -= (long double)a * b;
            m += std::fabs(a * b);
        }
        ref[q] = s;
        mag[q] = m;
    }
    std::vector<double> out((size_t)M * M);
    auto check = [&](const char *name) {
        CK(cudaMemcpy(out.data(), dU, cbytes, cudaMemcpyDeviceToHost));
        double worst = 0, mean = 0;
        for (size_t q = 0; q < si.size(); q++) {
            const double e = std::fabs((double)((long double)out[si[q] + (size_t)sj[q] * M] - ref[q])) /
                             (mag[q] * std::ldexp(1.0, -53));
            worst = std::fmax(worst, e);
            mean += e;
        }
        printf("  %-10s error / (u sum|a b|): max %.3f mean %.4f\n", name, worst, mean / si.size());
    };
    // DMMA reference path
    std::vector<TileTask> tiles;
    for (int tj = 0; tj < (N + 63) / 64; tj++)
        for (int ti = 0; ti < (M + 63) / 64; ti++)
            if ((ti + 1) * 64 > tj * 64) tiles.push_back({0, (ti << 16) | tj});
    TileTask *dtt;
    CK(cudaMalloc(&dtt, tiles.size() * sizeof(TileTask)));
    CK(cudaMemcpy(dtt, tiles.data(), tiles.size() * sizeof(TileTask), cudaMemcpyHostToDevice));
    cudaFuncSetAttribute(k_update_t<Big, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Big::SMEM);
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float bd = 1e30f;
    for (int r = 0; r < 4; r++) {
        CK(cudaMemcpy(dU, dC0, cbytes, cudaMemcpyDeviceToDevice));
        cudaEventRecord(e0);
        k_update_t<Big, true><<<(unsigned)tiles.size(), Big::NT, Big::SMEM>>>(dL, dU, dprob, dtt, UpdGather{});
        cudaEventRecord(e1);
        CK(cudaEventSynchronize(e1));
        float t;
        cudaEventElapsedTime(&t, e0, e1);
        bd = std::fmin(bd, t);
    }
    printf("  dmma fp64: %.3f ms = %.2f TF/s\n", bd, flops / bd / 1e9);
    check("dmma");
    float t8 = run_oz<8>(dL, dU, dprob, M, N, K, 4, dC0, cbytes);
    printf("  -> %.2f TF/s fp64-equivalent, %.2fx dmma\n", flops / t8 / 1e9, bd / t8);
    check("ozaki8");
    float t8w = run_oz<8>(dL, dU, dprob, M, N, K, 4, dC0, cbytes, 1);
    printf("  -> %.2f TF/s fp64-equivalent, %.2fx dmma\n", flops / t8w / 1e9, bd / t8w);
    check("ozaki8w");
    float t4w = run_oz<4>(dL, dU, dprob, M, N, K, 4, dC0, cbytes, 1);
    printf("  -> %.2f TF/s fp64-equivalent, %.2fx dmma\n", flops / t4w / 1e9, bd / t4w);
    check("ozaki4w");
    float t7 = run_oz<7>(dL, dU, dprob, M, N, K, 4, dC0, cbytes);
    printf("  -> %.2f TF/s fp64-equivalent, %.2fx dmma\n", flops / t7 / 1e9, bd / t7);
    check("ozaki7");
    float t4 = run_oz<4>(dL, dU, dprob, M, N, K, 4, dC0, cbytes);
    printf("  -> %.2f TF/s fp64-equivalent, %.2fx dmma\n", flops / t4 / 1e9, bd / t4);
    check("ozaki4");
    return 0;
}
