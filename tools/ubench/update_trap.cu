// Reproducer for the trailing-update shape: A and C in the same panel
// (A = columns [0, K) rows K.., C = columns [K, K+N) rows K..), several
// fronts per launch; bulk (VAR 1) vs cp.async (VAR 0), bitwise, repeated.
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>
#include "dmma_update.cuh"
using namespace mf;
#define CK(x) do { cudaError_t e_ = (x); if (e_ != cudaSuccess) { printf("CUDA %s @%d\n", cudaGetErrorString(e_), __LINE__); exit(1); } } while (0)

int main(int argc, char **argv) {
    setvbuf(stdout, nullptr, _IONBF, 0);
    const int nf = argc > 1 ? atoi(argv[1]) : 8;        // fronts
    const int f0 = argc > 2 ? atoi(argv[2]) : 4000;     // front order
    const int K = argc > 3 ? atoi(argv[3]) : 512;       // inner dimension (A columns)
    const int N = argc > 4 ? atoi(argv[4]) : 512;       // C columns
    const int reps = argc > 5 ? atoi(argv[5]) : 10;
    const int VARB = argc > 6 ? atoi(argv[6]) : 1;
    using Cfg = UpdCfg<64, 64, 16, 3, 2, 2, 4>;
    std::vector<GemmProb> probs;
    std::vector<TileTask> tiles;
    std::vector<int64_t> off;
    if (nf > 32) { printf("nf <= 32\n"); return 1; }
    int64_t tot = 0;
    for (int q = 0; q < nf; q++) {
        int f = f0 - 37 * q; f += f & 1;       // vary the order, keep ld even
        const int ld = f;
        off.push_back(tot);
        GemmProb g{};
        g.a_off = tot + K;                      // column 0, row K
        g.c_off = tot + (int64_t)K * ld + K;    // column K, row K
        g.lda = g.ldc = ld;
        g.M = f - K; g.N = N; g.K = K; g.flags = 0;
        const int pid = (int)probs.size();
        probs.push_back(g);
        for (int tj = 0; tj * 64 < g.N; tj++)
            for (int ti = tj; ti * 64 < g.M; ti++) tiles.push_back({pid, (ti << 16) | tj});
        tot += (int64_t)ld * (K + N);
    }
    tot += 128;
    std::vector<double> h(tot);
    srand(7);
    for (auto &x : h) x = (double)(rand() % 9 - 4);
    double *L0, *L1, *U;
    CK(cudaMalloc(&L0, tot * 8)); CK(cudaMalloc(&L1, tot * 8)); CK(cudaMalloc(&U, 64));
    GemmProb *dp; TileTask *dt;
    CK(cudaMalloc(&dp, probs.size() * sizeof(GemmProb)));
    CK(cudaMalloc(&dt, tiles.size() * sizeof(TileTask)));
    CK(cudaMemcpy(dp, probs.data(), probs.size() * sizeof(GemmProb), cudaMemcpyHostToDevice));
    CK(cudaMemcpy(dt, tiles.data(), tiles.size() * sizeof(TileTask), cudaMemcpyHostToDevice));
    std::vector<double> r0(tot), r1(tot);
    int bad = 0;
    for (int r = 0; r < reps; r++) {
        CK(cudaMemcpy(L0, h.data(), tot * 8, cudaMemcpyHostToDevice));
        CK(cudaMemcpy(L1, h.data(), tot * 8, cudaMemcpyHostToDevice));
        launch_update_t<Cfg, 0>(L0, U, dp, dt, (int64_t)tiles.size(), 0);
        if (VARB == 3) launch_update_t<Cfg, 3>(L1, U, dp, dt, (int64_t)tiles.size(), 0);
        else launch_update_t<Cfg, 1>(L1, U, dp, dt, (int64_t)tiles.size(), 0);
        CK(cudaDeviceSynchronize());
        CK(cudaMemcpy(r0.data(), L0, tot * 8, cudaMemcpyDeviceToHost));
        CK(cudaMemcpy(r1.data(), L1, tot * 8, cudaMemcpyDeviceToHost));
        int64_t nd = 0, first = -1;
        for (int64_t i = 0; i < tot; i++)
            if (r0[i] != r1[i]) { if (first < 0) first = i; nd++; }
        if (nd) {
            bad++;
            // every differing word: front, tile, local (row, col)
            int shown = 0;
            for (int64_t x = 0; x < tot && shown < 40; x++) {
                if (r0[x] == r1[x]) continue;
                int qq = 0;
                while (qq + 1 < nf && off[qq + 1] <= x) qq++;
                const int ldq = probs[qq].lda;
                const int cc = (int)((x - off[qq]) / ldq) - K, rr = (int)((x - off[qq]) % ldq) - K;
                printf("   q%d t(%d,%d) l(%d,%d) d=%g\n", qq, rr / 64, cc / 64, rr % 64, cc % 64, r1[x] - r0[x]);
                shown++;
            }
            int q = 0;
            while (q + 1 < nf && off[q + 1] <= first) q++;
            const int ld = probs[q].lda;
            const int64_t w = first - off[q];
            const int col = (int)(w / ld), row = (int)(w % ld);
            double ref = h[first];   // C(row, col) - sum_p A(row, p) A(col, p)
            for (int p = 0; p < K; p++) ref -= h[off[q] + (int64_t)p * ld + row] * h[off[q] + (int64_t)p * ld + col];
            printf("rep %d: %lld words differ; first: front %d col %d row %d (i %d j %d) cp.async %g bulk %g ref %g\n", r,
                   (long long)nd, q, col, row, row - K, col - K, r0[first], r1[first], ref);
        }
    }
    printf("nf=%d f0=%d K=%d N=%d tiles=%zu: %d of %d reps differ\n", nf, f0, K, N, tiles.size(), bad, reps);
    return 0;
}
