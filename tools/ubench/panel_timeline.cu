// Phase timeline of the dataflow panel kernel (k_panel) on one dense front (f rows,
// k pivot columns, nbk blocks at j0 = 0): %globaltimer stamps per task (PANEL_TL in
// kernels.cu), printed for the band tasks; plus the launch time (CUDA events).
//   nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a \
//        -I include -I paper_conf_ipps_georgesgsc11_b200/csrc tools/ubench/panel_timeline.cu -o tools/ubench/panel_timeline
#define MF_PANEL_TL 1
#include "../../paper_conf_ipps_georgesgsc11_b200/csrc/kernels.cu"

#include <cstdlib>
#include <vector>
#include <cstring>

using namespace mf;

int main(int argc, char **argv) {
    const int f = argc > 1 ? atoi(argv[1]) : 8192, k = argc > 2 ? atoi(argv[2]) : 8192;
    const int nbk = argc > 3 ? atoi(argv[3]) : 4;
    const int ld = f + (f & 1);
    std::vector<double> h((size_t)ld * k, 0.0);
    srand(1);
    for (int j = 0; j < k; j++)
        for (int i = j; i < f; i++) h[i + (size_t)j * ld] = (i == j) ? 4.0 * f : (rand() / (double)RAND_MAX - 0.5);
    double *L, *L0;
    cudaMalloc(&L, (h.size() + 2) * 8);
    cudaMalloc(&L0, (h.size() + 2) * 8);
    cudaMemcpy(L0, h.data(), h.size() * 8, cudaMemcpyHostToDevice);
    int32_t hs[4] = {0, k, f, ld};
    int64_t hoff = 0;
    int32_t *dfirst, *dk, *df, *dld;
    int64_t *doff;
    cudaMalloc(&dfirst, 4); cudaMemcpy(dfirst, &hs[0], 4, cudaMemcpyHostToDevice);
    cudaMalloc(&dk, 4); cudaMemcpy(dk, &hs[1], 4, cudaMemcpyHostToDevice);
    cudaMalloc(&df, 4); cudaMemcpy(df, &hs[2], 4, cudaMemcpyHostToDevice);
    cudaMalloc(&dld, 4); cudaMemcpy(dld, &hs[3], 4, cudaMemcpyHostToDevice);
    cudaMalloc(&doff, 8); cudaMemcpy(doff, &hoff, 8, cudaMemcpyHostToDevice);
    int *failed; cudaMalloc(&failed, 16);
    int hf[4] = {INT_MAX, 1, 0, 0};
    cudaMemcpy(failed, hf, 16, cudaMemcpyHostToDevice);
    unsigned *pflag; cudaMalloc(&pflag, kPanelFlags * 4);
    unsigned *tk; cudaMalloc(&tk, 8); cudaMemset(tk, 0, 8);
    DevPlan d{};
    d.L = L; d.sn_first = dfirst; d.sn_k = dk; d.sn_f = df; d.sn_ld = dld; d.L_off = doff;
    d.failed = failed; d.epoch = reinterpret_cast<const unsigned *>(failed + 1); d.panel_flag = pflag;
    const int nch = (f + 63) / 64;
    std::vector<int32_t> tasks;
    for (int c = 0; c < nch; c++) { tasks.push_back(0); tasks.push_back(c); }
    int32_t *dt; cudaMalloc(&dt, tasks.size() * 4);
    cudaMemcpy(dt, tasks.data(), tasks.size() * 4, cudaMemcpyHostToDevice);
    cudaFuncSetAttribute(k_panel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kPanelSmem);
    unsigned long long *tl; cudaMalloc(&tl, (size_t)nch * 64 * 8);
    cudaMemcpyToSymbol(g_panel_tl, &tl, sizeof(tl));
    cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
    float best = 1e9;
    for (int rep = 0; rep < 10; rep++) {
        cudaMemcpy(L, L0, h.size() * 8, cudaMemcpyDeviceToDevice);
        cudaMemset(pflag, 0, kPanelFlags * 4);
        cudaMemset(tl, 0, (size_t)nch * 64 * 8);
        cudaEventRecord(e0);
        launch_panel(d, dt, nch, 0, nbk, tk, 0);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms; cudaEventElapsedTime(&ms, e0, e1);
        if (ms < best) best = ms;
    }
    cudaError_t err = cudaGetLastError();
    {
        std::vector<unsigned long long> t((size_t)nch * 64);
        cudaMemcpy(t.data(), tl, t.size() * 8, cudaMemcpyDeviceToHost);
        unsigned long long t0 = ~0ull, tend = 0;
        for (auto v : t) if (v) { t0 = std::min(t0, v); tend = std::max(tend, v); }
        auto r = [&](int task, int ev) { unsigned long long v = t[(size_t)task * 64 + ev]; return v ? (double)(v - t0) * 1e-3 : -1.0; };
        printf("last rep: first stamp -> last stamp %.2f us\n", (tend - t0) * 1e-3);
        for (int c = 0; c < std::min(nbk, nch); c++) {
            printf("band %d:", c);
            for (int b = 0; b < c; b++)
                printf(" [b%d start %.1f gemm %.1f Lbb %.1f trsm %.1f store %.1f pub %.1f]", b, r(c, 6 * b), r(c, 6 * b + 1),
                       r(c, 6 * b + 2), r(c, 6 * b + 3), r(c, 6 * b + 4), r(c, 6 * b + 5));
            printf(" potrf %.1f -> %.1f pub %.1f\n", r(c, 60), r(c, 61), r(c, 62));
            if (c == 0 || c == 3) {   // potrf steps: after the row solve / after the update + next pivot block
                printf("   potrf steps:");
                for (int st = 0; st < 8; st++) printf(" %.2f", r(c, 44 + 2 * st) - r(c, 60));
                printf("\n");
            }
        }
        for (int c : {nbk, nbk + 1, nch / 2, nch - 1}) {
            if (c >= nch) continue;
            printf("row %d:", c);
            for (int b = 0; b < nbk; b++) printf(" [b%d %.1f g %.1f w %.1f t %.1f]", b, r(c, 6 * b), r(c, 6 * b + 1), r(c, 6 * b + 2), r(c, 6 * b + 3));
            printf("\n");
        }
    }
    printf("f=%d k=%d nbk=%d tasks=%d: best %.2f us (%s)\n", f, k, nbk, nch, best * 1e3, cudaGetErrorString(err));
    // check: the leading W x W block of L L^T reproduces A (W = 64 nbk), and the rows
    // below: (L L^T)(i, j) = A(i, j) for j < W
    std::vector<double> Lh(h.size());
    cudaMemcpy(Lh.data(), L, h.size() * 8, cudaMemcpyDeviceToHost);
    const int W = std::min(64 * nbk, k);
    double maxerr = 0;
    for (int j = 0; j < W; j++)
        for (int i = j; i < f; i += (i < W ? 1 : 37)) {
            double sum = 0;
            for (int p = 0; p <= j; p++) sum += Lh[i + (size_t)p * ld] * Lh[j + (size_t)p * ld];
            maxerr = std::max(maxerr, fabs(sum - h[i + (size_t)j * ld]) / (4.0 * f));
        }
    printf("max |L L^T - A| / |A|_max over the panel columns: %.3e\n", maxerr);
    unsigned long long hsh = 1469598103934665603ull;   // FNV-1a of the panel columns' bits (bitwise A/B)
    for (int j = 0; j < W; j++)
        for (int i = j; i < f; i++) {
            unsigned long long b;
            memcpy(&b, &Lh[i + (size_t)j * ld], 8);
            hsh = (hsh ^ b) * 1099511628211ull;
        }
    printf("panel hash %016llx\n", hsh);
    return 0;
}
