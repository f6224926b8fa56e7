// kernels.cu -- sm_100a kernels of the multifrontal factor-update hot path.
//
// What each kernel computes follows PAPER.md L27 (Sec. II-A) and Fig. 1
// (L33-65): per supernode, F^n = A entries (+) extend-add of the children's
// U^c, then potrf on L1 (k x k), trsm on L2 (m x k), U^n = U^n - L2 L2^T.
// The large-front path is the blocked variant of PAPER.md L325 / Fig. 9
// (w x w potrf kernel, trsm on the panel below it, trailing update), with the
// syrk on U^n done once with inner dimension k.  All arithmetic is fp64
// (reading C7).  FP64 tensor-core work uses DMMA (mma.sync m8n8k4 f64): on
// sm_100a tcgen05 has no f64 kind (probe 1).
//
// Determinism: extend-add has no atomics; every destination entry receives
// 0, then its A value, then the children's contributions in ascending child
// order (reading C6) -- the same summation order as the oracle.
#include <climits>
#include <cstdio>

#include "dmma_update.cuh"
#include "kernels.cuh"

namespace mf {

// ------------------------------------------------------------------ helpers
__device__ __forceinline__ double sum_values(const DevPlan &d, const double *__restrict__ values, int64_t e) {
    const int64_t b = d.bvptr[e], q = d.bvptr[e + 1];
    double v = values[d.bvidx[b]];
    for (int64_t t = b + 1; t < q; t++) v += values[d.bvidx[t]];
    return v;
}

__device__ __forceinline__ void note_pivot(const DevPlan &d, double djj, int col) {
    if (!(djj > 0.0)) atomicMin(d.failed, col);   // non-positive or NaN pivot (reading C8)
}

__global__ void k_init_failed(int *failed) { *failed = INT_MAX; }

// ============================================================ small fronts
// One CTA per front; the whole f x f front lives in shared memory (column-major,
// leading dimension f).  Assembly, potrf, trsm and the syrk on U^n are fused:
// the k pivot columns are eliminated right-looking, which produces L1, L2 and
// U^n = F22 - L2 L2^T in place.  Writes the L panel and U^n to HBM.
template <int NT>
__global__ void __launch_bounds__(NT) k_small_front(DevPlan d, const int32_t *__restrict__ list,
                                                    const double *__restrict__ values) {
    extern __shared__ double F[];
    const int s = list[blockIdx.x];
    const int k = d.sn_k[s], f = d.sn_f[s], m = f - k, first = d.sn_first[s];
    const int tid = threadIdx.x;
    for (int i = tid; i < f * f; i += NT) F[i] = 0.0;
    __syncthreads();
    // A entries of the k pivot columns: warp per column, lanes over entries
    {
        const int warp = tid >> 5, lane = tid & 31;
        for (int j = warp; j < k; j += NT / 32) {
            const int64_t e0 = d.bcolptr[first + j], e1 = d.bcolptr[first + j + 1];
            for (int64_t e = e0 + lane; e < e1; e += 32) F[d.blrow[e] + j * f] = sum_values(d, values, e);
        }
    }
    __syncthreads();
    // extend-add of the children's U^c, ascending child order
    for (int q = d.child_ptr[s]; q < d.child_ptr[s + 1]; q++) {
        const int c = d.child_list[q];
        const int mc = d.sn_f[c] - d.sn_k[c];
        const int32_t *__restrict__ rel = d.relmap + d.relmap_ptr[c];
        const double *__restrict__ Uc = d.U + d.U_off[c];
        for (int idx = tid; idx < mc * mc; idx += NT) {
            const int p = idx % mc, qq = idx / mc;
            if (p >= qq) F[rel[p] + rel[qq] * f] += Uc[idx];
        }
        __syncthreads();
    }
    // right-looking elimination of the k pivot columns over the whole front
    for (int j = 0; j < k; j++) {
        const double djj = F[j + j * f];
        const double piv = sqrt(djj);
        for (int i = j + 1 + tid; i < f; i += NT) F[i + j * f] /= piv;
        __syncthreads();
        if (tid == 0) {
            note_pivot(d, djj, first + j);
            F[j + j * f] = piv;
        }
        const int nr = f - j - 1;
        for (int idx = tid; idx < nr * nr; idx += NT) {
            const int i = j + 1 + idx % nr, c = j + 1 + idx / nr;
            if (i >= c) F[i + c * f] -= F[i + j * f] * F[c + j * f];
        }
        __syncthreads();
    }
    // write the L panel (upper triangle of L1 = 0) and U^n (lower triangle)
    double *__restrict__ P = d.L + d.L_off[s];
    const int ld = d.sn_ld[s];
    for (int idx = tid; idx < f * k; idx += NT) {
        const int i = idx % f, j = idx / f;
        P[i + (int64_t)j * ld] = i >= j ? F[i + j * f] : 0.0;
    }
    if (m > 0) {
        double *__restrict__ Us = d.U + d.U_off[s];
        for (int idx = tid; idx < m * m; idx += NT) {
            const int i = idx % m, c = idx / m;
            if (i >= c) Us[idx] = F[(k + i) + (k + c) * f];
        }
    }
}

int small_front_smem_ok(int fmax) { return (size_t)fmax * fmax * sizeof(double) <= 227 * 1024; }

void launch_small_fronts(const DevPlan &d, const int32_t *list, int count, int fmax, const double *values,
                         cudaStream_t st) {
    if (count <= 0) return;
    const size_t smem = (size_t)fmax * fmax * sizeof(double);
    if (fmax <= 32) {
        k_small_front<64><<<count, 64, smem, st>>>(d, list, values);
    } else if (fmax <= 64) {
        k_small_front<128><<<count, 128, smem, st>>>(d, list, values);
    } else {
        static bool attr = false;
        if (!attr) {
            cudaFuncSetAttribute(k_small_front<256>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
            attr = true;
        }
        k_small_front<256><<<count, 256, smem, st>>>(d, list, values);
    }
}

// ============================================================ large-front assembly
// Task = (front s, first local column c0): zero columns [c0, c0+32) of the
// front, write the A entries, then extend-add every child's U^c columns that
// map into these columns (child order ascending, barrier between children, so
// the summation order is fixed).  Columns < k live in the L panel, columns >= k
// in U^s.
constexpr int kAsmThreads = 256;
__global__ void __launch_bounds__(kAsmThreads) k_assemble(DevPlan d, const int32_t *__restrict__ tasks,
                                                          const double *__restrict__ values) {
    const int s = tasks[2 * blockIdx.x], c0 = tasks[2 * blockIdx.x + 1];
    const int k = d.sn_k[s], f = d.sn_f[s], m = f - k, ld = d.sn_ld[s], first = d.sn_first[s];
    const int c1 = min(c0 + kAsmCols, f);
    double *__restrict__ P = d.L + d.L_off[s];
    double *__restrict__ Us = d.U + d.U_off[s];
    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    constexpr int NW = kAsmThreads / 32;
    for (int c = c0 + warp; c < c1; c += NW) {
        if (c < k) {
            for (int i = lane; i < f; i += 32) P[i + (int64_t)c * ld] = 0.0;
        } else {
            const int cu = c - k;
            for (int i = cu + lane; i < m; i += 32) Us[i + (int64_t)cu * m] = 0.0;
        }
    }
    __syncthreads();
    for (int c = c0 + warp; c < min(c1, k); c += NW) {
        const int64_t e0 = d.bcolptr[first + c], e1 = d.bcolptr[first + c + 1];
        for (int64_t e = e0 + lane; e < e1; e += 32) P[d.blrow[e] + (int64_t)c * ld] = sum_values(d, values, e);
    }
    __syncthreads();
    __shared__ int qrange[2];
    for (int q = d.child_ptr[s]; q < d.child_ptr[s + 1]; q++) {
        const int ch = d.child_list[q];
        const int mc = d.sn_f[ch] - d.sn_k[ch];
        const int32_t *__restrict__ rel = d.relmap + d.relmap_ptr[ch];
        const double *__restrict__ Uc = d.U + d.U_off[ch];
        if (tid < 2) {   // child columns qa..qb-1 map into [c0, c1): rel is increasing
            const int target = tid == 0 ? c0 : c1;
            int lo = 0, hi = mc;
            while (lo < hi) {
                const int mid = (lo + hi) >> 1;
                if (rel[mid] < target) lo = mid + 1; else hi = mid;
            }
            qrange[tid] = lo;
        }
        __syncthreads();
        const int qa = qrange[0], qb = qrange[1];
        for (int qc = qa + warp; qc < qb; qc += NW) {
            const int dc = rel[qc];
            const double *__restrict__ ucol = Uc + (int64_t)qc * mc;
            if (dc < k) {
                double *__restrict__ pcol = P + (int64_t)dc * ld;
                for (int p = qc + lane; p < mc; p += 32) pcol[rel[p]] += ucol[p];
            } else {
                double *__restrict__ ucol_dst = Us + (int64_t)(dc - k) * m - k;
                for (int p = qc + lane; p < mc; p += 32) ucol_dst[rel[p]] += ucol[p];
            }
        }
        __syncthreads();
    }
}

void launch_assemble(const DevPlan &d, const int32_t *tasks, int64_t count, const double *values, cudaStream_t st) {
    if (count <= 0) return;
    k_assemble<<<(unsigned)count, kAsmThreads, 0, st>>>(d, tasks, values);
}

// ============================================================ diagonal-block potrf
// The "light-weight GPU kernel ... performing potrf on a w x w matrix" of
// one CTA per active front factors its diagonal block
// [j0, j0+we) x [j0, j0+we) in shared memory (right-looking, unblocked).
constexpr int kWmax = 64;
constexpr int kPotrfThreads = 256;   // 4 threads per row of the 64 x 64 block
__global__ void __launch_bounds__(kPotrfThreads) k_potrf_diag(DevPlan d, const int32_t *__restrict__ fronts,
                                                              int j0, int w) {
    constexpr int LDA = kWmax + 1;        // row-major, odd stride: conflict-free row-per-thread access
    __shared__ double A[kWmax * LDA];
    __shared__ double sh_inv;
    const int s = fronts[blockIdx.x];
    const int k = d.sn_k[s], ld = d.sn_ld[s], first = d.sn_first[s];
    const int we = min(w, k - j0);
    double *__restrict__ P = d.L + d.L_off[s] + (int64_t)j0 * ld + j0;
    const int tid = threadIdx.x, i = tid >> 2, h = tid & 3;
    for (int c = tid >> 6; c < we; c += kPotrfThreads / 64) {
        const int r = tid & 63;
        if (r < we) A[r * LDA + c] = P[r + (int64_t)c * ld];
    }
    __syncthreads();
    for (int j = 0; j < we; j++) {
        // phase 1: the thread that last updated A[j][j] takes the pivot
        if (i == j && h == 0) {
            const double djj = A[j * LDA + j];
            const double piv = sqrt(djj);
            note_pivot(d, djj, first + j0 + j);
            A[j * LDA + j] = piv;
            sh_inv = 1.0 / piv;
        }
        __syncthreads();
        // phase 2: scale column j
        if (h == 0 && i > j && i < we) A[i * LDA + j] *= sh_inv;
        __syncthreads();
        // phase 3: rank-1 update of row i, columns (j, i]; A[c][j] is final for c <= i
        if (i > j && i < we) {
            const double l = A[i * LDA + j];
            for (int c = j + 1 + h; c <= i; c += 4) A[i * LDA + c] -= l * A[c * LDA + j];
        }
    }
    __syncthreads();
    for (int c = tid >> 6; c < we; c += kPotrfThreads / 64) {
        const int r = tid & 63;
        if (r < we && r >= c) P[r + (int64_t)c * ld] = A[r * LDA + c];
    }
}

void launch_potrf_diag(const DevPlan &d, const int32_t *fronts, int count, int j0, int w, cudaStream_t st) {
    if (count <= 0) return;
    k_potrf_diag<<<count, kPotrfThreads, 0, st>>>(d, fronts, j0, w);
}

// ============================================================ panel trsm
// X L11^T = B for the rows [r0, r0+64) below the diagonal block (these rows
// span the rest of L1 and all of L2: "we perform trsm on a (m + k - w) x w
// matrix which spans both L1 and L2").  Substitution order
// (ascending columns), no explicit inverse: integer-exact on manufactured inputs.
constexpr int kTrsmThreads = kTrsmRows;   // one thread per row
__global__ void __launch_bounds__(kTrsmThreads, 2) k_trsm_panel(DevPlan d, const int32_t *__restrict__ tasks,
                                                                int j0, int w) {
    __shared__ __align__(16) double Ls[kWmax * kWmax];   // column-major L11 (padded with identity)
    __shared__ double inv[kWmax];
    const int s = tasks[2 * blockIdx.x], r0 = tasks[2 * blockIdx.x + 1];
    const int k = d.sn_k[s], f = d.sn_f[s], ld = d.sn_ld[s];
    const int we = min(w, k - j0);
    const double *__restrict__ D = d.L + d.L_off[s] + (int64_t)j0 * ld + j0;
    double *__restrict__ B = d.L + d.L_off[s] + (int64_t)j0 * ld + r0;
    const int tid = threadIdx.x;
    for (int idx = tid; idx < kWmax * kWmax; idx += kTrsmThreads) {
        const int i = idx & (kWmax - 1), c = idx / kWmax;
        double v = (i == c) ? 1.0 : 0.0;
        if (i < we && c < we && i >= c) v = D[i + (int64_t)c * ld];
        Ls[idx] = v;
    }
    __syncthreads();
    if (tid < kWmax) inv[tid] = 1.0 / Ls[tid * kWmax + tid];
    const bool row_ok = tid < f - r0;
    double x[kWmax];
#pragma unroll
    for (int c = 0; c < kWmax; c++) x[c] = (row_ok && c < we) ? B[tid + (int64_t)c * ld] : 0.0;
    __syncthreads();
    // x L11^T = b by substitution, ascending columns (no explicit inverse of L11):
    // x_c = (b_c - sum_{p<c} x_p L_cp) / L_cc, the sum accumulated in ascending p
#pragma unroll
    for (int c = 0; c < kWmax; c++) {
        const double *Lr = Ls + c;                 // row c of L11: Ls[c + p * kWmax]
        double acc = x[c];
#pragma unroll
        for (int p = 0; p < c; p++) acc -= x[p] * Lr[p * kWmax];
        x[c] = acc * inv[c];
    }
    if (row_ok) {
#pragma unroll
        for (int c = 0; c < kWmax; c++)
            if (c < we) B[tid + (int64_t)c * ld] = x[c];
    }
}

void launch_trsm_panel(const DevPlan &d, const int32_t *tasks, int64_t count, int j0, int w, cudaStream_t st) {
    if (count <= 0) return;
    k_trsm_panel<<<(unsigned)count, kTrsmThreads, 0, st>>>(d, tasks, j0, w);
}

// ============================================================ DMMA Schur update
// The production tile shape (kTileM x kTileN in mf_plan.h); variants are
// benchmarked in tools/ubench/update_variants.cu.
using UpdProd = UpdCfg<kTileM, kTileN, 16, 3, 2, 2, 4>;   // 29.3 TF/s on M=N=8192,K=4096 (ubench)

void launch_update(const DevPlan &d, const GemmProb *probs, const TileTask *tiles, int64_t ntiles, cudaStream_t st) {
    launch_update_t<UpdProd>(d.L, d.U, probs, tiles, ntiles, st);
}

void launch_init_failed(int *failed, cudaStream_t st) { k_init_failed<<<1, 1, 0, st>>>(failed); }

// diag(L) in final labels (one warp per supernode)
__global__ void k_export_diag(DevPlan d, int nsuper, double *__restrict__ out) {
    const int s = blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5);
    if (s >= nsuper) return;
    const int k = d.sn_k[s], ld = d.sn_ld[s], first = d.sn_first[s];
    const double *__restrict__ P = d.L + d.L_off[s];
    for (int j = threadIdx.x & 31; j < k; j += 32) out[first + j] = P[j + (int64_t)j * ld];
}
void launch_export_diag(const DevPlan &d, int nsuper, double *out, cudaStream_t st) {
    if (nsuper > 0) k_export_diag<<<(nsuper + 7) / 8, 256, 0, st>>>(d, nsuper, out);
}

// ============================================================ triangular solves
// "a forward triangular solve Ly = b and a backward triangular
// solve L^T x = y".  Supernodal, level by level; the forward sweep carries
// per-front update vectors that the parent gathers through the same relative
// maps as the extend-add (deterministic, no atomics).
__global__ void k_permute_in(const int32_t *__restrict__ perm, const double *__restrict__ b, double *__restrict__ y,
                             int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        y[i] = b[perm[i]];
}
__global__ void k_permute_out(const int32_t *__restrict__ perm, const double *__restrict__ xf, double *__restrict__ x,
                              int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        x[perm[i]] = xf[i];
}
void launch_permute_in(const DevPlan &d, const double *b, double *y, int64_t n, cudaStream_t st) {
    if (n > 0) k_permute_in<<<(unsigned)((n + 255) / 256 < 4096 ? (n + 255) / 256 : 4096), 256, 0, st>>>(d.perm, b, y, n);
}
void launch_permute_out(const DevPlan &d, const double *xf, double *x, int64_t n, cudaStream_t st) {
    if (n > 0) k_permute_out<<<(unsigned)((n + 255) / 256 < 4096 ? (n + 255) / 256 : 4096), 256, 0, st>>>(d.perm, xf, x, n);
}

constexpr int kSolveThreads = 256;
__global__ void __launch_bounds__(kSolveThreads) k_fwd_solve(DevPlan d, const int32_t *__restrict__ list,
                                                             double *__restrict__ y) {
    const int s = list[blockIdx.x];
    const int k = d.sn_k[s], f = d.sn_f[s], ld = d.sn_ld[s], first = d.sn_first[s];
    double *__restrict__ v = d.fv + d.fv_off[s];
    const double *__restrict__ P = d.L + d.L_off[s];
    const int tid = threadIdx.x;
    for (int i = tid; i < f; i += kSolveThreads) v[i] = i < k ? y[first + i] : 0.0;
    __syncthreads();
    for (int q = d.child_ptr[s]; q < d.child_ptr[s + 1]; q++) {
        const int c = d.child_list[q];
        const int kc = d.sn_k[c], mc = d.sn_f[c] - kc;
        const int32_t *__restrict__ rel = d.relmap + d.relmap_ptr[c];
        const double *__restrict__ vc = d.fv + d.fv_off[c] + kc;
        for (int p = tid; p < mc; p += kSolveThreads) v[rel[p]] += vc[p];
        __syncthreads();
    }
    for (int j = 0; j < k; j++) {
        const double xj = v[j] / P[j + (int64_t)j * ld];
        if (tid == 0) y[first + j] = xj;
        const double *__restrict__ col = P + (int64_t)j * ld;
        for (int i = j + 1 + tid; i < f; i += kSolveThreads) v[i] -= col[i] * xj;
        __syncthreads();
    }
}

__global__ void __launch_bounds__(kSolveThreads) k_bwd_solve(DevPlan d, const int32_t *__restrict__ list,
                                                             double *__restrict__ y,
                                                             const int32_t *__restrict__ sn_rows,
                                                             const int64_t *__restrict__ sn_rowptr) {
    const int s = list[blockIdx.x];
    const int k = d.sn_k[s], f = d.sn_f[s], ld = d.sn_ld[s], first = d.sn_first[s];
    double *__restrict__ v = d.fv + d.fv_off[s];
    const double *__restrict__ P = d.L + d.L_off[s];
    const int32_t *__restrict__ R = sn_rows + sn_rowptr[s];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    __shared__ double red[kSolveThreads / 32];
    for (int i = k + tid; i < f; i += kSolveThreads) v[i] = y[R[i]];   // ancestors are final
    __syncthreads();
    for (int j = k - 1; j >= 0; j--) {
        const double *__restrict__ col = P + (int64_t)j * ld;
        double part = 0.0;
        for (int i = j + 1 + tid; i < f; i += kSolveThreads) part += col[i] * v[i];
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
        if (lane == 0) red[warp] = part;
        __syncthreads();
        if (tid == 0) {
            double tot = 0.0;
            for (int w = 0; w < kSolveThreads / 32; w++) tot += red[w];
            const double xj = (y[first + j] - tot) / col[j];
            v[j] = xj;
            y[first + j] = xj;
        }
        __syncthreads();
    }
}

// ---- large supernodes: blocked by w = 64 columns, many CTAs per supernode
__global__ void __launch_bounds__(kSolveThreads) k_fsolve_init(DevPlan d, const int32_t *__restrict__ list,
                                                               const double *__restrict__ y) {
    const int s = list[blockIdx.x];
    const int k = d.sn_k[s], f = d.sn_f[s], first = d.sn_first[s];
    double *__restrict__ v = d.fv + d.fv_off[s];
    for (int i = threadIdx.x; i < f; i += kSolveThreads) v[i] = i < k ? y[first + i] : 0.0;
    __syncthreads();
    for (int q = d.child_ptr[s]; q < d.child_ptr[s + 1]; q++) {
        const int c = d.child_list[q];
        const int kc = d.sn_k[c], mc = d.sn_f[c] - kc;
        const int32_t *__restrict__ rel = d.relmap + d.relmap_ptr[c];
        const double *__restrict__ vc = d.fv + d.fv_off[c] + kc;
        for (int p = threadIdx.x; p < mc; p += kSolveThreads) v[rel[p]] += vc[p];
        __syncthreads();
    }
}

constexpr int kSW = 64, kSLD = 65;   // solve block width and smem leading dimension

__device__ __forceinline__ void load_diag_block(const double *__restrict__ P, int ld, int j0, int we,
                                                double *__restrict__ Lb) {
    for (int c = threadIdx.x >> 6; c < we; c += kSolveThreads / 64) {
        const int r = threadIdx.x & 63;
        if (r < we && r >= c) Lb[r + c * kSLD] = P[(j0 + r) + (int64_t)(j0 + c) * ld];
    }
}

__global__ void __launch_bounds__(kSolveThreads) k_fsolve_wave(DevPlan d, const int32_t *__restrict__ tasks, int j0,
                                                               int w, double *__restrict__ y) {
    __shared__ double Lb[kSW * kSLD];
    __shared__ double xs[kSW];
    const int s = tasks[3 * blockIdx.x], row0 = tasks[3 * blockIdx.x + 1], writer = tasks[3 * blockIdx.x + 2];
    const int k = d.sn_k[s], f = d.sn_f[s], ld = d.sn_ld[s], first = d.sn_first[s];
    const int we = min(w, k - j0);
    const double *__restrict__ P = d.L + d.L_off[s];
    double *__restrict__ v = d.fv + d.fv_off[s];
    const int tid = threadIdx.x, lane = tid & 31;
    load_diag_block(P, ld, j0, we, Lb);
    __syncthreads();
    if (tid < 32) {   // L11 x = v[j0:j0+we], right-looking, two entries per lane
        double a0 = lane < we ? v[j0 + lane] : 0.0, a1 = lane + 32 < we ? v[j0 + lane + 32] : 0.0;
        for (int c = 0; c < we; c++) {
            const double xc = __shfl_sync(0xffffffffu, c < 32 ? a0 : a1, c & 31) / Lb[c + c * kSLD];
            if (lane == 0) xs[c] = xc;
            if (lane > c && lane < we) a0 -= Lb[lane + c * kSLD] * xc;
            if (lane + 32 > c && lane + 32 < we) a1 -= Lb[lane + 32 + c * kSLD] * xc;
        }
    }
    __syncthreads();
    if (writer && tid < we) y[first + j0 + tid] = xs[tid];
    const int r = row0 + tid;
    if (r < min(row0 + kSolveRows, f)) {
        double acc = v[r];
        for (int c = 0; c < we; c++) acc -= P[r + (int64_t)(j0 + c) * ld] * xs[c];
        v[r] = acc;
    }
}

__global__ void __launch_bounds__(kSolveThreads) k_bsolve_init(DevPlan d, const int32_t *__restrict__ list,
                                                               const double *__restrict__ y,
                                                               const int32_t *__restrict__ sn_rows,
                                                               const int64_t *__restrict__ sn_rowptr) {
    const int s = list[blockIdx.x];
    const int k = d.sn_k[s], f = d.sn_f[s];
    double *__restrict__ v = d.fv + d.fv_off[s];
    const int32_t *__restrict__ R = sn_rows + sn_rowptr[s];
    for (int i = k + threadIdx.x; i < f; i += kSolveThreads) v[i] = y[R[i]];
}

__global__ void __launch_bounds__(kSolveThreads) k_bsolve_wave(DevPlan d, const int32_t *__restrict__ tasks,
                                                               int64_t task_base, const int32_t *__restrict__ groups,
                                                               int j0, int w, double *__restrict__ y,
                                                               double *__restrict__ partials, int *__restrict__ counters) {
    __shared__ double red[kSolveThreads / 32][kSW];
    __shared__ double Lb[kSW * kSLD];
    __shared__ double tv[kSW];
    __shared__ int is_last;
    const int s = tasks[3 * blockIdx.x], row0 = tasks[3 * blockIdx.x + 1], grp = tasks[3 * blockIdx.x + 2];
    const int k = d.sn_k[s], f = d.sn_f[s], ld = d.sn_ld[s], first = d.sn_first[s];
    const int we = min(w, k - j0);
    const double *__restrict__ P = d.L + d.L_off[s];
    double *__restrict__ v = d.fv + d.fv_off[s];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    // partial (L2^T v)_c over this CTA's row chunk
    const int r = row0 + tid;
    const bool rok = r < min(row0 + kSolveRows, f);
    const double rv = rok ? v[r] : 0.0;
    for (int c = 0; c < we; c++) {
        double p = rok ? P[r + (int64_t)(j0 + c) * ld] * rv : 0.0;
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) p += __shfl_xor_sync(0xffffffffu, p, o);
        if (lane == 0) red[warp][c] = p;
    }
    __syncthreads();
    if (tid < we) {
        double t = 0.0;
        for (int q = 0; q < kSolveThreads / 32; q++) t += red[q][tid];
        partials[(task_base + blockIdx.x) * kSW + tid] = t;
    }
    __threadfence();
    __syncthreads();
    if (tid == 0) is_last = atomicAdd(&counters[grp], 1) == groups[2 * grp + 1] - 1;
    __syncthreads();
    if (!is_last) return;
    __threadfence();
    // the last CTA of the group reduces the partials in task order (deterministic) and solves L11^T x = t
    load_diag_block(P, ld, j0, we, Lb);
    if (tid < we) {
        const int t0 = groups[2 * grp], nt = groups[2 * grp + 1];
        double t = y[first + j0 + tid];
        for (int q = 0; q < nt; q++) t -= __ldcg(&partials[(int64_t)(t0 + q) * kSW + tid]);
        tv[tid] = t;
    }
    __syncthreads();
    if (tid < 32) {
        double a0 = lane < we ? tv[lane] : 0.0, a1 = lane + 32 < we ? tv[lane + 32] : 0.0;
        for (int c = we - 1; c >= 0; c--) {
            const double xc = __shfl_sync(0xffffffffu, c < 32 ? a0 : a1, c & 31) / Lb[c + c * kSLD];
            if (lane == (c & 31)) {
                if (c < 32) a0 = xc; else a1 = xc;
            }
            if (lane < c) a0 -= Lb[c + lane * kSLD] * xc;
            if (lane + 32 < c) a1 -= Lb[c + (lane + 32) * kSLD] * xc;
        }
        if (lane < we) {
            y[first + j0 + lane] = a0;
            v[j0 + lane] = a0;
        }
        if (lane + 32 < we) {
            y[first + j0 + lane + 32] = a1;
            v[j0 + lane + 32] = a1;
        }
    }
}

void launch_fsolve_init(const DevPlan &d, const int32_t *list, int count, const double *y, cudaStream_t st) {
    if (count > 0) k_fsolve_init<<<count, kSolveThreads, 0, st>>>(d, list, y);
}
void launch_fsolve_wave(const DevPlan &d, const int32_t *tasks, int64_t count, int j0, int w, double *y,
                        cudaStream_t st) {
    if (count > 0) k_fsolve_wave<<<(unsigned)count, kSolveThreads, 0, st>>>(d, tasks, j0, w, y);
}
void launch_bsolve_init(const DevPlan &d, const int32_t *list, int count, const double *y, const int32_t *sn_rows,
                        const int64_t *sn_rowptr, cudaStream_t st) {
    if (count > 0) k_bsolve_init<<<count, kSolveThreads, 0, st>>>(d, list, y, sn_rows, sn_rowptr);
}
void launch_bsolve_wave(const DevPlan &d, const int32_t *tasks, int64_t task_base, int64_t count, const int32_t *groups,
                        int j0, int w, double *y, double *partials, int *counters, cudaStream_t st) {
    if (count > 0)
        k_bsolve_wave<<<(unsigned)count, kSolveThreads, 0, st>>>(d, tasks, task_base, groups, j0, w, y, partials,
                                                                  counters);
}

void launch_fwd_solve(const DevPlan &d, const int32_t *list, int count, double *y, cudaStream_t st) {
    if (count > 0) k_fwd_solve<<<count, kSolveThreads, 0, st>>>(d, list, y);
}
void launch_bwd_solve(const DevPlan &d, const int32_t *list, int count, double *y, const int32_t *sn_rows,
                      const int64_t *sn_rowptr, cudaStream_t st) {
    if (count > 0) k_bwd_solve<<<count, kSolveThreads, 0, st>>>(d, list, y, sn_rows, sn_rowptr);
}

}  // namespace mf
