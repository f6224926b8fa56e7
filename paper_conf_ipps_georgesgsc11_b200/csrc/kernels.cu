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
#include <algorithm>
#include <cstdlib>
#include <climits>
#include <cstdio>

#include "dmma_update.cuh"
#include "kernels.cuh"
#include "ozaki_update.cuh"

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

__global__ void k_init_failed(int *failed, unsigned *epoch) {
    *failed = INT_MAX;
    *epoch += 1;   // new factorization: fused-leaf flags of the previous one no longer match
}

// 1/sqrt(x) for a pivot: float MUFU seed + two fp64 Newton steps (~1 ulp; exactly
// 2^-p for x = 4^p, so the manufactured integer factors stay exact).  Outside the
// float range (or for x <= 0 / NaN) it falls back to the library rsqrt.
__device__ __forceinline__ double pivot_rsqrt(double x) {
    if (!(x > 1e-30 && x < 1e30)) return rsqrt(x);
    double y = (double)rsqrtf((float)x);
    double h = x * y;
    double r = fma(-h, y, 1.0);
    y = fma(0.5 * y, r, y);
    h = x * y;
    r = fma(-h, y, 1.0);
    return fma(0.5 * y, r, y);
}

// ============================================================ shared building block
// Factor the nb x nb diagonal sub-block A[s0:s0+nb, s0:s0+nb] (nb <= 16,
// column-major, leading dimension lda, already updated) in the registers of the
// calling warp: lane l < 16 owns row s0+l, pivots are broadcast by shuffles, so
// the pivot chain needs no block barrier.  Writes L back to A (and to gP, if
// given), 1/L_jj to sinv[s0+j], and flags non-positive pivots (reading C8).
__device__ __forceinline__ void warp_factor16(double *A, int lda, int s0, int nb, double *sinv, const DevPlan &d,
                                              int first_col, double *__restrict__ gP, int64_t gld) {
    const int lane = threadIdx.x & 31, l = lane & 15;
    double a[16];
#pragma unroll
    for (int q = 0; q < 16; q++) a[q] = (q <= l && l < nb) ? A[(s0 + q) * lda + s0 + l] : 0.0;
#pragma unroll
    for (int q = 0; q < 16; q++) {
        if (q < nb) {
            const double dq = __shfl_sync(0xffffffffu, a[q], q);
            const double inv = rsqrt(dq);
            const double piv = dq * inv;
            if (lane == q) {
                note_pivot(d, dq, first_col + q);
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
    __syncwarp();   // every lane's reads of the block precede the write-back
    if (lane < nb) {
#pragma unroll
        for (int q = 0; q < 16; q++)
            if (q <= lane) {
                A[(s0 + q) * lda + s0 + lane] = a[q];
                if (gP) gP[(s0 + lane) + (s0 + q) * gld] = a[q];
            }
    }
}

// ============================================================ small fronts
// One CTA per front; the whole f x f front lives in shared memory (column-major,
// leading dimension f).  Assembly (zero, A entries, extend-add of the children
// in ascending order), then the F-U step on the k pivot columns in blocks of
// 16: the diagonal sub-block in the registers of warp 0, the rows below it one
// thread per row (substitution), and the rank-16 update of the trailing lower
// triangle (which includes U^n = F22 - L2 L2^T).  Writes the L panel and U^n.
template <int NT>
__global__ void __launch_bounds__(NT) k_small_front(DevPlan d, const int32_t *__restrict__ list,
                                                    const double *__restrict__ values) {
    extern __shared__ double F[];
    constexpr int NW = NT / 32;
    constexpr int RP = NT < 128 ? NT : 128;   // rows per pass of the trailing update
    constexpr int H = NT / RP;                // column groups
    const int s = list[blockIdx.x];
    const int k = d.sn_k[s], f = d.sn_f[s], m = f - k, first = d.sn_first[s];
    double *sinv = F + f * f;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    for (int i = tid; i < f * f; i += NT) F[i] = 0.0;
    __syncthreads();
    for (int j = warp; j < k; j += NW) {        // A entries: warp per column
        const int64_t e0 = d.bcolptr[first + j], e1 = d.bcolptr[first + j + 1];
        for (int64_t e = e0 + lane; e < e1; e += 32) F[d.blrow[e] + j * f] = sum_values(d, values, e);
    }
    __syncthreads();
    for (int q = d.child_ptr[s]; q < d.child_ptr[s + 1]; q++) {   // extend-add, ascending children
        const int c = d.child_list[q];
        const int mc = d.sn_f[c] - d.sn_k[c];
        const int32_t *__restrict__ rel = d.relmap + d.relmap_ptr[c];
        const double *__restrict__ Uc = d.U + d.U_off[c];
        for (int qq = warp; qq < mc; qq += NW) {
            double *dst = F + rel[qq] * f;
            const double *ucol = Uc + upk_col(qq, mc) - qq;   // packed column qq, indexed by row
            for (int p = qq + lane; p < mc; p += 32) dst[rel[p]] += ucol[p];
        }
        __syncthreads();
    }
    for (int s0 = 0; s0 < k; s0 += 16) {
        const int nb = min(16, k - s0);
        if (warp == 0) warp_factor16(F, f, s0, nb, sinv, d, first + s0, nullptr, 0);
        __syncthreads();
        const int r0 = s0 + nb;
        if (r0 >= f) break;
        for (int r = r0 + tid; r < f; r += NT) {   // rows below: x L_sub^T = a
            double x[16];
#pragma unroll
            for (int q = 0; q < 16; q++) x[q] = q < nb ? F[r + (s0 + q) * f] : 0.0;
#pragma unroll
            for (int q = 0; q < 16; q++) {
                if (q < nb) {
                    x[q] *= sinv[s0 + q];
#pragma unroll
                    for (int q2 = q + 1; q2 < 16; q2++)
                        if (q2 < nb) x[q2] -= x[q] * F[(s0 + q2) + (s0 + q) * f];
                }
            }
#pragma unroll
            for (int q = 0; q < 16; q++)
                if (q < nb) F[r + (s0 + q) * f] = x[q];
        }
        __syncthreads();
        // trailing update, rows/cols [r0, f): F[i][c] -= sum_q L[i][q] L[c][q]
        for (int i = r0 + (tid % RP), h = tid / RP; i < f; i += RP) {
            {
                double li[16];
#pragma unroll
                for (int q = 0; q < 16; q++) li[q] = q < nb ? F[i + (s0 + q) * f] : 0.0;
                for (int c = r0 + h; c <= i; c += H) {
                    double acc = F[i + c * f];
#pragma unroll
                    for (int q = 0; q < 16; q++)
                        if (q < nb) acc -= li[q] * F[c + (s0 + q) * f];
                    F[i + c * f] = acc;
                }
            }
        }
        __syncthreads();
    }
    // write the L panel (upper triangle of L1 = 0) and U^n (lower triangle)
    double *__restrict__ P = d.L + d.L_off[s];
    const int ld = d.sn_ld[s];
    for (int j = warp; j < k; j += NW)
        for (int i = lane; i < f; i += 32) P[i + (int64_t)j * ld] = i >= j ? F[i + j * f] : 0.0;
    if (m > 0) {
        double *__restrict__ Us = d.U + d.U_off[s];
        for (int c = warp; c < m; c += NW)
            for (int i = c + lane; i < m; i += 32) Us[upk(i, c, m)] = F[(k + i) + (k + c) * f];
    }
}

// ============================================================ tiny fronts (f <= 32)
// One WARP per front (4 fronts per CTA), no block barriers: the front is
// assembled in a per-warp shared-memory tile (zero, A entries, children's U^c
// in ascending order), then lane i holds row i in registers and the k pivots
// are eliminated right-looking with shuffles over the WHOLE front, which
// yields L1, L2 and U^n = F22 - L2 L2^T together.  c2 (9-point 1000^2) has
// ~230k such fronts.
constexpr int kTinyF = 32, kTinyWarps = 4;
template <int TF>
__global__ void __launch_bounds__(32 * kTinyWarps, TF <= 16 ? 8 : 4)
    k_tiny_fronts(DevPlan d, const int32_t *__restrict__ list, int count, const double *__restrict__ values) {
    constexpr int kTinyLD = TF + 1;
    __shared__ double Fs[kTinyWarps][TF * kTinyLD];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int idx = blockIdx.x * kTinyWarps + warp;
    if (idx >= count) return;
    double *F = Fs[warp];
    const int s = list[idx];
    const int k = d.sn_k[s], f = d.sn_f[s], m = f - k, first = d.sn_first[s];
    if (lane < TF)
        for (int c = 0; c < f; c++) F[lane + c * kTinyLD] = 0.0;
    __syncwarp();
    for (int j = 0; j < k; j++) {
        const int64_t e0 = d.bcolptr[first + j], e1 = d.bcolptr[first + j + 1];
        for (int64_t e = e0 + lane; e < e1; e += 32) F[d.blrow[e] + j * kTinyLD] = sum_values(d, values, e);
    }
    __syncwarp();
    for (int q = d.child_ptr[s]; q < d.child_ptr[s + 1]; q++) {
        const int c = d.child_list[q];
        const int mc = d.sn_f[c] - d.sn_k[c];
        const int32_t *__restrict__ rel = d.relmap + d.relmap_ptr[c];
        const double *__restrict__ Uc = d.U + d.U_off[c];
        const int myrel = lane < mc ? rel[lane] : 0;
        for (int qq = 0; qq < mc; qq++) {
            const int dc = __shfl_sync(0xffffffffu, myrel, qq);
            if (lane >= qq && lane < mc) F[myrel + dc * kTinyLD] += Uc[upk(lane, qq, mc)];
        }
        __syncwarp();
    }
    double a[TF];
#pragma unroll
    for (int c = 0; c < TF; c++) a[c] = lane < TF ? F[lane + c * kTinyLD] : 0.0;
#pragma unroll
    for (int j = 0; j < TF; j++) {
        if (j >= k) break;   // (uniform) the instruction stream stops at the front's k and f,
        const double dj = __shfl_sync(0xffffffffu, a[j], j);   // not at the class bound TF
        const double inv = rsqrt(dj);
        if (lane == j) {
            note_pivot(d, dj, first + j);
            a[j] = dj * inv;
        } else if (lane > j) {
            a[j] *= inv;
        }
#pragma unroll
        for (int c = j + 1; c < TF; c++) {
            if (c >= f) break;
            const double lc = __shfl_sync(0xffffffffu, a[j], c);
            if (lane >= c) a[c] -= a[j] * lc;
        }
    }
    if (lane < f) {
        double *__restrict__ P = d.L + d.L_off[s];
        const int ld = d.sn_ld[s];
#pragma unroll
        for (int j = 0; j < TF; j++) {
            if (j >= k) break;
            P[lane + (int64_t)j * ld] = lane >= j ? a[j] : 0.0;
        }
        if (m > 0) {
            double *__restrict__ Us = d.U + d.U_off[s];
#pragma unroll
            for (int c = 0; c < TF; c++) {
                if (c >= f) break;
                if (c >= k && lane >= c) Us[upk(lane - k, c - k, m)] = a[c];
            }
        }
    }
}

int small_front_smem_ok(int fmax) { return (size_t)(fmax * fmax + fmax) * sizeof(double) <= 227 * 1024; }

void launch_small_fronts(const DevPlan &d, const int32_t *list, int count, int fmax, const double *values,
                         cudaStream_t st) {
    if (count <= 0) return;
    const size_t smem = (size_t)(fmax * fmax + fmax) * sizeof(double);
    if (fmax <= 16) {
        k_tiny_fronts<16><<<(count + kTinyWarps - 1) / kTinyWarps, 32 * kTinyWarps, 0, st>>>(d, list, count, values);
    } else if (fmax <= kTinyF) {   // kTinyF = 32: every f <= 32 class is one warp per front
        k_tiny_fronts<32><<<(count + kTinyWarps - 1) / kTinyWarps, 32 * kTinyWarps, 0, st>>>(d, list, count, values);
    } else if (fmax <= 64) {
        k_small_front<128><<<count, 128, smem, st>>>(d, list, values);
    } else {
        k_small_front<256><<<count, 256, smem, st>>>(d, list, values);
    }
}

// ============================================================ large-front assembly
// Task = (front s, first local column c0): columns [c0, c0+32) of the front.
// Columns < k live in the L panel, columns >= k in U^s.
constexpr int kAsmThreads = 256;
constexpr int kAsmChunk = 512;   // rows per shared-memory staging chunk (per warp)
// Each warp owns whole destination columns (round-robin over the task's 32
// columns) and builds each column chunk by chunk in shared memory: zero, its A
// entries, then every child's matching U^c column in ascending child order --
// and writes the finished chunk to HBM once.  One warp performs every update of
// its entries, so the summation order (0 + A + U^c1 + U^c2 + ...) is fixed
// without barriers or atomics, and the destination is written exactly once
// (no zero-fill pass, no read-modify-write).  Child column q lands in
// destination column c iff rel[q] == c (rel is increasing: binary search); its
// rows falling in a chunk are a contiguous range of rel.
__device__ __forceinline__ int lower_bound_rel(const int32_t *__restrict__ rel, int lo, int hi, int key) {
    while (lo < hi) {
        const int mid = (lo + hi) >> 1;
        if (__ldg(rel + mid) < key) lo = mid + 1; else hi = mid;
    }
    return lo;
}

constexpr int kAsmMaxCh = 32;   // children handled through the shared column map (more: searched per column)
static_assert(kAsmRowBlock % kAsmChunk == 0, "row blocks are whole chunks");
__global__ void __launch_bounds__(kAsmThreads) k_assemble(DevPlan d, const int32_t *__restrict__ tasks,
                                                          const double *__restrict__ values) {
    constexpr int NW = kAsmThreads / 32;
    __shared__ double sbuf[NW][kAsmChunk];
    __shared__ int colmap[kAsmMaxCh][kAsmCols];   // child column landing in column c0 + x, or -1
    __shared__ int s_cp[NW][kAsmMaxCh];           // per warp and child: next child row to add
    // task = (front, c0 | row block << 20): columns [c0, c0 + kAsmCols), rows of row block
    // rb = [rb kAsmRowBlock, (rb + 1) kAsmRowBlock) -- tall fronts are split by rows so that
    // their assembly spreads over the SMs (every element is still built by one warp:
    // 0 + A + U^c1 + U^c2 ..., reading C6)
    const int s = tasks[2 * blockIdx.x], c0 = tasks[2 * blockIdx.x + 1] & 0xfffff;
    const int rb = tasks[2 * blockIdx.x + 1] >> 20;
    const int k = d.sn_k[s], f = d.sn_f[s], m = f - k, ld = d.sn_ld[s], first = d.sn_first[s];
    const int c1 = min(c0 + kAsmCols, d.fuse_ea ? k : f);   // fused extend-add: U^s is gathered by the syrk
    double *__restrict__ P = d.L + d.L_off[s];
    double *__restrict__ Us = d.U + d.U_off[s];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    double *buf = sbuf[warp];
    int *cp = s_cp[warp];
    const int q0 = d.child_ptr[s], q1 = d.child_ptr[s + 1];
    const int nch = q1 - q0, nmap = min(nch, kAsmMaxCh);
    // column map: the child columns q with rel[q] in [c0, c1) form one contiguous range per child
    for (int i = tid; i < nmap * kAsmCols; i += kAsmThreads) colmap[i / kAsmCols][i % kAsmCols] = -1;
    __syncthreads();
    for (int j = warp; j < nmap; j += NW) {
        const int ch = d.child_list[q0 + j];
        const int mc = d.sn_f[ch] - d.sn_k[ch];
        const int32_t *__restrict__ rel = d.relmap + d.relmap_ptr[ch];
        const int qa = lower_bound_rel(rel, 0, mc, c0);
        const int qb = lower_bound_rel(rel, qa, mc, c1);
        for (int q = qa + lane; q < qb; q += 32) colmap[j][__ldg(rel + q) - c0] = q;
    }
    __syncthreads();
    for (int c = c0 + warp; c < c1; c += NW) {
        // destination column: panel column c (rows 0..f-1) or U column c-k (rows c..f-1)
        double *__restrict__ col;
        int rlo;
        if (c < k) {
            col = P + (int64_t)c * ld;
            rlo = 0;
        } else {
            col = Us + upk_col(c - k, m) - c;   // packed column c - k, indexed by front row r >= c
            rlo = c;
        }
        const int rbeg = max(rlo, rb * kAsmRowBlock), rend = min(f, (rb + 1) * kAsmRowBlock);
        if (rbeg >= rend) continue;   // (uniform over the warp)
        if (lane < nmap) {            // rel[qc] = c: the child's rows start at the diagonal
            int qc = colmap[lane][c - c0];
            if (qc >= 0 && rbeg > c) {   // ... or, in a lower row block, at its first row >= rbeg
                const int ch = d.child_list[q0 + lane];
                qc = lower_bound_rel(d.relmap + d.relmap_ptr[ch], qc, d.sn_f[ch] - d.sn_k[ch], rbeg);
            }
            cp[lane] = qc;
        }
        __syncwarp();
        const int64_t e0 = c < k ? d.bcolptr[first + c] : 0, e1 = c < k ? d.bcolptr[first + c + 1] : 0;
        for (int r0 = rbeg; r0 < rend; r0 += kAsmChunk) {
            const int r1 = min(r0 + kAsmChunk, rend);
            for (int r = r0 + lane; r < r1; r += 32) buf[r - r0] = 0.0;
            __syncwarp();
            for (int64_t e = e0 + lane; e < e1; e += 32) {
                const int r = d.blrow[e];
                if (r >= r0 && r < r1) buf[r - r0] = sum_values(d, values, e);
            }
            __syncwarp();
            for (int j = 0; j < nch; j++) {
                const int ch = d.child_list[q0 + j];
                const int mc = d.sn_f[ch] - d.sn_k[ch];
                const int32_t *__restrict__ rel = d.relmap + d.relmap_ptr[ch];
                int qc, p;
                if (j < kAsmMaxCh) {
                    qc = colmap[j][c - c0];
                    if (qc < 0) continue;
                    p = cp[j];
                } else {   // rare: more children than the map holds
                    qc = lower_bound_rel(rel, 0, mc, c);
                    if (qc >= mc || __ldg(rel + qc) != c) continue;
                    p = lower_bound_rel(rel, qc, mc, r0);
                }
                const double *__restrict__ ucol = d.U + d.U_off[ch] + upk_col(qc, mc) - qc;   // packed column qc
                // consume child rows p, p+1, ... while rel < r1 (rel is increasing): 256 rows per
                // step (8 loads of each kind in flight per lane), the stop found by warp ballots
                while (p < mc) {
                    int rr[8];
                    double uu[8];
#pragma unroll
                    for (int t = 0; t < 8; t++) {
                        const int idx = p + 32 * t + lane;
                        rr[t] = idx < mc ? __ldg(rel + idx) : INT_MAX;
                        uu[t] = idx < mc ? __ldg(ucol + idx) : 0.0;
                    }
                    int taken = 0;
                    bool stop = false;
#pragma unroll
                    for (int t = 0; t < 8; t++) {
                        const bool in = rr[t] < r1;
                        if (in) buf[rr[t] - r0] += uu[t];
                        const int n_in = __popc(__ballot_sync(0xffffffffu, in));
                        if (!stop) taken += n_in;
                        stop = stop || n_in < 32;
                    }
                    p += taken;
                    if (stop) break;
                }
                __syncwarp();
                if (j < kAsmMaxCh && lane == 0) cp[j] = p;
            }
            __syncwarp();
            for (int r = r0 + lane; r < r1; r += 32) col[r] = buf[r - r0];
            __syncwarp();
        }
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
constexpr int kPotrfThreads = 256;
// Blocked in-CTA potrf of the 64 x 64 diagonal block, 8 columns at a time:
//  (a) one thread factors the 8 x 8 diagonal sub-block in registers (measured:
//      ~100 cycles per pivot, vs ~450 for a warp exchanging rows by shuffles),
//  (b) one thread per row solves the rows below it against that sub-block,
//  (c) all threads apply the rank-8 update to the trailing lower triangle;
// the finished block is written back once, coalesced.  1/L_jj uses rsqrt
// (exact for the power-of-4 pivots of the manufactured inputs); L_jj = d*rsqrt(d).
template <int NT>
__device__ __forceinline__ void potrf_block(const DevPlan &d, int s, int j0, int w, double *A, double *sinv) {
    constexpr int LDA = kWmax;            // column-major: A[c * LDA + r]
    constexpr int G = NT / 64;            // column groups
    constexpr int SB = 8;                 // sub-block width
    const int k = d.sn_k[s], ld = d.sn_ld[s], first = d.sn_first[s];
    const int we = min(w, k - j0);
    double *__restrict__ P = d.L + d.L_off[s] + (int64_t)j0 * ld + j0;
    const int tid = threadIdx.x;
    {
        const int i = tid & 63, h = tid >> 6;
        double v[kWmax / G];
#pragma unroll
        for (int t = 0; t < kWmax / G; t++) {
            const int c = h + G * t;
            v[t] = (i < we && c < we) ? P[i + (int64_t)c * ld] : 0.0;
        }
#pragma unroll
        for (int t = 0; t < kWmax / G; t++) A[(h + G * t) * LDA + i] = v[t];
    }
    __syncthreads();
#pragma unroll 1
    for (int s0 = 0; s0 < we; s0 += SB) {
        const int nb = min(SB, we - s0);
        // (a) the 8 x 8 diagonal sub-block in the registers of ONE thread: the pivot
        //     chain is rsqrt + a few dependent FMAs, everything else pipelines
        if (tid == 0) {
            double a[SB][SB];
#pragma unroll
            for (int c = 0; c < SB; c++)
#pragma unroll
                for (int r = c; r < SB; r++) a[r][c] = (r < nb) ? A[(s0 + c) * LDA + s0 + r] : (r == c ? 1.0 : 0.0);
#pragma unroll
            for (int q = 0; q < SB; q++) {
                if (q < nb) note_pivot(d, a[q][q], first + j0 + s0 + q);
                const double inv = rsqrt(a[q][q]);
                a[q][q] *= inv;
                sinv[s0 + q] = inv;
#pragma unroll
                for (int r = q + 1; r < SB; r++) a[r][q] *= inv;
#pragma unroll
                for (int c = q + 1; c < SB; c++)
#pragma unroll
                    for (int r = c; r < SB; r++) a[r][c] = fma(-a[r][q], a[c][q], a[r][c]);
            }
#pragma unroll
            for (int c = 0; c < SB; c++)
#pragma unroll
                for (int r = c; r < SB; r++)
                    if (r < nb) A[(s0 + c) * LDA + s0 + r] = a[r][c];
        }
        __syncthreads();
        const int r0 = s0 + SB;
        if (r0 >= we) break;
        // (b) rows r in [r0, we): x L_sub^T = a  (one thread per row)
        if (tid < we - r0) {
            const int r = r0 + tid;
            double x[SB];
#pragma unroll
            for (int q = 0; q < SB; q++) x[q] = A[(s0 + q) * LDA + r];
#pragma unroll
            for (int q = 0; q < SB; q++) {
                x[q] *= sinv[s0 + q];
#pragma unroll
                for (int q2 = q + 1; q2 < SB; q2++) x[q2] -= x[q] * A[(s0 + q) * LDA + s0 + q2];
            }
#pragma unroll
            for (int q = 0; q < SB; q++) A[(s0 + q) * LDA + r] = x[q];
        }
        __syncthreads();
        // (c) trailing update: A[c][i] -= sum_q L[i][q] L[c][q], r0 <= c <= i < we
        {
            const int i = tid & 63, h = tid >> 6;
            if (i >= r0 && i < we) {
                double li[SB];
#pragma unroll
                for (int q = 0; q < SB; q++) li[q] = A[(s0 + q) * LDA + i];
                for (int c = r0 + h; c <= i; c += G) {
                    double acc = A[c * LDA + i];
#pragma unroll
                    for (int q = 0; q < SB; q++) acc -= li[q] * A[(s0 + q) * LDA + c];
                    A[c * LDA + i] = acc;
                }
            }
        }
        __syncthreads();
    }
    __syncthreads();
    // coalesced write-back of the finished lower triangle
    for (int c = tid >> 6; c < we; c += G) {
        const int i = tid & 63;
        if (i < we && i >= c) P[i + (int64_t)c * ld] = A[c * LDA + i];
    }
}

__global__ void __launch_bounds__(kPotrfThreads) k_potrf_diag(DevPlan d, const int32_t *__restrict__ fronts,
                                                              int j0, int w) {
    __shared__ double A[kWmax * kWmax];
    __shared__ double sinv[kWmax];
    potrf_block<kPotrfThreads>(d, fronts[blockIdx.x], j0, w, A, sinv);
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
constexpr int kTrsmThreads = kTrsmRows;   // 4 warps, each owning 32 rows
constexpr int kLLD = kWmax + 2;             // L11 smem: column-major, even stride (16-byte cp.async)
constexpr int kXLD = kTrsmRows + 2;         // X smem: column-major, even stride
constexpr size_t kTrsmSmem = (size_t)(kWmax * kLLD + kWmax * kXLD + kWmax) * sizeof(double);
// X L11^T = B by blocked substitution: for each 8-column block, every thread
// solves its own row over the block (scalar), then its warp applies the block
// to the remaining columns of its 32 rows with DMMA (m8n8k4 f64).  Warps never
// share rows, so only warp-level synchronisation is needed.  No explicit
// inverse of L11: integer-exact on the manufactured inputs.  L11 and the row
// block are staged with cp.async (all loads in flight at once).
// wait until `flag` holds `expect` (written by the CTA that factored the diagonal
// block, after a fence); used by the fused potrf+trsm leaf launch
__device__ __forceinline__ void wait_flag(const unsigned *flag, unsigned expect) {
    if (threadIdx.x == 0) {
        unsigned v;
        do {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(flag) : "memory");
            if (v != expect) __nanosleep(32);
        } while (v != expect);
    }
    __syncthreads();
}

__device__ __forceinline__ void trsm_block(const DevPlan &d, int s, int r0, int j0, int w, double *tsm,
                                           const unsigned *flag, unsigned expect) {
    double *Ls = tsm;                           // L11[r][c] at Ls[r + c * kLLD]
    double *X = tsm + kWmax * kLLD;             // X[r][c]   at X[r + c * kXLD]
    double *inv = X + kWmax * kXLD;
    const int k = d.sn_k[s], f = d.sn_f[s], ld = d.sn_ld[s];
    const int we = min(w, k - j0);
    const int nr = min(kTrsmRows, f - r0);
    const double *__restrict__ D = d.L + d.L_off[s] + (int64_t)j0 * ld + j0;   // 16B aligned: j0 even, ld even
    double *__restrict__ B = d.L + d.L_off[s] + (int64_t)j0 * ld + r0;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    // the row block first (independent of the diagonal block) ...
    if ((r0 & 1) == 0) {
        for (int q = tid; q < (kTrsmRows / 2) * kWmax; q += kTrsmThreads) {
            const int rr = 2 * (q % (kTrsmRows / 2)), c = q / (kTrsmRows / 2);
            const bool ok = c < we && rr < nr;
            cp_async16(X + rr + c * kXLD, ok ? B + rr + (int64_t)c * ld : B, ok);
        }
    } else {
        for (int c = 0; c < kWmax; c++) {
            const bool ok = c < we && tid < nr;
            cp_async8(X + tid + c * kXLD, ok ? B + tid + (int64_t)c * ld : B, ok);
        }
    }
    cp_async_commit();
    // ... then L11 (64 x we, pairs of rows per 16-byte chunk; rows >= we padded below),
    // once the diagonal block is final (fused leaf launch: wait for its flag; the
    // 16-byte cp.async.cg path reads L2, never a stale L1 line)
    if (flag) wait_flag(flag, expect);
    for (int q = tid; q < (kWmax / 2) * kWmax; q += kTrsmThreads) {
        const int rr = 2 * (q % (kWmax / 2)), c = q / (kWmax / 2);
        const bool ok = c < we && rr < we;
        cp_async16(Ls + rr + c * kLLD, ok ? D + rr + (int64_t)c * ld : D, ok);
    }
    cp_async_commit();
    cp_async_wait<0>();
    __syncthreads();
    // identity padding of L11 beyond we (rows/cols); strict upper part is never read
    if (tid < kWmax) {
        if (tid >= we) {
            for (int c = 0; c < kWmax; c++) Ls[tid + c * kLLD] = (c == tid) ? 1.0 : 0.0;
        } else {
            for (int c = we; c < kWmax; c++) Ls[tid + c * kLLD] = 0.0;
        }
    }
    __syncthreads();
    if (tid < kWmax) inv[tid] = __drcp_rn(Ls[tid + tid * kLLD]);
    __syncthreads();
    const int gq = lane >> 2, tq = lane & 3;
    double *Xw = X + warp * 32;                 // this warp's 32 rows
    const int ncb = (we + 7) / 8;
#pragma unroll
    for (int cb = 0; cb < kWmax / 8; cb++) {
        if (cb >= ncb) break;
        const int c0 = cb * 8;
        double xv[8];
#pragma unroll
        for (int q = 0; q < 8; q++) xv[q] = X[tid + (c0 + q) * kXLD];
#pragma unroll
        for (int q = 0; q < 8; q++) {
            xv[q] *= inv[c0 + q];
#pragma unroll
            for (int q2 = q + 1; q2 < 8; q2++) xv[q2] -= xv[q] * Ls[(c0 + q2) + (c0 + q) * kLLD];
        }
#pragma unroll
        for (int q = 0; q < 8; q++) X[tid + (c0 + q) * kXLD] = xv[q];
        __syncwarp();
        // X[:, c0+8:] -= X[:, c0:c0+8] * L[c0+8:, c0:c0+8]^T  (rows of this warp)
#pragma unroll
        for (int nb = cb + 1; nb < kWmax / 8; nb++) {
            if (nb >= ncb) break;
#pragma unroll
            for (int mb = 0; mb < 4; mb++) {
                double *xr = Xw + mb * 8 + gq;
                double acc0 = xr[(nb * 8 + 2 * tq) * kXLD], acc1 = xr[(nb * 8 + 2 * tq + 1) * kXLD];
#pragma unroll
                for (int kk = 0; kk < 2; kk++) {
                    const double a = -xr[(c0 + kk * 4 + tq) * kXLD];
                    const double b = Ls[(nb * 8 + gq) + (c0 + kk * 4 + tq) * kLLD];
                    dmma(acc0, acc1, a, b);
                }
                xr[(nb * 8 + 2 * tq) * kXLD] = acc0;
                xr[(nb * 8 + 2 * tq + 1) * kXLD] = acc1;
            }
        }
        __syncwarp();
    }
    __syncthreads();
    for (int c = 0; c < we; c++)
        if (tid < nr) B[tid + (int64_t)c * ld] = X[tid + c * kXLD];
}

__global__ void __launch_bounds__(kTrsmThreads, 2) k_trsm_panel(DevPlan d, const int32_t *__restrict__ tasks,
                                                                int j0, int w) {
    extern __shared__ __align__(16) double tsm[];
    trsm_block(d, tasks[2 * blockIdx.x], tasks[2 * blockIdx.x + 1], j0, w, tsm, nullptr, 0);
}

// Ticket-ordered task ids.  The dataflow kernels below spin-
// wait on tasks with smaller ids; a CTA takes the next ticket as its task id when it
// starts, so every smaller ticket belongs to a CTA that is already resident and
// forward progress never depends on the hardware dispatching CTAs in blockIdx
// order (nor on how concurrent graph branches share the SMs).  Each launch slot
// owns a pair of counters; the last CTA to finish resets it for the next launch of
// the slot (stream-ordered, so no other launch of the slot is in flight).
__device__ __forceinline__ int take_ticket(unsigned *tk) {
    __shared__ int tkt;
    if (threadIdx.x == 0) tkt = (int)atomicAdd(tk, 1u);
    __syncthreads();
    return tkt;
}
__device__ __forceinline__ void drop_ticket(unsigned *tk) {
    __syncthreads();
    if (threadIdx.x == 0 && atomicAdd(tk + 1, 1u) == gridDim.x - 1) {
        tk[0] = 0u;
        tk[1] = 0u;
        tk[2] = 0u;   // the fused-init count of the solve launches (kTkWords)
        __threadfence();
    }
}

// Fused leaf: blocks [0, npotrf) factor the diagonal blocks of the active fronts
// (then publish a per-front flag), blocks [npotrf, ...) solve the row blocks below;
// each TRSM block stages its rows, waits for its front's flag, then loads L11.
// The diagonal-block CTAs have the lowest block indices, so they are dispatched
// first and never wait: no deadlock.  Saves one launch (and the row-block load
// latency) per leaf on the sequential chain of the top fronts.
__device__ __forceinline__ void leaf_task(const DevPlan &d, const int32_t *__restrict__ fronts, int npotrf,
                                          const int32_t *__restrict__ tasks, int j0, int w, const int task) {
    extern __shared__ __align__(16) double tsm[];
    // tag = (epoch mod 2^16) << 16 | leaf index + 1: consecutive factorizations differ in
    // the epoch bits, and the leaf index (k / w < 2^16 - 1, checked by build_plan) never
    // spills into them (10 bits overflowed for k > 1023 w)
    const unsigned expect = ((*d.epoch & 0xffffu) << 16) | (unsigned)(j0 / w + 1);
    if (task < npotrf) {
        const int s = fronts[task];
        potrf_block<kTrsmThreads>(d, s, j0, w, tsm, tsm + kWmax * kWmax);
        __threadfence();
        __syncthreads();
        if (threadIdx.x == 0)
            asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(d.leaf_flag + s), "r"(expect) : "memory");
        return;
    }
    const int t = task - npotrf;
    const int s = tasks[2 * t];
    trsm_block(d, s, tasks[2 * t + 1], j0, w, tsm, d.leaf_flag + s, expect);
}
__global__ void __launch_bounds__(kTrsmThreads, 2) k_leaf(DevPlan d, const int32_t *__restrict__ fronts, int npotrf,
                                                          const int32_t *__restrict__ tasks, int j0, int w,
                                                          unsigned *tk) {
    leaf_task(d, fronts, npotrf, tasks, j0, w, take_ticket(tk));
    drop_ticket(tk);
}

void launch_leaf(const DevPlan &d, const int32_t *fronts, int npotrf, const int32_t *tasks, int64_t ntrsm, int j0,
                 int w, unsigned *tk, cudaStream_t st) {
    if (npotrf <= 0) return;
    k_leaf<<<(unsigned)(npotrf + ntrsm), kTrsmThreads, kTrsmSmem, st>>>(d, fronts, npotrf, tasks, j0, w, tk);
}

// ============================================================ dataflow panel ("super-leaf")
// The base case of the recursive blocked factorization of the large fronts
// (Fig. 9: "a light-weight GPU kernel performing potrf on a w x w
// matrix", trsm on the rows below, the trailing update of the panel) for up to
// kPanelMaxBlocks blocks of 64 pivot columns [j0, j0 + 64 nbk), in ONE launch.
// A task is one 64-row tile row c (rows j0 + 64c ...) of one front; the tiles
// (c, b), b <= c, of that row are produced in order b = 0, 1, ...:
//   off-diagonal (b < c): X(c,b) -= sum_{b' < b} X(c,b') X(b,b')^T  (DMMA, K = 64 b,
//       operands from L2), wait for the diagonal tile (b,b), X(c,b) <- X(c,b) L_bb^-T
//       (substitution), store;
//   diagonal (b = c, the "band" tiles c < nb): the row's own products
//       X(c,b) X(c,b)^T are subtracted as each X(c,b) is finished (registers),
//       then potrf in shared memory, store, publish.
// Tiles publish epoch-tagged flags (band tiles (c,b) and the diagonal tiles);
// a task only waits on tasks of the same front with a smaller row index, which
// have smaller block indices (tasks are ordered row-major over the fronts), so
// the launch cannot deadlock.  This replaces, per panel of 4 blocks, 4 fused
// leaf launches and 3 narrow update launches whose latency serialised the
// factorization of the top fronts.
constexpr int kPanelThreads = 128;
constexpr int kPLD = 68;   // 64-row tiles in shared memory: stride = 4 mod 16 (conflict-free fragments), even (16-byte cp.async)
#ifndef MF_PANEL_STAGES
#define MF_PANEL_STAGES 2
#endif
#ifndef MF_PANEL_MINB
#define MF_PANEL_MINB 3
#endif
// 2-stage cp.async ring of 16-wide A / B slices: 70 KB of shared memory and <= 168
// registers give 3 CTAs / SM (3 stages: 87.5 KB, 255 registers, 2 CTAs / SM) --
// the many-front levels' panels are throughput-bound on their non-band tasks
constexpr int kPanelStages = MF_PANEL_STAGES;
constexpr int kPanelRingWords = kPanelStages * 16 * (2 * kPLD);
constexpr size_t kPanelSmem = (size_t)(kPanelRingWords + 64 * kPLD + 64) * sizeof(double);
static_assert(64 * kPLD <= kPanelRingWords, "the L_bb tile aliases the staging ring");

__device__ __forceinline__ int panel_tri(int c, int b) { return c * (c + 1) / 2 + b; }

// Phase timeline of the dataflow panel (tools/ubench/panel_timeline.cu defines
// MF_PANEL_TL; compiled out otherwise): %globaltimer at fixed event slots per task.
#ifdef MF_PANEL_TL
__device__ unsigned long long *g_panel_tl;
#define PANEL_TL(task, ev)                                                                   \
    do {                                                                                     \
        if (threadIdx.x == 0 && g_panel_tl) {                                                \
            unsigned long long t_;                                                           \
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_));                           \
            g_panel_tl[(int64_t)(task) * 64 + (ev)] = t_;                                    \
        }                                                                                    \
    } while (0)
#else
#define PANEL_TL(task, ev) do { } while (0)
#endif

// acc(64 x 64 tile; this warp's 32 x 32 fragment) -= A B^T with A = rows [ra0, ra0+64),
// B = rows [rb0, rb0+64), columns [kc0, kc0 + K) of the panel Pn (column-major, ld);
// rows >= arows / brows read as zero.  K is a multiple of 16.
__device__ __forceinline__ void panel_tile_mma(double (&acc)[4][4][2], double *ring, const double *__restrict__ Pn,
                                               int ld, int ra0, int arows, int rb0, int brows, int kc0, int K) {
    constexpr int BK = 16, STAGES = kPanelStages, STW = BK * 2 * kPLD;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int wm = warp & 1, wn = warp >> 1, gq = lane >> 2, tq = lane & 3;
    const int rr = 2 * lane, pt = warp;   // staging slot: row pair rr, k offsets pt + 4 i
    const bool oka = rr < arows, okb = rr < brows;
    auto load_stage = [&](int stage, int kt) {
        double *As = ring + stage * STW, *Bs = As + BK * kPLD;
        const double *__restrict__ Ak = Pn + (int64_t)(kc0 + kt * BK) * ld;
#pragma unroll
        for (int i = 0; i < 4; i++) {
            const int p = pt + 4 * i;
            cp_async16(As + p * kPLD + rr, oka ? Ak + (int64_t)p * ld + ra0 + rr : Pn, oka);
            cp_async16(Bs + p * kPLD + rr, okb ? Ak + (int64_t)p * ld + rb0 + rr : Pn, okb);
        }
    };
    const int KT = K / BK;
#pragma unroll
    for (int st = 0; st < STAGES - 1; st++) {
        if (st < KT) load_stage(st, st);
        cp_async_commit();
    }
    for (int kt = 0; kt < KT; kt++) {
        cp_async_wait<STAGES - 2>();
        __syncthreads();
        {
            const int nk = kt + STAGES - 1;
            if (nk < KT) load_stage(nk % STAGES, nk);
            cp_async_commit();
        }
        const double *As = ring + (kt % STAGES) * STW + wm * 32 + gq;
        const double *Bs = ring + (kt % STAGES) * STW + BK * kPLD + wn * 32 + gq;
#pragma unroll
        for (int kk = 0; kk < BK / 4; kk++) {
            double a[4], b[4];
#pragma unroll
            for (int mb = 0; mb < 4; mb++) a[mb] = -As[(kk * 4 + tq) * kPLD + mb * 8];
#pragma unroll
            for (int nb = 0; nb < 4; nb++) b[nb] = Bs[(kk * 4 + tq) * kPLD + nb * 8];
#pragma unroll
            for (int mb = 0; mb < 4; mb++)
#pragma unroll
                for (int nb = 0; nb < 4; nb++) dmma(acc[mb][nb][0], acc[mb][nb][1], a[mb], b[nb]);
        }
    }
    cp_async_wait<0>();
    __syncthreads();   // the ring is reused by the caller
}

// tile (rows r0.., cols c0..) of the panel <-> fragment registers / shared memory
__device__ __forceinline__ void panel_frag_load(double (&acc)[4][4][2], const double *__restrict__ Pn, int ld, int r0,
                                                int rows, int c0, int cols) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, wm = warp & 1, wn = warp >> 1;
#pragma unroll
    for (int mb = 0; mb < 4; mb++) {
        const int i = wm * 32 + mb * 8 + (lane >> 2);
#pragma unroll
        for (int nb = 0; nb < 4; nb++)
#pragma unroll
            for (int e = 0; e < 2; e++) {
                const int j = wn * 32 + nb * 8 + 2 * (lane & 3) + e;
                acc[mb][nb][e] = (i < rows && j < cols) ? Pn[(r0 + i) + (int64_t)(c0 + j) * ld] : 0.0;
            }
    }
}
__device__ __forceinline__ void panel_frag_to_smem(const double (&acc)[4][4][2], double *Xs) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, wm = warp & 1, wn = warp >> 1;
#pragma unroll
    for (int mb = 0; mb < 4; mb++) {
        const int i = wm * 32 + mb * 8 + (lane >> 2);
#pragma unroll
        for (int nb = 0; nb < 4; nb++)
#pragma unroll
            for (int e = 0; e < 2; e++) Xs[i + (wn * 32 + nb * 8 + 2 * (lane & 3) + e) * kPLD] = acc[mb][nb][e];
    }
}


// 1/sqrt(x): MUFU.RSQ64H seed (relative error e < 2^-22) + ONE second-order
// refinement y (1 + r/2 + 3r^2/8), r = 1 - x y^2, whose error is O(e^3) < 2^-66:
// four dependent operations on the pivot chain instead of the six of two Newton
// steps (tools/ubench/potrf_parts.cu: the 8 x 8 pivot block 982 -> 765 cycles).
// Exactly 2^-p for x = 4^p (the manufactured integer factors stay exact); ~1 ulp
// otherwise (reading C9).  Non-positive / NaN pivots come out NaN and are flagged
// by the caller.
__device__ __forceinline__ double rsqrt_nr(double x) {
    double y;
    asm("rsqrt.approx.ftz.f64 %0, %1;" : "=d"(y) : "d"(x));
    const double r = fma(-x * y, y, 1.0);
    const double p = fma(0.375, r, 0.5);
    return fma(y * r, p, y);
}

// Factor the nb x nb (nb <= 8) pivot block at (s0, s0) of A (shared memory, stride
// kPLD) in ONE thread's registers; 1/L_jj to sinv[s0 + j].  The pivot chain is
// written first in each step; the first non-positive / NaN pivot is reported once
// at the end (reading C8: only later columns can be contaminated).
__device__ __forceinline__ void factor_diag8(const DevPlan &d, double *A, double *sinv, int s0, int nb, int first_col) {
    constexpr int SB = 8;
    double a[SB][SB];
#pragma unroll
    for (int c = 0; c < SB; c++)
#pragma unroll
        for (int r = c; r < SB; r++) a[r][c] = (r < nb) ? A[(s0 + c) * kPLD + s0 + r] : (r == c ? 1.0 : 0.0);
    int bad = SB;
#pragma unroll
    for (int q = 0; q < SB; q++) {
        const double dq = a[q][q];
        if (!(dq > 0.0) && q < nb && bad == SB) bad = q;
        const double inv = rsqrt_nr(dq);
        if (q + 1 < SB) {   // the next pivot first
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
                if (r != q + 1) a[r][c] = fma(-a[r][q], a[c][q], a[r][c]);   // (q+1, q+1) was done first
    }
#pragma unroll
    for (int c = 0; c < SB; c++)
#pragma unroll
        for (int r = c; r < SB; r++)
            if (r < nb) A[(s0 + c) * kPLD + s0 + r] = a[r][c];
    if (bad < SB) atomicMin(d.failed, first_col + s0 + bad);
}

// C_IJ -= L_I L_J^T for the 8 x 8 blocks (I, J) of A over the 8 columns [s0, s0+8)
// (one warp, DMMA m8n8k4 twice)
__device__ __forceinline__ void upd_block8(double *A, int I, int J, int s0) {
    const int lane = threadIdx.x & 31, gq = lane >> 2, tq = lane & 3;
    double *Ci = A + I * 8 + gq;
    double c0 = Ci[(J * 8 + 2 * tq) * kPLD], c1 = Ci[(J * 8 + 2 * tq + 1) * kPLD];
#pragma unroll
    for (int kk = 0; kk < 2; kk++) {
        const double av = -Ci[(s0 + kk * 4 + tq) * kPLD];
        const double bv = A[J * 8 + gq + (s0 + kk * 4 + tq) * kPLD];
        dmma(c0, c1, av, bv);
    }
    Ci[(J * 8 + 2 * tq) * kPLD] = c0;
    Ci[(J * 8 + 2 * tq + 1) * kPLD] = c1;
}

// Same contract as panel_potrf, restructured for latency: per 8-column step the
// 8 x 8 pivot block is factored by one thread in registers (factor_diag8), the
// rows below solve it one thread per row, and the trailing lower 8 x 8 blocks are
// updated with DMMA (K = 8).  Look-ahead: warp 0 updates the next block column
// and its lane 0 factors the next pivot block while warps 1-3 update the rest.
__device__ __forceinline__ void panel_potrf_dmma(const DevPlan &d, double *A, double *sinv, int R, int we,
                                                 int first_col, int tl_task = 0) {
    constexpr int SB = 8;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int nrb = (R + 7) / 8, ncb = (we + 7) / 8;
    if (tid == 0) factor_diag8(d, A, sinv, 0, min(SB, we), first_col);
    __syncthreads();
#pragma unroll 1
    for (int st = 0; st < ncb; st++) {
        const int s0 = st * SB, nb = min(SB, we - s0);
        const int rb = s0 + nb;
        if (rb >= R) break;
        // rows [rb, R) against the factored pivot block st
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
                    for (int q2 = q + 1; q2 < SB; q2++)   // (q2 < nb: rows past the pivot block are other threads')
                        if (q2 < nb) x[q2] = fma(-x[q], A[(s0 + q) * kPLD + s0 + q2], x[q2]);
                }
            }
#pragma unroll
            for (int q = 0; q < SB; q++)
                if (q < nb) A[(s0 + q) * kPLD + r] = x[q];
        }
        __syncthreads();
        PANEL_TL(tl_task, 44 + 2 * st);
        if (st + 1 < ncb) {
            const int J1 = st + 1;
            if (warp == 0) {
                // the next pivot block only, then its factorization (the critical chain)
                upd_block8(A, J1, J1, s0);
                __syncwarp();
                if (lane == 0) factor_diag8(d, A, sinv, J1 * SB, min(SB, we - J1 * SB), first_col);
            } else {
                // by block column (tools/ubench/potrf_parts.cu: the trailing update of the
                // first steps 3373 -> 1835 cycles against block-by-block round robin):
                // column J's B fragments are loaded once and its row blocks follow one
                // another; columns go to warps 1-3 in zigzag order of decreasing length
                // (0 1 2 2 1 0 0 1 2 ...) for balance.  Every block gets the same two DMMAs
                // in the same order as upd_block8: bitwise-equal results.
                const int gq = lane >> 2, tq = lane & 3;
                for (int J = J1; J < ncb; J++) {
                    const int idx = J - J1, rnd = idx / 3, pos = idx - 3 * rnd;
                    if (((rnd & 1) ? 2 - pos : pos) != warp - 1) continue;
                    const double b0 = A[J * 8 + gq + (s0 + tq) * kPLD], b1 = A[J * 8 + gq + (s0 + 4 + tq) * kPLD];
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
            }
        }
        __syncthreads();
        PANEL_TL(tl_task, 45 + 2 * st);
    }
}

// X <- X L^-T for the 64 rows of Xs over wb columns; Ls = the wb x wb lower factor
// (identity-padded to a multiple of 8), inv = 1 / diag.  Each warp owns 16 rows and
// keeps them in registers as DMMA accumulators: per 8-column block, the block goes
// to shared memory, 16 lanes solve their rows over it (substitution, written back),
// and the warp applies it to the remaining column blocks with DMMA into the
// registers -- no shared-memory round trip per block update, so the updates of
// different blocks pipeline (same operations, same order per element as a
// shared-memory-resident update).  Xs holds the solved X on return.
__device__ __forceinline__ void panel_trsm(double *Xs, const double *Ls, const double *inv, int wb) {
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, gq = lane >> 2, tq = lane & 3;
    const int ncb = (wb + 7) / 8;
    const int row = warp * 16 + (lane & 15);
    double acc[2][8][2];
#pragma unroll
    for (int mb = 0; mb < 2; mb++)
#pragma unroll
        for (int nb = 0; nb < 8; nb++)
#pragma unroll
            for (int e = 0; e < 2; e++) acc[mb][nb][e] = Xs[warp * 16 + mb * 8 + gq + (nb * 8 + 2 * tq + e) * kPLD];
#pragma unroll
    for (int cb = 0; cb < 8; cb++) {
        if (cb >= ncb) break;
        const int c0 = cb * 8;
        // block cb of this warp's rows (updated by every earlier block) -> shared memory
#pragma unroll
        for (int mb = 0; mb < 2; mb++)
#pragma unroll
            for (int e = 0; e < 2; e++) Xs[warp * 16 + mb * 8 + gq + (c0 + 2 * tq + e) * kPLD] = acc[mb][cb][e];
        __syncwarp();
        if (lane < 16) {
            double xv[8];
#pragma unroll
            for (int q = 0; q < 8; q++) xv[q] = Xs[row + (c0 + q) * kPLD];
#pragma unroll
            for (int q = 0; q < 8; q++) {
                xv[q] *= inv[c0 + q];
#pragma unroll
                for (int q2 = q + 1; q2 < 8; q2++) xv[q2] -= xv[q] * Ls[(c0 + q2) + (c0 + q) * kPLD];
            }
#pragma unroll
            for (int q = 0; q < 8; q++) Xs[row + (c0 + q) * kPLD] = xv[q];
        }
        __syncwarp();
        // X[:, nbk] -= X[:, cb] L[nbk, cb]^T for nbk > cb, in registers
        double av[2][2];
#pragma unroll
        for (int mb = 0; mb < 2; mb++)
#pragma unroll
            for (int kk = 0; kk < 2; kk++) av[mb][kk] = -Xs[warp * 16 + mb * 8 + gq + (c0 + kk * 4 + tq) * kPLD];
#pragma unroll
        for (int nbk = 1; nbk < 8; nbk++) {
            if (nbk <= cb || nbk >= ncb) continue;
            const double b0 = Ls[(nbk * 8 + gq) + (c0 + tq) * kPLD], b1 = Ls[(nbk * 8 + gq) + (c0 + 4 + tq) * kPLD];
#pragma unroll
            for (int mb = 0; mb < 2; mb++) {
                dmma(acc[mb][nbk][0], acc[mb][nbk][1], av[mb][0], b0);
                dmma(acc[mb][nbk][0], acc[mb][nbk][1], av[mb][1], b1);
            }
        }
    }
    __syncthreads();   // callers read other warps' rows next
}

__device__ __forceinline__ void panel_publish(unsigned *flag, unsigned tag) {
    __threadfence();
    __syncthreads();
    if (threadIdx.x == 0) asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(flag), "r"(tag) : "memory");
}

__device__ __forceinline__ void panel_task(const DevPlan &d, const int32_t *__restrict__ tasks, int j0, int nbk,
                                           const int task) {
    extern __shared__ __align__(16) double psm[];
    double *ring = psm;                         // accumulate staging; the L_bb tile afterwards
    double *Xs = psm + kPanelRingWords;         // the tile being finished
    double *inv = Xs + 64 * kPLD;
    const int s = tasks[2 * task], c = tasks[2 * task + 1];
    const int k = d.sn_k[s], f = d.sn_f[s], ld = d.sn_ld[s];
    const int nb = min(nbk, (k - j0 + 63) / 64);
    const int r0 = j0 + 64 * c, rows = min(64, f - r0);
    double *__restrict__ Pn = d.L + d.L_off[s];
    unsigned *F = d.panel_flag + (int64_t)s * kPanelFlags;
    const unsigned tag = ((*d.epoch & 0xffffu) << 16) | (unsigned)(j0 / 64 + 1);   // as in k_leaf
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, gq = lane >> 2, tq = lane & 3;
    const bool band = c < nb;
    // the diagonal tile's accumulator: its 36 lower 8 x 8 blocks, 9 per warp
    // (block rows `warp` and 7 - warp), so the row's own products cost 144 DMMA per warp
    double dacc[9][2];
    if (band) {
        const int cols = min(64, k - r0);
#pragma unroll
        for (int t = 0; t < 9; t++) {
            const int I = t <= warp ? warp : 7 - warp, J = t <= warp ? t : t - warp - 1;
            const int i = I * 8 + gq;
#pragma unroll
            for (int e = 0; e < 2; e++) {
                const int j = J * 8 + 2 * tq + e;
                dacc[t][e] = (i < rows && j < cols) ? Pn[(r0 + i) + (int64_t)(r0 + j) * ld] : 0.0;
            }
        }
    }
    const int nsteps = min(c, nb);
#pragma unroll 1
    for (int b = 0; b < nsteps; b++) {
        const int cb0 = j0 + 64 * b, wb = min(64, k - cb0);
        double acc[4][4][2];
        PANEL_TL(task, 6 * b);
        panel_frag_load(acc, Pn, ld, r0, rows, cb0, wb);
        if (b > 0) {
            wait_flag(F + panel_tri(b, b - 1), tag);   // band tiles (b, 0..b-1) are final
            panel_tile_mma(acc, ring, Pn, ld, r0, rows, cb0, min(64, f - cb0), j0, 64 * b);
        }
        panel_frag_to_smem(acc, Xs);
        PANEL_TL(task, 6 * b + 1);
        wait_flag(F + panel_tri(b, b), tag);           // L_bb is final
        PANEL_TL(task, 6 * b + 2);
        {
            const double *__restrict__ D = Pn + (int64_t)cb0 * ld + cb0;
            for (int q = tid; q < 32 * 64; q += kPanelThreads) {
                const int rr = 2 * (q & 31), cc = q >> 5;
                const bool ok = cc < wb && rr < wb;
                cp_async16(ring + rr + cc * kPLD, ok ? D + rr + (int64_t)cc * ld : D, ok);
            }
            cp_async_commit();
            cp_async_wait<0>();
            __syncthreads();
            if (tid < 64) {
                if (tid >= wb) {
                    for (int cc = 0; cc < 64; cc++) ring[tid + cc * kPLD] = (cc == tid) ? 1.0 : 0.0;
                } else {
                    for (int cc = wb; cc < 64; cc++) ring[tid + cc * kPLD] = 0.0;
                }
            }
            __syncthreads();
            if (tid < 64) inv[tid] = __drcp_rn(ring[tid + tid * kPLD]);
            __syncthreads();
        }
        panel_trsm(Xs, ring, inv, wb);
        PANEL_TL(task, 6 * b + 3);
        for (int q = tid; q < 64 * 64; q += kPanelThreads) {
            const int i = q & 63, j = q >> 6;
            if (i < rows && j < wb) Pn[(r0 + i) + (int64_t)(cb0 + j) * ld] = Xs[i + j * kPLD];
        }
        if (band) {
            // the row's own product first: dacc -= X(c,b) X(c,b)^T (b < c < nb, so wb =
            // 64), from shared memory, while the stores above drain -- so the fence of
            // the publish below no longer waits for them (3.6 us -> the product's 2.4)
            const double *Xg = Xs + gq;
#pragma unroll 2
            for (int kk = 0; kk < 16; kk++) {
                const double *Xk = Xg + (kk * 4 + tq) * kPLD;
                const double a0 = -Xk[warp * 8], a1 = -Xk[(7 - warp) * 8];
                double bj[9];
#pragma unroll
                for (int t = 0; t < 9; t++) bj[t] = Xk[(t <= warp ? t : t - warp - 1) * 8];
#pragma unroll
                for (int t = 0; t < 9; t++) dmma(dacc[t][0], dacc[t][1], t <= warp ? a0 : a1, bj[t]);
            }
            PANEL_TL(task, 6 * b + 4);
            panel_publish(F + panel_tri(c, b), tag);   // X(c,b) is stored: band tile final (+ CTA barrier:
                                                       // Xs / ring are rewritten by the next step)
            PANEL_TL(task, 6 * b + 5);
        } else {
            __syncthreads();   // Xs / ring are rewritten by the next step
        }
    }
    if (band) {
        const int we = min(64, k - r0);
        __syncthreads();
#pragma unroll
        for (int t = 0; t < 9; t++) {
            const int I = t <= warp ? warp : 7 - warp, J = t <= warp ? t : t - warp - 1;
#pragma unroll
            for (int e = 0; e < 2; e++) Xs[I * 8 + gq + (J * 8 + 2 * tq + e) * kPLD] = dacc[t][e];
        }
        __syncthreads();
        PANEL_TL(task, 60);
        panel_potrf_dmma(d, Xs, inv, rows, we, d.sn_first[s] + r0, task);
        PANEL_TL(task, 61);
        for (int q = tid; q < 64 * 64; q += kPanelThreads) {
            const int i = q & 63, j = q >> 6;
            if (i < rows && j < we && i >= j) Pn[(r0 + i) + (int64_t)(r0 + j) * ld] = Xs[i + j * kPLD];
        }
        panel_publish(F + panel_tri(c, c), tag);
        PANEL_TL(task, 62);
    }
}

__global__ void __launch_bounds__(kPanelThreads, MF_PANEL_MINB) k_panel(DevPlan d, const int32_t *__restrict__ tasks,
                                                                         int j0, int nbk, unsigned *tk) {
    panel_task(d, tasks, j0, nbk, take_ticket(tk));
    drop_ticket(tk);
}

void launch_panel(const DevPlan &d, const int32_t *tasks, int64_t count, int j0, int nbk, unsigned *tk,
                  cudaStream_t st) {
    if (count <= 0) return;
    k_panel<<<(unsigned)count, kPanelThreads, kPanelSmem, st>>>(d, tasks, j0, nbk, tk);
}

void launch_trsm_panel(const DevPlan &d, const int32_t *tasks, int64_t count, int j0, int w, cudaStream_t st) {
    if (count <= 0) return;
    k_trsm_panel<<<(unsigned)count, kTrsmThreads, kTrsmSmem, st>>>(d, tasks, j0, w);
}

// ============================================================ DMMA Schur update
// The production tile shape (kTileM x kTileN in mf_plan.h); variants are
// benchmarked in tools/ubench/update_variants.cu.
// 64 x 64 tiles, BK 16, 3 stages, 4 CTAs / SM; staged by per-thread 16-byte
// cp.async (33.2 TF/s on M=N=8192, K=4096) or, for launches of many long-K waves,
// by the mbarrier + bulk-copy pipeline (33.8 TF/s there)
using UpdProd = UpdCfg<kTileM, kTileN, 16, 3, 2, 2, 4>;
// short-K launches: 2 stages (35 KB), 96 registers -> 5 CTAs / SM (20 warps) for
// more loads in flight on the latency-bound C gather and U store
using UpdLowK = UpdCfg<kTileM, kTileN, 16, 2, 2, 2, 5>;

void launch_update(const DevPlan &d, const GemmProb *probs, const TileTask *tiles, int64_t ntiles, double kavg,
                   cudaStream_t st) {
    if (ntiles <= 0) return;   // attributes were set by kernels_init()
    const UpdGather gv{d.child_ptr, d.child_list, d.sn_k, d.sn_f, d.U_off, d.relmap_ptr, d.relmap, d.ea_qs};
    // MF_UPD_BULK / MF_UPD_LOWK (A/B checks): 0 = never, 1 = every launch; unset = per launch
    static const int mode = [] {
        const char *e = getenv("MF_UPD_BULK");
        return e ? atoi(e) : -1;
    }();
    static const int lowk_mode = [] {
        const char *e = getenv("MF_UPD_LOWK");
        return e ? atoi(e) : -1;
    }();
    static const double bulk_min_tiles = [] {   // MF_UPD_BULK_TILES / MF_UPD_BULK_K: tuning overrides
        const char *e = getenv("MF_UPD_BULK_TILES");
        return e ? atof(e) : (double)kBulkMinTiles;
    }();
    static const double bulk_min_k = [] {
        const char *e = getenv("MF_UPD_BULK_K");
        return e ? atof(e) : kBulkMinK;
    }();
    bool bulk = (double)ntiles >= bulk_min_tiles && kavg >= bulk_min_k;
    if (mode >= 0) bulk = mode == 1;
    static const double lowk_max = [] {   // MF_UPD_LOWK_MAX: tuning override of kLowKMax
        const char *e = getenv("MF_UPD_LOWK_MAX");
        return e ? atof(e) : kLowKMax;
    }();
    bool lowk = !bulk && kavg < lowk_max;
    if (lowk_mode >= 0) lowk = !bulk && lowk_mode == 1;
#define MF_UPD_LAUNCH(C, V) k_update_t<C, V><<<(unsigned)ntiles, C::NT, C::SMEM, st>>>(d.L, d.U, probs, tiles, gv)
    if (bulk)
        MF_UPD_LAUNCH(UpdProd, true);
    else if (lowk)
        MF_UPD_LAUNCH(UpdLowK, false);
    else
        MF_UPD_LAUNCH(UpdProd, false);
#undef MF_UPD_LAUNCH
}

void launch_init_failed(int *failed, cudaStream_t st) { k_init_failed<<<1, 1, 0, st>>>(failed, reinterpret_cast<unsigned *>(failed + 1)); }

// Kernel attributes (dynamic shared memory above 48 KB), set once per device
// before any launch -- in particular before the factorization is captured
// into a CUDA graph.
int kernels_init() {
    cudaError_t e = cudaSuccess;
    e = cudaFuncSetAttribute(k_small_front<256>, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(k_trsm_panel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kTrsmSmem);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(k_leaf, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kTrsmSmem);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(k_panel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kPanelSmem);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(k_update_t<UpdProd, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)UpdProd::SMEM);
    for (auto fn : {k_update_t<UpdProd, true>})
        if (e == cudaSuccess) e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)UpdProd::SMEM);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(k_update_t<UpdLowK, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                 (int)UpdLowK::SMEM);
    if (e == cudaSuccess) e = oz_set_attr<3>();
    if (e == cudaSuccess) e = oz_set_attr<4>();
    if (e == cudaSuccess) e = oz_set_attr<5>();
    if (e == cudaSuccess) e = oz_set_attr<6>();
    if (e == cudaSuccess) e = oz_set_attr<7>();
    if (e == cudaSuccess) e = oz_set_attr<8>();
    return e == cudaSuccess ? 0 : -1;
}

// Ozaki-scheme Schur update of one KC_UPDATE launch (S = slices, 3..8)
void launch_update_oz(const DevPlan &d, const GemmProb *probs, const OzProb *oprobs, const int32_t *split,
                      int64_t nsplit, const OzTile *tiles, int64_t ntiles, int8_t *scratch, int32_t *expo,
                      int64_t expo_words, int S, int wide, cudaStream_t st) {
    const UpdGather gv{d.child_ptr, d.child_list, d.sn_k, d.sn_f, d.U_off, d.relmap_ptr, d.relmap, d.ea_qs};
    switch (S) {
        case 3: launch_oz<3>(d.L, d.U, probs, oprobs, split, nsplit, tiles, ntiles, scratch, expo, expo_words, st, gv, wide); break;
        case 4: launch_oz<4>(d.L, d.U, probs, oprobs, split, nsplit, tiles, ntiles, scratch, expo, expo_words, st, gv, wide); break;
        case 5: launch_oz<5>(d.L, d.U, probs, oprobs, split, nsplit, tiles, ntiles, scratch, expo, expo_words, st, gv, wide); break;
        case 6: launch_oz<6>(d.L, d.U, probs, oprobs, split, nsplit, tiles, ntiles, scratch, expo, expo_words, st, gv, wide); break;
        case 7: launch_oz<7>(d.L, d.U, probs, oprobs, split, nsplit, tiles, ntiles, scratch, expo, expo_words, st, gv, wide); break;
        default: launch_oz<8>(d.L, d.U, probs, oprobs, split, nsplit, tiles, ntiles, scratch, expo, expo_words, st, gv, wide); break;
    }
}

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
// Small supernodes (f <= kSolveSmallMax): one WARP per front, the front vector in
// shared memory, lane l holding rows l + 32 t; the L column of the next step is
// loaded while the current one is applied (register double buffer).
constexpr int kSmallSolveWarps = 8, kSmallSolveR = kSolveSmallMax / 32;
__device__ __forceinline__ void small_col_load(const double *__restrict__ col, int lo, int f, double (&c)[kSmallSolveR]) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int t = 0; t < kSmallSolveR; t++) {
        const int i = lane + 32 * t;
        c[t] = (i >= lo && i < f) ? col[i] : 0.0;
    }
}
__global__ void __launch_bounds__(32 * kSmallSolveWarps) k_fwd_solve(DevPlan d, const int32_t *__restrict__ list,
                                                                     int count, double *__restrict__ y) {
    __shared__ double vsm[kSmallSolveWarps][kSolveSmallMax];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int idx = blockIdx.x * kSmallSolveWarps + warp;
    if (idx >= count) return;
    const int s = list[idx];
    const int k = d.sn_k[s], f = d.sn_f[s], ld = d.sn_ld[s], first = d.sn_first[s];
    const double *__restrict__ P = d.L + d.L_off[s];
    double *__restrict__ vs = vsm[warp];
    double cur[kSmallSolveR], nxt[kSmallSolveR];
    small_col_load(P, 1, f, cur);   // column 0 (rows below the pivot), in flight during the gather
    for (int i = lane; i < f; i += 32) vs[i] = i < k ? y[first + i] : 0.0;
    __syncwarp();
    for (int q = d.child_ptr[s]; q < d.child_ptr[s + 1]; q++) {
        const int c = d.child_list[q];
        const int kc = d.sn_k[c], mc = d.sn_f[c] - kc;
        const int32_t *__restrict__ rel = d.relmap + d.relmap_ptr[c];
        const double *__restrict__ vc = d.fv + d.fv_off[c] + kc;
        for (int p = lane; p < mc; p += 32) vs[rel[p]] += vc[p];   // rel is injective: no conflicts
        __syncwarp();
    }
    for (int j = 0; j < k; j++) {
        if (j + 1 < k) small_col_load(P + (int64_t)(j + 1) * ld, j + 2, f, nxt);
        const double xj = vs[j] / P[j + (int64_t)j * ld];
        __syncwarp();   // every lane read vs[j]
        if (lane == 0) {
            y[first + j] = xj;
            vs[j] = xj;
        }
#pragma unroll
        for (int t = 0; t < kSmallSolveR; t++) {
            const int i = lane + 32 * t;
            if (i > j && i < f) vs[i] = fma(-cur[t], xj, vs[i]);
        }
        __syncwarp();
#pragma unroll
        for (int t = 0; t < kSmallSolveR; t++) cur[t] = nxt[t];
    }
    double *__restrict__ v = d.fv + d.fv_off[s];
    for (int i = k + lane; i < f; i += 32) v[i] = vs[i];   // the update vector the parent gathers
}

__global__ void __launch_bounds__(32 * kSmallSolveWarps) k_bwd_solve(DevPlan d, const int32_t *__restrict__ list,
                                                                     int count, double *__restrict__ y,
                                                                     const int32_t *__restrict__ sn_rows,
                                                                     const int64_t *__restrict__ sn_rowptr) {
    __shared__ double vsm[kSmallSolveWarps][kSolveSmallMax];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const int idx = blockIdx.x * kSmallSolveWarps + warp;
    if (idx >= count) return;
    const int s = list[idx];
    const int k = d.sn_k[s], f = d.sn_f[s], ld = d.sn_ld[s], first = d.sn_first[s];
    const double *__restrict__ P = d.L + d.L_off[s];
    const int32_t *__restrict__ R = sn_rows + sn_rowptr[s];
    double *__restrict__ vs = vsm[warp];
    double cur[kSmallSolveR], nxt[kSmallSolveR];
    if (k > 0) small_col_load(P + (int64_t)(k - 1) * ld, k, f, cur);
    for (int i = lane; i < f; i += 32) vs[i] = i < k ? y[first + i] : y[R[i]];   // ancestors are final
    __syncwarp();
    for (int j = k - 1; j >= 0; j--) {
        if (j > 0) small_col_load(P + (int64_t)(j - 1) * ld, j, f, nxt);
        double part = 0.0;
#pragma unroll
        for (int t = 0; t < kSmallSolveR; t++) {
            const int i = lane + 32 * t;
            if (i > j && i < f) part = fma(cur[t], vs[i], part);
        }
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) part += __shfl_xor_sync(0xffffffffu, part, o);
        const double xj = (vs[j] - part) / P[j + (int64_t)j * ld];
        __syncwarp();
        if (lane == 0) {
            vs[j] = xj;
            y[first + j] = xj;
        }
        __syncwarp();
#pragma unroll
        for (int t = 0; t < kSmallSolveR; t++) cur[t] = nxt[t];
    }
}

// ---- dataflow solve hand-off: every published value is its own flag.  A slot that
// is not yet written holds kSolvePending, a signaling-NaN bit pattern that no fp64
// arithmetic produces (NaN results are quiet), so a consumer polls the value itself
// (one L2 round trip; no flag word, no fence on the producer).  k_fsolve_init sets the
// forward block entries of y pending, k_bsolve_init the backward x slots.
constexpr unsigned long long kSolvePending = 0x7ff40000df5e0001ull;
__device__ __forceinline__ double ld_relaxed_f64(const double *p) {
    double v;
    asm volatile("ld.relaxed.gpu.global.f64 %0, [%1];" : "=d"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ double wait_value(const double *p) {
    double v;
    while ((unsigned long long)__double_as_longlong(v = ld_relaxed_f64(p)) == kSolvePending) {
    }
    return v;
}
__device__ __forceinline__ double pending_value() { return __longlong_as_double((long long)kSolvePending); }
__global__ void k_fill_pending(double *__restrict__ p, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        p[i] = pending_value();
}
void launch_fill_pending(double *p, int64_t n, cudaStream_t st) {
    if (n > 0) k_fill_pending<<<(unsigned)std::min<int64_t>((n + 255) / 256, 2048), 256, 0, st>>>(p, n);
}

#ifndef MF_DF_BUF
#define MF_DF_BUF 2
#endif
constexpr int kSW = 64, kSLD = 65;   // solve block width and smem leading dimension
constexpr int kDfThreads = 256;      // dataflow solve CTA: 64 rows x 4 groups of 16 columns
constexpr int kDfRB = 64;            // rows per forward task / per backward slab
constexpr int kDfBuf = MF_DF_BUF;    // register ring: blocks (forward) / slabs (backward) in flight
#ifndef MF_YPRE
#define MF_YPRE 8
#endif
constexpr int kYPre = MF_YPRE;       // forward: block solutions read per batch (a multiple of 4)
static_assert(kYPre * 64 % 256 == 0, "kYPre blocks of 64 values over 256 threads");
constexpr int kInitRows = kSolveInitRows;   // rows of a front vector per init task
constexpr int kBsSegSlabs = kSolveSegSlabs;  // backward: tail slabs per segment task

// First p in [0, n) with rel[p] >= key (rel increasing; n if none), by the whole CTA
// of kSolveThreads in 256-way rounds (two dependent loads for n <= 65536 instead of
// a log2(n) chain).  Uniform call.
__device__ __forceinline__ int lower_bound_cta(const int32_t *__restrict__ rel, int n, int key) {
    const int t = threadIdx.x;
    int lo = 0, hi = n;   // the answer lies in [lo, hi]
    while (hi - lo > kSolveThreads) {
        const int len = hi - lo;
        const int bt = lo + (int)((int64_t)t * len / kSolveThreads);
        const int c = __syncthreads_count(t > 0 && __ldg(rel + bt - 1) < key);
        hi = lo + (int)((int64_t)(c + 1) * len / kSolveThreads);
        lo = lo + (int)((int64_t)c * len / kSolveThreads);
    }
    const int p = lo + t;
    return lo + __syncthreads_count(p < hi && __ldg(rel + p) < key);
}

// ---- large supernodes: v = [y(cols); 0] + the children's update vectors, one task
// per (supernode, 2048-row part); a part finds each child's entries that land in it
// by binary search (rel is increasing), children in a fixed order: deterministic.
__device__ __forceinline__ void fsolve_init_task(const DevPlan &d, const int32_t *__restrict__ tasks,
                                                 double *__restrict__ y, const int task) {
    const int s = tasks[2 * task], part = tasks[2 * task + 1];
    const int k = d.sn_k[s], f = d.sn_f[s], first = d.sn_first[s];
    const int p0 = part * kInitRows, p1 = min(f, p0 + kInitRows);
    double *__restrict__ v = d.fv + d.fv_off[s];
    for (int i = p0 + threadIdx.x; i < p1; i += kSolveThreads) {
        v[i] = i < k ? y[first + i] : 0.0;
        if (i < k) y[first + i] = pending_value();   // x of this column: published by k_fsolve_df
    }
    for (int q = d.child_ptr[s]; q < d.child_ptr[s + 1]; q++) {
        __syncthreads();
        const int c = d.child_list[q];
        const int kc = d.sn_k[c], mc = d.sn_f[c] - kc;
        const int32_t *__restrict__ rel = d.relmap + d.relmap_ptr[c];
        const double *__restrict__ vc = d.fv + d.fv_off[c] + kc;
        const bool whole = p0 == 0 && p1 == f;   // one part: no search
        const int lo = whole ? 0 : lower_bound_cta(rel, mc, p0), hi = whole ? mc : lower_bound_cta(rel, mc, p1);
        for (int p = lo + threadIdx.x; p < hi; p += kSolveThreads) v[rel[p]] += vc[p];
    }
}

__global__ void __launch_bounds__(kSolveThreads) k_fsolve_init(DevPlan d, const int32_t *__restrict__ tasks,
                                                               double *__restrict__ y) {
    fsolve_init_task(d, tasks, y, blockIdx.x);
}
void launch_fsolve_init(const DevPlan &d, const int32_t *tasks, int64_t count, double *y, cudaStream_t st) {
    if (count > 0) k_fsolve_init<<<(unsigned)count, kSolveThreads, 0, st>>>(d, tasks, y);
}

// The init tasks of a level with few of them run in the level's dataflow launch
// (SolveLaunch.off2; levels of many small fronts keep a launch of their own, whose
// light CTAs cover them in fewer waves than the dataflow kernel's):
// they take the lowest tickets, then count themselves done in tk[2]; every dataflow
// task of the launch waits for that count (thread 0 polls) before it touches a front
// vector, a y / x slot of the level or a partial -- its L loads are issued before.
__device__ __forceinline__ void init_done(unsigned *cnt) {
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        atomicAdd(cnt, 1u);
    }
}
__device__ __forceinline__ void wait_inits(const unsigned *cnt, int ninit) {
    if (ninit <= 0) return;
    if (threadIdx.x == 0) {
        unsigned v;
        do {
            asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(cnt) : "memory");
        } while (v < (unsigned)ninit);
    }
    __syncthreads();
}

// v(k:f) = x(R(k:f)) (ancestors are final); the backward x slots of the pivot columns pending
__device__ __forceinline__ void bsolve_init_task(const DevPlan &d, const int32_t *__restrict__ tasks,
                                                 const double *__restrict__ y, const int32_t *__restrict__ sn_rows,
                                                 const int64_t *__restrict__ sn_rowptr, const int task) {
    const int s = tasks[2 * task], part = tasks[2 * task + 1];
    const int k = d.sn_k[s], f = d.sn_f[s];
    const int p0 = part * kInitRows, p1 = min(f, p0 + kInitRows);
    double *__restrict__ v = d.fv + d.fv_off[s];
    double *__restrict__ xp = d.df_parts + d.df_part_off[s];
    const int32_t *__restrict__ R = sn_rows + sn_rowptr[s];
    for (int i = p0 + threadIdx.x; i < p1; i += kSolveThreads) {
        if (i >= k) v[i] = y[R[i]];
        else xp[i] = pending_value();
    }
}
__global__ void __launch_bounds__(kSolveThreads) k_bsolve_init(DevPlan d, const int32_t *__restrict__ tasks,
                                                               const double *__restrict__ y,
                                                               const int32_t *__restrict__ sn_rows,
                                                               const int64_t *__restrict__ sn_rowptr) {
    bsolve_init_task(d, tasks, y, sn_rows, sn_rowptr, blockIdx.x);
}
void launch_bsolve_init(const DevPlan &d, const int32_t *tasks, int64_t count, const double *y,
                        const int32_t *sn_rows, const int64_t *sn_rowptr, cudaStream_t st) {
    if (count > 0) k_bsolve_init<<<(unsigned)count, kSolveThreads, 0, st>>>(d, tasks, y, sn_rows, sn_rowptr);
}

// ---- solve setup: inv(L_bb) of every 64 x 64 diagonal block of the dataflow-solved
// supernodes (once per factorization, by the first solve), so the block chains of the
// sweeps below apply a 64 x 64 matrix-vector product (x_b = inv(L_bb) t_b, all threads)
// instead of a 64-step substitution on one warp.  One CTA of 64 threads per block;
// thread j forms column j of the inverse by forward substitution, L_bb in shared memory.
// Stored column-major 64 x 64 (zero above the diagonal; a ragged last block is
// extended by the identity).  Power-of-two pivots give exact inverses (the
// manufactured factors stay exact through the solve).
__global__ void __launch_bounds__(64) k_diag_inv(DevPlan d, const int32_t *__restrict__ tasks, int w) {
    __shared__ double Ls[kSW * kSLD];
    const int s = tasks[2 * blockIdx.x], b = tasks[2 * blockIdx.x + 1];
    const int k = d.sn_k[s], ld = d.sn_ld[s];
    const int j0 = b * w, we = min(w, k - j0);   // block b of width w (<= 64) in a 64 x 64 slot
    const double *__restrict__ D = d.L + d.L_off[s] + (int64_t)j0 * ld + j0;
    const int j = threadIdx.x;
    for (int q = 0; q < kSW; q++)   // row j, column q of the (identity-extended) block
        Ls[j + q * kSLD] = (j < we && q < we) ? (q <= j ? D[j + (int64_t)q * ld] : 0.0) : (j == q ? 1.0 : 0.0);
    __syncthreads();
    // column j of inv(L): x_i = (delta_ij - sum_{q < i} L_iq x_q) / L_ii, x_q = 0 for q < j
    // (fully unrolled: x stays in registers; the terms with q < j add exact zeros)
    double x[kSW];
#pragma unroll
    for (int i = 0; i < kSW; i++) {
        double t = (i == j) ? 1.0 : 0.0;
#pragma unroll
        for (int q = 0; q < i; q++) t = fma(-Ls[i + q * kSLD], x[q], t);
        x[i] = (i >= j) ? t / Ls[i + i * kSLD] : 0.0;
    }
    __syncthreads();
#pragma unroll
    for (int i = 0; i < kSW; i++) Ls[i + j * kSLD] = x[i];   // column j
    __syncthreads();
    double *__restrict__ out = d.dinv + d.dinv_off[s] + (int64_t)b * kSW * kSW;
    for (int q = 0; q < kSW; q++) out[j + q * kSW] = Ls[j + q * kSLD];   // coalesced
}
void launch_diag_inv(const DevPlan &d, const int32_t *tasks, int64_t count, int w, cudaStream_t st) {
    if (count > 0) k_diag_inv<<<(unsigned)count, 64, 0, st>>>(d, tasks, w);
}

// ---- dataflow solves: one launch per level for all its large supernodes.  A CTA is
// 64 rows x 4 column groups (thread (i, g) = row i, columns [16 g, 16 g + 16) of a
// 64-column block); the L data streams through a ring of kDfBuf register blocks, issued
// ahead of the values they multiply, so a task's only waits are for values.
//
// Forward (L y = b), row-oriented: task = 64 rows [r0, r0 + 64) of front s.  For
// every column block b reaching the rows: wait for y_b (value by value), then each
// thread adds its 16 products to a private partial sum.  The block the rows own
// (j0 >= r0: the diagonal block) is solved in place: the partials are reduced into
// t_b, x_b = inv(L_bb) t_b (all 256 threads, inverse staged in shared memory at task
// start, off the chain) and published into y.  Rows >= k keep v for the parent.
// The chain per block is one value hand-off + one 64 x 64 product + the inverse.
__device__ __forceinline__ void fsolve_load(const double *__restrict__ P, int ld, int k, int w, int r, bool rok,
                                            int b, double (&Lb)[16]) {
    const int g = threadIdx.x >> 6, j0 = b * w, we = min(w, k - j0);
    const bool ok = rok && r >= j0 + we;   // the diagonal block's own rows take no part
#pragma unroll
    for (int u = 0; u < 16; u++) {
        const int c = 16 * g + u;
        Lb[u] = (ok && c < we) ? P[(int64_t)(j0 + c) * ld + r] : 0.0;
    }
}
template <int NBUF>
__device__ __forceinline__ void fsolve_rows_task(const DevPlan &d, const int32_t *__restrict__ tasks, int w,
                                                 double *__restrict__ y, const int task, const unsigned *cnt,
                                                 int ninit) {
    __shared__ double Ms[kSW * kSLD];   // inv(L_bb) of the owned block: element (q, c) at q + c kSLD
    __shared__ double ys[2][kSW];
    __shared__ double yp[kYPre][kSW];   // solutions of the next kYPre blocks above, read in one batch
    __shared__ double red[4][kSW];
    __shared__ double vrow[kSW];
    const int s = tasks[2 * task], rb = tasks[2 * task + 1];
    const int k = d.sn_k[s], f = d.sn_f[s], ld = d.sn_ld[s], first = d.sn_first[s];
    const double *__restrict__ P = d.L + d.L_off[s];
    const double *__restrict__ Dinv = d.dinv + d.dinv_off[s];
    double *__restrict__ v = d.fv + d.fv_off[s];
    const int tid = threadIdx.x, i = tid & 63, g = tid >> 6;
    const int r0 = rb * kDfRB, r = r0 + i;
    const bool rok = r < f;
    const int nbr = (min(k, r0 + kDfRB) + w - 1) / w;   // column blocks reaching these rows
    const int bown = r0 < k ? r0 / w : nbr;              // first owned block (w divides 64)
    auto load_inv = [&](int b) {
        const double *__restrict__ M = Dinv + (int64_t)b * kSW * kSW;
        for (int q = tid; q < kSW * kSW; q += kDfThreads) Ms[(q & 63) + (q >> 6) * kSLD] = __ldg(M + q);
    };
    if (bown < nbr) load_inv(bown);
    double Lb[NBUF][16];
#pragma unroll
    for (int q = 0; q < NBUF; q++)
        if (q < nbr) fsolve_load(P, ld, k, w, r, rok, q, Lb[q]);
    wait_inits(cnt, ninit);   // v and the level's y slots are set by the fused init tasks
    if (tid < kSW) vrow[tid] = rok ? v[r] : 0.0;
    double acc = 0.0;
    for (int b0 = 0; b0 < nbr; b0 += NBUF) {
#pragma unroll
        for (int q = 0; q < NBUF; q++) {
            const int b = b0 + q;
            if (b >= nbr) break;
            const int j0 = b * w, we = min(w, k - j0);
            double *yb = ys[b & 1];
            const bool owned = j0 >= r0;
            if (b % kYPre == 0) {
                // one batch of loads for the solutions of blocks b .. b + kYPre - 1 above the
                // task's rows: a task walking blocks published long ago pays one L2 round
                // trip per batch instead of one per block (the walk, not the hand-off, set
                // the pace of the long chains); a slot still pending is polled at its block
#pragma unroll
                for (int t = 0; t < kYPre * kSW / kDfThreads; t++) {
                    const int qq = (tid + t * kDfThreads) >> 6, e = tid & 63, bb = b + qq;
                    double val = pending_value();
                    if (bb < nbr && bb * w < r0 && e < min(w, k - bb * w)) val = ld_relaxed_f64(y + first + bb * w + e);
                    yp[qq][e] = val;
                }
                __syncthreads();
            }
            if (owned) {   // t_b = v - partials (rows of the block), x_b = inv(L_bb) t_b
                red[g][i] = acc;
                acc = 0.0;
                __syncthreads();
                if (tid < kSW) vrow[i] -= (red[0][i] + red[1][i]) + (red[2][i] + red[3][i]);
                __syncthreads();
                double a = 0.0;
#pragma unroll
                for (int u = 0; u < 16; u++) {
                    const int c = 16 * g + u;
                    a = fma(Ms[i + c * kSLD], c < we ? vrow[j0 - r0 + c] : 0.0, a);
                }
                red[g][i] = a;
                __syncthreads();
                if (tid < kSW) {
                    const double x = (red[0][i] + red[1][i]) + (red[2][i] + red[3][i]);
                    if (i < we) {
                        __stcg(y + first + j0 + i, x);   // published: the value is its flag
                        vrow[j0 - r0 + i] = x;
                    }
                    yb[i] = i < we ? x : 0.0;
                }
            } else if (tid < kSW) {   // a block above: its solution, value by value
                double val = 0.0;
                if (tid < we) {
                    val = yp[b % kYPre][tid];
                    if ((unsigned long long)__double_as_longlong(val) == kSolvePending) val = wait_value(y + first + j0 + tid);
                }
                yb[tid] = val;
            }
            __syncthreads();
            if (owned && b + 1 < nbr && (b + 1) * w < r0 + kDfRB) load_inv(b + 1);   // w < 64: the next owned block
#pragma unroll
            for (int u = 0; u < 16; u++) acc = fma(Lb[q][u], yb[16 * g + u], acc);
            if (b + NBUF < nbr) fsolve_load(P, ld, k, w, r, rok, b + NBUF, Lb[q]);
        }
    }
    red[g][i] = acc;
    __syncthreads();
    if (tid < kSW && rok && r >= k) v[r] = vrow[i] - ((red[0][i] + red[1][i]) + (red[2][i] + red[3][i]));
}
// NBUF = ring depth, MINB = CTAs / SM (tools/gpu/job_df_variants.sh: c5 solve 8.26 ms at <4, 1>,
// 7.12 at <2, 2>); levels of small fronts take the shallow ring at 3 CTAs / SM
template <int NBUF, int MINB>
__global__ void __launch_bounds__(kDfThreads, MINB) k_fsolve_df(DevPlan d, const int32_t *__restrict__ tasks, int w,
                                                                double *__restrict__ y, unsigned *tk,
                                                                const int32_t *__restrict__ itasks, int ninit) {
    static_assert(kDfThreads == kSolveThreads, "init tasks run in dataflow CTAs");
    const int t = take_ticket(tk);
    if (t < ninit) {
        fsolve_init_task(d, itasks, y, t);
        init_done(tk + 2);
    } else {
        fsolve_rows_task<NBUF>(d, tasks, w, y, t - ninit, tk + 2, ninit);
    }
    drop_ticket(tk);
}

// Backward (L^T x = y), column-oriented: task = column block b of front s.  Its
// dot products L(r, b)^T x_r run over the rows below the block in 64-row slabs:
// first the rows >= k (final, from the ancestors), then the pivot rows from the top
// block down (each thread waits for its own row's x, published by the task of that
// block).  16 column partials per thread, reduced over the 64 rows at the end
// (butterfly, fixed order); x_b = inv(L_bb)^T (y_b - dot) is published into y and
// into the front's x slots.  The chain per block is one value hand-off + one slab +
// the reduction and the inverse.
__device__ __forceinline__ void bsolve_load(const double *__restrict__ P, int ld, int f, int j0, int we, int rlo,
                                            int r, double (&Lb)[16]) {
    const int g = threadIdx.x >> 6;
    const bool ok = r >= rlo && r < f;
#pragma unroll
    for (int u = 0; u < 16; u++) {
        const int c = 16 * g + u;
        Lb[u] = (ok && c < we) ? P[(int64_t)(j0 + c) * ld + r] : 0.0;
    }
}
// Butterfly reduce-scatter over the warp: 16 values per lane in; lane l ends with the
// warp sum of value (l >> 1) & 15 in p[0] (16 shuffles).
__device__ __forceinline__ void warp_reduce_scatter16(double (&p)[16]) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int st = 0; st < 4; st++) {
        const int half = 8 >> st, off = 16 >> st;
        const bool up = (lane & off) != 0;
#pragma unroll
        for (int j = 0; j < half; j++) {
            const double send = up ? p[j] : p[j + half];
            const double keep = up ? p[j + half] : p[j];
            p[j] = keep + __shfl_xor_sync(0xffffffffu, send, off);
        }
    }
    p[0] += __shfl_xor_sync(0xffffffffu, p[0], 1);
}
template <int NBUF>
__device__ __forceinline__ void bsolve_cols_task(const DevPlan &d, const int32_t *__restrict__ tasks, int w,
                                                 double *__restrict__ y, const int task, const unsigned *cnt,
                                                 int ninit) {
    __shared__ double Ms[kSW * kSLD];   // inv(L_bb)^T: element (q, c) = inv(c, q) at q + c kSLD
    __shared__ double red[8][16];
    __shared__ double tv[kSW];
    __shared__ double rx[4][kSW];
    const int s = tasks[2 * task], b = tasks[2 * task + 1] & 0xffff, seg = tasks[2 * task + 1] >> 16;
    const int k = d.sn_k[s], f = d.sn_f[s], ld = d.sn_ld[s], first = d.sn_first[s];
    const double *__restrict__ P = d.L + d.L_off[s];
    const double *__restrict__ v = d.fv + d.fv_off[s];
    double *__restrict__ xp = d.df_parts + d.df_part_off[s];
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5, i = tid & 63, g = tid >> 6;
    const int j0 = b * w, we = min(w, k - j0), rlo = j0 + we;   // rows below the block
    // slabs of 64 rows: the pure tail ones (rows >= k, from slab T0 on), then the pivot
    // ones from slab ktop (holding row k - 1; it may also hold rows >= k) down to the
    // one holding row rlo.  A tall tail is cut into segments of kBsSegSlabs slabs, each
    // a task of its own (seg >= 1, lower tickets, never waits) that publishes the 64
    // column partials of its rows; the chain task (seg = 0) then streams no tail.
    const int ktop = (k - 1) / kDfRB, T0 = ktop + 1, nsl = (f + kDfRB - 1) / kDfRB;
    const int ntail = max(0, nsl - T0), nseg = ntail > kBsSegSlabs ? (ntail + kBsSegSlabs - 1) / kBsSegSlabs : 0;
    double *__restrict__ segp = nseg ? d.df_seg + d.df_seg_off[s] + (int64_t)b * nseg * kSW : nullptr;
    int t0, nt, np;
    if (seg > 0) {
        t0 = T0 + (seg - 1) * kBsSegSlabs;
        nt = min(kBsSegSlabs, nsl - t0);
        np = 0;
    } else {
        t0 = T0;
        nt = nseg ? 0 : ntail;
        np = max(0, ktop - rlo / kDfRB + 1);
    }
    double yb = 0.0;
    if (seg == 0) {
        const double *__restrict__ M = d.dinv + d.dinv_off[s] + (int64_t)b * kSW * kSW;
        for (int q = tid; q < kSW * kSW; q += kDfThreads) Ms[(q >> 6) + (q & 63) * kSLD] = __ldg(M + q);
        if (tid < we) yb = y[first + j0 + tid];   // forward result of the block (this task rewrites it)
    }
    const int ns = nt + np;
    auto slab_row = [&](int q) { return (q < nt ? t0 + q : ktop - (q - nt)) * kDfRB + i; };
    double Lb[NBUF][16];
#pragma unroll
    for (int q = 0; q < NBUF; q++)
        if (q < ns) bsolve_load(P, ld, f, j0, we, rlo, slab_row(q), Lb[q]);
    wait_inits(cnt, ninit);   // v and the x slots of the level are set by the fused init tasks
    // the tail segments' partials (lower tickets: they are done or nearly so) -- read
    // now, while the chain is still above this block, not on its critical path
    double segsum = 0.0;
    if (seg == 0 && tid < we)
        for (int q = 0; q < nseg; q++) {
            double *pq = segp + (int64_t)q * kSW + tid;
            segsum += wait_value(pq);
            __stcg(pq, pending_value());   // re-armed for the next solve (this task is its only reader)
        }
    double acc[16];
#pragma unroll
    for (int u = 0; u < 16; u++) acc[u] = 0.0;
    // the x values of XP slabs (this thread's row in each) are loaded in one batch: a
    // task walking rows whose x was published long ago pays one L2 round trip per
    // batch instead of one per slab; a value still pending is polled at its slab
    constexpr int XP = NBUF == 1 ? 1 : (4 % NBUF == 0 ? 4 : NBUF);   // (NBUF = 1 at 3 CTAs / SM: no room)
    for (int q0 = 0; q0 < ns; q0 += XP) {
        double xq[XP];
#pragma unroll
        for (int t = 0; t < XP; t++) {
            const int sq = q0 + t, r = slab_row(sq);
            xq[t] = (sq < ns && r >= rlo && r < f) ? (r >= k ? v[r] : ld_relaxed_f64(xp + r)) : 0.0;
        }
#pragma unroll
        for (int t = 0; t < XP; t++) {
            const int sq = q0 + t, q = t % NBUF;   // (q0 is a multiple of NBUF)
            if (sq >= ns) break;
            const int r = slab_row(sq);
            double xr = xq[t];
            if ((unsigned long long)__double_as_longlong(xr) == kSolvePending) xr = wait_value(xp + r);
#pragma unroll
            for (int u = 0; u < 16; u++) acc[u] = fma(Lb[q][u], xr, acc[u]);
            if (sq + NBUF < ns) bsolve_load(P, ld, f, j0, we, rlo, slab_row(sq + NBUF), Lb[q]);
        }
    }
    warp_reduce_scatter16(acc);   // lane l: value (l >> 1) & 15 over this warp's 32 rows
    if ((lane & 1) == 0) red[warp][lane >> 1] = acc[0];
    __syncthreads();
    if (seg > 0) {   // a tail segment: publish its column partials
        if (tid < we) {
            const int gc = tid >> 4, u = tid & 15;
            __stcg(segp + (int64_t)(seg - 1) * kSW + tid, red[2 * gc][u] + red[2 * gc + 1][u]);
        }
        return;
    }
    if (tid < kSW) {   // column c = 16 g' + u': the two warps of group g', then the tail segments in order
        const int gc = tid >> 4, u = tid & 15;
        tv[tid] = tid < we ? yb - ((red[2 * gc][u] + red[2 * gc + 1][u]) + segsum) : 0.0;
    }
    __syncthreads();
    double a = 0.0;
#pragma unroll
    for (int u = 0; u < 16; u++) a = fma(Ms[i + (16 * g + u) * kSLD], tv[16 * g + u], a);
    rx[g][i] = a;
    __syncthreads();
    if (tid < we) {
        const double x = (rx[0][i] + rx[1][i]) + (rx[2][i] + rx[3][i]);
        y[first + j0 + i] = x;
        __stcg(xp + j0 + i, x);   // published: the value is its flag
    }
}
template <int NBUF, int MINB>
__global__ void __launch_bounds__(kDfThreads, MINB) k_bsolve_df(DevPlan d, const int32_t *__restrict__ tasks, int w,
                                                                double *__restrict__ y, unsigned *tk,
                                                                const int32_t *__restrict__ itasks, int ninit,
                                                                const int32_t *__restrict__ sn_rows,
                                                                const int64_t *__restrict__ sn_rowptr) {
    const int t = take_ticket(tk);
    if (t < ninit) {
        bsolve_init_task(d, itasks, y, sn_rows, sn_rowptr, t);
        init_done(tk + 2);
    } else {
        bsolve_cols_task<NBUF>(d, tasks, w, y, t - ninit, tk + 2, ninit);
    }
    drop_ticket(tk);
}

// MF_DF_VARIANT (tuning A/B): deep ring 0 = <2 blocks, 2 CTAs/SM>, 1 = <3, 2>, 2 = <4, 1>, 3 = <2, 3>
static int df_variant() {
    static const int v = [] {
        const char *e = getenv("MF_DF_VARIANT");
        return e ? atoi(e) : 0;
    }();
    return v;
}
void launch_fsolve_df(const DevPlan &d, const int32_t *tasks, int64_t count, const int32_t *itasks, int64_t ninit,
                      int w, int deep, double *y, unsigned *tk, cudaStream_t st) {
    if (count <= 0) return;
    const unsigned n = (unsigned)(count + ninit);
    const int ni = (int)ninit;
    if (!deep)
        k_fsolve_df<1, 3><<<n, kDfThreads, 0, st>>>(d, tasks, w, y, tk, itasks, ni);
    else if (df_variant() == 1)
        k_fsolve_df<3, 2><<<n, kDfThreads, 0, st>>>(d, tasks, w, y, tk, itasks, ni);
    else if (df_variant() == 2)
        k_fsolve_df<4, 1><<<n, kDfThreads, 0, st>>>(d, tasks, w, y, tk, itasks, ni);
    else if (df_variant() == 3)
        k_fsolve_df<2, 3><<<n, kDfThreads, 0, st>>>(d, tasks, w, y, tk, itasks, ni);
    else
        k_fsolve_df<kDfBuf, 2><<<n, kDfThreads, 0, st>>>(d, tasks, w, y, tk, itasks, ni);
}
void launch_bsolve_df(const DevPlan &d, const int32_t *tasks, int64_t count, const int32_t *itasks, int64_t ninit,
                      int w, int deep, double *y, const int32_t *sn_rows, const int64_t *sn_rowptr, unsigned *tk,
                      cudaStream_t st) {
    if (count <= 0) return;
    const unsigned n = (unsigned)(count + ninit);
    const int ni = (int)ninit;
    if (!deep)
        k_bsolve_df<1, 3><<<n, kDfThreads, 0, st>>>(d, tasks, w, y, tk, itasks, ni, sn_rows, sn_rowptr);
    else if (df_variant() == 1)
        k_bsolve_df<3, 2><<<n, kDfThreads, 0, st>>>(d, tasks, w, y, tk, itasks, ni, sn_rows, sn_rowptr);
    else if (df_variant() == 2)
        k_bsolve_df<4, 1><<<n, kDfThreads, 0, st>>>(d, tasks, w, y, tk, itasks, ni, sn_rows, sn_rowptr);
    else if (df_variant() == 3)
        k_bsolve_df<2, 3><<<n, kDfThreads, 0, st>>>(d, tasks, w, y, tk, itasks, ni, sn_rows, sn_rowptr);
    else
        k_bsolve_df<kDfBuf, 2><<<n, kDfThreads, 0, st>>>(d, tasks, w, y, tk, itasks, ni, sn_rows, sn_rowptr);
}

// dst[first_s + j] = src[first_s + j] for the columns of the listed supernodes
__global__ void k_copy_cols(DevPlan d, const int32_t *__restrict__ list, const double *__restrict__ src,
                            double *__restrict__ dst) {
    const int s = list[blockIdx.x];
    const int k = d.sn_k[s], first = d.sn_first[s];
    for (int j = threadIdx.x; j < k; j += blockDim.x) dst[first + j] = src[first + j];
}
void launch_copy_cols(const DevPlan &d, const int32_t *list, int count, const double *src, double *dst,
                      cudaStream_t st) {
    if (count > 0) k_copy_cols<<<count, 128, 0, st>>>(d, list, src, dst);
}

void launch_fwd_solve(const DevPlan &d, const int32_t *list, int count, double *y, cudaStream_t st) {
    if (count > 0)
        k_fwd_solve<<<(count + kSmallSolveWarps - 1) / kSmallSolveWarps, 32 * kSmallSolveWarps, 0, st>>>(d, list, count, y);
}
void launch_bwd_solve(const DevPlan &d, const int32_t *list, int count, double *y, const int32_t *sn_rows,
                      const int64_t *sn_rowptr, cudaStream_t st) {
    if (count > 0)
        k_bwd_solve<<<(count + kSmallSolveWarps - 1) / kSmallSolveWarps, 32 * kSmallSolveWarps, 0, st>>>(
            d, list, count, y, sn_rows, sn_rowptr);
}

}  // namespace mf

// ============================================================ fp64 iterative refinement
// (mixed-precision mode; "single precision on the
// GPU ... iterative refinement in double precision")  r = b - A x in fp64 from the
// caller's values, in ORIGINAL labels (rows / columns reached through the final
// perm), over the symmetric CSR of B = P A P^T built at analyze time: row k lists
// (column k', B entry e) for every stored entry of row k and of column k.
namespace mf {
// bval[e] = sum of the caller's values of B entry e, in input order (reading C6)
__global__ void k_refine_bval(const int64_t *__restrict__ bvptr, const int64_t *__restrict__ bvidx,
                              const double *__restrict__ values, double *__restrict__ bval, int64_t nb) {
    for (int64_t e = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; e < nb; e += (int64_t)gridDim.x * blockDim.x) {
        double v = 0.0;
        for (int64_t q = bvptr[e]; q < bvptr[e + 1]; q++) v += values[bvidx[q]];
        bval[e] = v;
    }
}
__device__ __forceinline__ void atomic_max_nonneg(double *addr, double v) {
    // non-negative doubles order like their bit patterns
    atomicMax(reinterpret_cast<unsigned long long *>(addr), (unsigned long long)__double_as_longlong(v));
}
// r = b - A x (original labels); norms[0] = ||r||, [1] = ||x||, [2] = ||b||, [3] = ||A|| (inf norms)
__global__ void k_refine_resid(const int64_t *__restrict__ rs_ptr, const int32_t *__restrict__ rs_col,
                               const int32_t *__restrict__ rs_ent, const double *__restrict__ bval,
                               const int32_t *__restrict__ perm, const double *__restrict__ b,
                               const double *__restrict__ x, double *__restrict__ r, double *__restrict__ norms,
                               int64_t n) {
    double mr = 0.0, mx = 0.0, mb = 0.0, ma = 0.0;
    for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x) {
        const int32_t i = perm[k];
        double ax = 0.0, aa = 0.0;
        for (int64_t q = rs_ptr[k]; q < rs_ptr[k + 1]; q++) {
            const double v = bval[rs_ent[q]];
            ax = fma(v, x[perm[rs_col[q]]], ax);
            aa += fabs(v);
        }
        const double ri = b[i] - ax;
        r[i] = ri;
        mr = fmax(mr, fabs(ri));
        mx = fmax(mx, fabs(x[i]));
        mb = fmax(mb, fabs(b[i]));
        ma = fmax(ma, aa);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) {
        mr = fmax(mr, __shfl_xor_sync(0xffffffffu, mr, o));
        mx = fmax(mx, __shfl_xor_sync(0xffffffffu, mx, o));
        mb = fmax(mb, __shfl_xor_sync(0xffffffffu, mb, o));
        ma = fmax(ma, __shfl_xor_sync(0xffffffffu, ma, o));
    }
    if ((threadIdx.x & 31) == 0) {
        atomic_max_nonneg(norms + 0, mr);
        atomic_max_nonneg(norms + 1, mx);
        atomic_max_nonneg(norms + 2, mb);
        atomic_max_nonneg(norms + 3, ma);
    }
}
__global__ void k_refine_axpy(double *__restrict__ x, const double *__restrict__ dx, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        x[i] += dx[i];
}
static unsigned grid_for(int64_t n) { return (unsigned)std::max<int64_t>(1, std::min<int64_t>((n + 255) / 256, 148 * 8)); }
void launch_refine_bval(const DevPlan &d, const double *values, double *bval, int64_t nb, cudaStream_t st) {
    if (nb > 0) k_refine_bval<<<grid_for(nb), 256, 0, st>>>(d.bvptr, d.bvidx, values, bval, nb);
}
void launch_refine_resid(const DevPlan &d, const int64_t *rs_ptr, const int32_t *rs_col, const int32_t *rs_ent,
                         const double *bval, const double *b, const double *x, double *r, double *norms, int64_t n,
                         cudaStream_t st) {
    cudaMemsetAsync(norms, 0, 4 * sizeof(double), st);
    if (n > 0) k_refine_resid<<<grid_for(n), 256, 0, st>>>(rs_ptr, rs_col, rs_ent, bval, d.perm, b, x, r, norms, n);
}
void launch_refine_axpy(double *x, const double *dx, int64_t n, cudaStream_t st) {
    if (n > 0) k_refine_axpy<<<grid_for(n), 256, 0, st>>>(x, dx, n);
}
}  // namespace mf
