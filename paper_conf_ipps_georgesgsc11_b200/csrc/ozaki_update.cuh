// ozaki_update.cuh -- the Schur update C -= A A[0:N]^T of the factor-update step
// (the syrk U^n = U^n - L2 L2^T of PAPER.md L27 / Fig. 1 and the trailing updates
// of the blocked potrf) with FP64 EMULATED on the int8 tensor cores
// (tcgen05.mma .kind::i8, accumulators in TMEM): the Ozaki scheme.
// NEXT-3: the paper's own mixed-precision variant ran the GPU part in single
// precision and refined in double (Sec. III-B); on B200 the FP64
// DMMA path tops out at ~37 TF/s while the int8 tensor cores peak at 4.5 POPS.
//
// Split (k_oz_split): every row i of A (K values) is scaled by its own power of
// two, 2^-E_i with |A[i,p]| < 2^(E_i - 1), and cut into S balanced 7-bit digits
// (round to nearest, so the digit errors are unbiased and their sums grow like
// sqrt(K), not K as truncated digits of same-sign entries would):
//     A[i,p] = 2^E_i * sum_{s=1..S} q_s[i,p] 2^{-7s} + r,  q_s in [-64, 64],
//     |r| <= 2^{E_i - 7S - 1}                 (every step exact in fp64)
// so that
//     (A A^T)[i,j] = 2^{E_i+E_j} sum_{s,t} 2^{-7(s+t)} (q_s[i,:] . q_t[j,:]).
// The int8 products q_s . q_t are exact in int32 (|sum| <= K 64^2 per pair); all
// pairs with the same d = s + t share one int32 accumulator in TMEM (exact while
// (pairs of d) K 2^12 < 2^31, i.e. K <= 65,000 for S <= 8; the planner caps K at
// kOzMaxK).  Pairs with s + t > S + 1 are dropped (weight below 2^{-7(S+2)});
// with S = 8 the representation and truncation errors are ~2^-57 of
// |A_i| |A_j| sqrt(K) (fp64 rounding: 2^-53 of sum_p |A_ip A_jp|); S = 3..7 give
// a reduced-precision update for the mixed-precision mode with fp64 refinement.
//
// GEMM (k_oz_gemm): one CTA per 128 x 64 output tile; warp 0 stages the S int8
// slices of the tile's 128 A rows and 64 B rows (B rows = A rows j0.. of the same
// problem) into a shared-memory ring with cp.async.bulk (completing on the
// stage's full mbarrier); one elected thread of warp 1 issues the S(S+1)/2 pair
// MMAs per 32-byte k step (M = 128, N = 64, K = 32, A and B K-major from shared
// memory, no swizzle) into S TMEM accumulators of 64 columns (S <= 8: 512
// columns) and releases the stage with tcgen05.commit; at the end the 4 warps
// read their 32 TMEM lanes (= rows) with tcgen05.ld, recombine the diagonals in
// fp64 from the smallest weight up, scale by 2^{E_i+E_j} and subtract from C.
#pragma once
#include <cstdint>

#include "dmma_update.cuh"
#include "mf_plan.h"

namespace mf {

constexpr int kOzThreads = 128;   // tile / k constants: mf_plan.h

// OzProb / OzTile (the problem and tile lists, built at analyze time): mf_plan.h.

// ------------------------------------------------------------------ split
// Task = (oprob, 128-row block, segment of kOzSeg k values); one thread per row.
// k_oz_rowexp: E_i = max over the segments of frexp(max |A[i, seg]|) (atomicMax
// on an int initialised to INT_MIN-ish by a memset: order-independent);
// k_oz_split: 16 k values at a time -> S 16-byte digit rows.
template <int S>
__global__ void __launch_bounds__(kOzBM) k_oz_rowexp(const double *__restrict__ Larena,
                                                     const GemmProb *__restrict__ probs,
                                                     const OzProb *__restrict__ oprobs,
                                                     const int32_t *__restrict__ tasks, int32_t *__restrict__ expo) {
    const int op = tasks[3 * blockIdx.x], rb = tasks[3 * blockIdx.x + 1], sg = tasks[3 * blockIdx.x + 2];
    const OzProb o = oprobs[op];
    const GemmProb g = probs[o.prob];
    const int i = rb * kOzBM + threadIdx.x;
    const int p0 = sg * kOzSeg, p1 = min(g.K, p0 + kOzSeg);
    double mx = 0.0;
    if (i < g.M) {
        const double *__restrict__ a = Larena + g.a_off + i;
#pragma unroll 8
        for (int p = p0; p < p1; p++) mx = fmax(mx, fabs(__ldg(a + (int64_t)p * g.lda)));
    }
    int E = 0;
    if (mx > 0.0) frexp(mx, &E);   // mx = f 2^E, f in [0.5, 1): |A[i, p]| < 2^E
    atomicMax(expo + o.ex_off + i, E + 1);   // scale 2^(E+1): |A[i, p]| 2^-(E+1) < 1/2
}

template <int S>
__global__ void __launch_bounds__(kOzBM) k_oz_split(const double *__restrict__ Larena, const GemmProb *__restrict__ probs,
                                                    const OzProb *__restrict__ oprobs, const int32_t *__restrict__ tasks,
                                                    int8_t *__restrict__ slices, const int32_t *__restrict__ expo) {
    const int op = tasks[3 * blockIdx.x], rb = tasks[3 * blockIdx.x + 1], sg = tasks[3 * blockIdx.x + 2];
    const OzProb o = oprobs[op];
    const GemmProb g = probs[o.prob];
    const int i = rb * kOzBM + threadIdx.x;
    const bool live = i < g.M;
    const double *__restrict__ a = Larena + g.a_off + i;
    const int64_t lda = g.lda;
    const int E = expo[o.ex_off + i];
    const int KC = o.Kpad / 16;
    int8_t *__restrict__ base = slices + o.sl_off + (int64_t)i * 16;
    const int64_t sstride = (int64_t)KC * o.Mpad * 16, kstride = (int64_t)o.Mpad * 16;
    const int kc0 = sg * (kOzSeg / 16), kc1 = min(KC, kc0 + kOzSeg / 16);
    for (int kc = kc0; kc < kc1; kc++) {
        uint32_t w[S][4];
#pragma unroll
        for (int q = 0; q < 16; q++) {
            const int p = kc * 16 + q;
            double r = (live && p < g.K) ? ldexp(__ldg(a + (int64_t)p * lda), -E) : 0.0;   // |r| < 1/2
#pragma unroll
            for (int s = 0; s < S; s++) {
                r *= 128.0;                   // |r| < 64
                const double qd = rint(r);    // balanced digit, |qd| <= 64
                r -= qd;                      // exact, |r| <= 1/2
                const uint32_t b = (uint32_t)(uint8_t)(int8_t)(int)qd;
                if (q % 4 == 0) w[s][q / 4] = b;
                else w[s][q / 4] |= b << (8 * (q % 4));
            }
        }
#pragma unroll
        for (int s = 0; s < S; s++)
            *reinterpret_cast<uint4 *>(base + s * sstride + kc * kstride) = make_uint4(w[s][0], w[s][1], w[s][2], w[s][3]);
    }
}

// ------------------------------------------------------------------ tcgen05 helpers
__device__ __forceinline__ uint64_t oz_desc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
    // shared-memory matrix descriptor, K-major, no swizzle: start >> 4 [0,14),
    // leading (K-direction core-matrix) byte offset >> 4 [16,30), stride (M/N
    // direction, 8-row core matrices) byte offset >> 4 [32,46), version 1 [46,48)
    return (uint64_t)((saddr >> 4) & 0x3fff) | ((uint64_t)((lbo >> 4) & 0x3fff) << 16) |
           ((uint64_t)((sbo >> 4) & 0x3fff) << 32) | (1ull << 46);
}
// instruction descriptor: D s32 [4,6) = 2, A s8 [7,10) = 1, B s8 [10,13) = 1,
// both K-major, N >> 3 at [17,23), M >> 4 at [24,29)
constexpr uint32_t kOzIdesc = (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(kOzBN >> 3) << 17) |
                              ((uint32_t)(kOzBM >> 4) << 24);

__device__ __forceinline__ void oz_mma(uint32_t dtmem, uint64_t adesc, uint64_t bdesc, uint32_t acc,
                                       uint32_t idesc = kOzIdesc) {
    asm volatile(
        "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
        " tcgen05.mma.cta_group::1.kind::i8 [%0], %1, %2, %3, p;\n}\n" ::"r"(dtmem),
        "l"(adesc), "l"(bdesc), "r"(idesc), "r"(acc)
        : "memory");
}
__device__ __forceinline__ void oz_commit(uint64_t *bar) {
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];\n" ::"l"(
                     (uint64_t)__cvta_generic_to_shared(bar))
                 : "memory");
}
#define OZ_LD32(taddr, r)                                                                                           \
    asm volatile(                                                                                                   \
        "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,%17,%18," \
        "%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31}, [%32];\n"                                            \
        : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),           \
          "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),     \
          "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),   \
          "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])    \
        : "r"(taddr))

template <int S>
struct OzCfg {
    static constexpr int A_BYTES = S * (kOzBK / 16) * kOzBM * 16;   // S slices x 4 k-cores x 128 rows x 16 B
    static constexpr int B_BYTES = S * (kOzBK / 16) * kOzBN * 16;
    static constexpr int STAGE = A_BYTES + B_BYTES;
    static constexpr int STAGES = (200 * 1024) / STAGE < 2 ? 2 : ((200 * 1024) / STAGE > 6 ? 6 : (200 * 1024) / STAGE);
    static constexpr size_t SMEM = (size_t)STAGES * STAGE + 1024;
    static_assert(S >= 1 && S * kOzBN <= 512, "TMEM: S accumulators of 64 columns");
};

template <int S>
__global__ void __launch_bounds__(kOzThreads, 1)
    k_oz_gemm(double *__restrict__ Larena, double *__restrict__ Uarena, const GemmProb *__restrict__ probs,
              const OzProb *__restrict__ oprobs, const OzTile *__restrict__ tiles, const int8_t *__restrict__ slices,
              const int32_t *__restrict__ expo, const UpdGather gv) {
    using Cfg = OzCfg<S>;
    constexpr int STAGES = Cfg::STAGES;
    extern __shared__ __align__(1024) uint8_t osm[];
    uint64_t *full = reinterpret_cast<uint64_t *>(osm + STAGES * Cfg::STAGE);
    uint64_t *empty = full + STAGES;
    uint64_t *tfull = empty + STAGES;
    uint32_t *tbase_sh = reinterpret_cast<uint32_t *>(tfull + 1);
    int32_t *ej = reinterpret_cast<int32_t *>(tbase_sh + 1);   // E of the tile's 64 columns
    const OzTile t = tiles[blockIdx.x];
    const OzProb o = oprobs[t.oprob];
    const GemmProb g = probs[o.prob];
    const int ti = t.tij >> 16, tj = t.tij & 0xffff;
    const int i0 = ti * kOzBM, j0 = tj * kOzBN;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int KB = o.Kpad / kOzBK, KC = o.Kpad / 16;

    if (tid == 0) {
        for (int st = 0; st < STAGES; st++) {
            mbar_init(full + st, 1);
            mbar_init(empty + st, 1);
        }
        mbar_init(tfull, 1);
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    if (warp == 2) {   // TMEM: S accumulators x 64 columns (allocation: power of two >= 32)
        constexpr uint32_t cols = S * kOzBN <= 32 ? 32 : S * kOzBN <= 64 ? 64 : S * kOzBN <= 128 ? 128
                                : S * kOzBN <= 256 ? 256 : 512;
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;\n" ::"r"(smem_u32(tbase_sh)),
                     "n"(cols)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n" ::: "memory");
    }
    if (tid < kOzBN) ej[tid] = expo[o.ex_off + j0 + tid];
    asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
    const uint32_t tbase = *tbase_sh;

    const int8_t *__restrict__ sl = slices + o.sl_off;
    const int64_t kstride = (int64_t)o.Mpad * 16;            // one 16-byte k-core of all rows
    const int64_t sstride = (int64_t)KC * kstride;
    if (warp == 0) {
        // ---- producer: stage kb = S slices x 4 k-cores x (128 A rows + 64 B rows)
        for (int kb = 0; kb < KB; kb++) {
            const int st = kb % STAGES;
            if (kb >= STAGES) mbar_wait(empty + st, ((kb / STAGES) - 1) & 1);
            if (lane == 0) mbar_arrive_tx(full + st, (unsigned)Cfg::STAGE);
            __syncwarp();
            uint8_t *As = osm + st * Cfg::STAGE, *Bs = As + Cfg::A_BYTES;
            for (int c = lane; c < 2 * S * 4; c += 32) {
                const int isB = c >= S * 4, sc = isB ? c - S * 4 : c, s = sc >> 2, kc = sc & 3;
                const int8_t *src = sl + s * sstride + (int64_t)(kb * 4 + kc) * kstride + (int64_t)(isB ? j0 : i0) * 16;
                if (isB) bulk_g2s(Bs + (s * 4 + kc) * (kOzBN * 16), src, kOzBN * 16, full + st);
                else bulk_g2s(As + (s * 4 + kc) * (kOzBM * 16), src, kOzBM * 16, full + st);
            }
        }
    } else if (warp == 1) {
        // ---- MMA issuer: per 32-byte k step, pairs (s, t), s + t <= S - 1 (0-based)
        for (int kb = 0; kb < KB; kb++) {
            const int st = kb % STAGES;
            mbar_wait(full + st, (kb / STAGES) & 1);
            asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
            if (lane == 0) {
                const uint32_t a0 = smem_u32(osm + st * Cfg::STAGE), b0 = a0 + Cfg::A_BYTES;
#pragma unroll
                for (int kk = 0; kk < kOzBK / 32; kk++)
#pragma unroll
                    for (int s = 0; s < S; s++) {
                        // k-cores 2kk, 2kk+1 of slice s: LBO = one k-core, SBO = 8 rows
                        const uint64_t ad = oz_desc(a0 + (s * 4 + 2 * kk) * (kOzBM * 16), kOzBM * 16, 128);
#pragma unroll
                        for (int u = 0; u < S - s; u++) {
                            const uint64_t bd = oz_desc(b0 + (u * 4 + 2 * kk) * (kOzBN * 16), kOzBN * 16, 128);
                            oz_mma(tbase + (uint32_t)((s + u) * kOzBN), ad, bd, (kb | kk | s) != 0);
                        }
                    }
                oz_commit(empty + st);   // the stage is free once these MMAs complete
            }
            __syncwarp();
        }
        if (lane == 0) oz_commit(tfull);
        __syncwarp();
    }
    // ---- epilogue: thread = tile row (TMEM lane 32 warp + lane).  The pipeline is
    // drained, so the stage memory holds P (the product, 2^{E_i+E_j} sum_d 2^{-7(d+2)}
    // D_d, fp64) and, for the syrk on U^s with the fused extend-add (flags bit 2),
    // G = 0 (+) U^c1 (+) U^c2 ... gathered in ascending child order (reading C6);
    // both column-major 128 x 64.  C = (G or C) - P, masked to the lower trapezoid.
    mbar_wait(tfull, 0);
    asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
    double *Ps = reinterpret_cast<double *>(osm), *Gs = Ps + kOzBM * kOzBN;
    int *rq = reinterpret_cast<int *>(Gs + kOzBM * kOzBN), *cq = rq + kOzBM;
    static_assert(Cfg::STAGES * Cfg::STAGE >= 2 * kOzBM * kOzBN * 8 + (kOzBM + kOzBN) * 4, "epilogue staging");
    const int il = warp * 32 + lane, i = i0 + il;
    const int sh = (g.flags >> 1) & 1;
    const int Ei = expo[o.ex_off + i];
#pragma unroll 1
    for (int c0 = 0; c0 < kOzBN; c0 += 32) {
        double v[32];
#pragma unroll
        for (int q = 0; q < 32; q++) v[q] = 0.0;
#pragma unroll 1
        for (int d = S - 1; d >= 0; d--) {   // smallest weight first
            uint32_t r[32];
            OZ_LD32(tbase + ((uint32_t)(warp * 32) << 16) + (uint32_t)(d * kOzBN + c0), r);
            asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
            const double w = ldexp(1.0, -7 * (d + 2));
#pragma unroll
            for (int q = 0; q < 32; q++) v[q] = fma((double)(int32_t)r[q], w, v[q]);
        }
#pragma unroll
        for (int q = 0; q < 32; q++) Ps[(c0 + q) * kOzBM + il] = ldexp(v[q], Ei + ej[c0 + q]);
    }
    const bool gather = (g.flags & 4) != 0;
    if (gather) {
        for (int x = tid; x < kOzBM * kOzBN; x += kOzThreads) Gs[x] = 0.0;
        const int q0 = gv.child_ptr[g.s], q1 = gv.child_ptr[g.s + 1], kp = gv.sn_k[g.s];
        const int ntr1 = (g.M + kTileM - 1) / kTileM + 1;   // ea_qs tables are per 64-row tile
        const int tr0 = i0 / kTileM, tr1 = min(tr0 + kOzBM / kTileM, ntr1 - 1);
        for (int jc = 0; jc < q1 - q0; jc++) {
            const int32_t *__restrict__ qs = gv.qs + g.qs_off + (int64_t)jc * ntr1;
            const int ra = qs[tr0], rb = qs[tr1], ca = qs[tj], cb = qs[tj + 1];
            if (ra == rb || ca == cb) continue;   // uniform over the CTA
            const int ch = gv.child_list[q0 + jc];
            const int mc = gv.sn_f[ch] - gv.sn_k[ch];
            const int32_t *__restrict__ rel = gv.relmap + gv.relmap_ptr[ch];
            const double *__restrict__ Uc = Uarena + gv.U_off[ch];
            __syncthreads();   // the previous child's maps are consumed
            for (int x = tid; x < kOzBM + kOzBN; x += kOzThreads) rq[x] = -1;
            __syncthreads();
            // front row r >= kp sits at shifted U row r - kp + sh
            for (int q = ra + tid; q < rb; q += kOzThreads) rq[__ldg(rel + q) - kp + sh - i0] = q;
            for (int q = ca + tid; q < cb; q += kOzThreads) cq[__ldg(rel + q) - kp + sh - j0] = q;
            __syncthreads();
            const int qi = rq[il];
            if (qi >= 0)
                for (int c = 0; c < kOzBN; c++) {
                    const int qj = cq[c];
                    if (qj >= 0 && qi >= qj) Gs[c * kOzBM + il] += __ldg(Uc + upk(qi, qj, mc));
                }
        }
    }
    __syncwarp();
    double *__restrict__ C = ((g.flags & 1) ? Uarena : Larena) + g.c_off;
    const int64_t ldc = g.ldc;
    const bool packed = (g.flags & 1) != 0;   // U^s: packed lower (mf_plan.h upk); L: column-major
    auto cidx = [&](int64_t i, int64_t j) -> int64_t { return packed ? upk(i, j, ldc) : i + j * ldc; };
    if (i < g.M && i >= sh) {
        for (int c = 0; c < kOzBN; c++) {
            const int j = j0 + c;
            if (j < g.N && i >= j && j >= sh) {
                double *cp = C + cidx(i - sh, j - sh);
                *cp = (gather ? Gs[c * kOzBM + il] : *cp) - Ps[c * kOzBM + il];
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
    __syncthreads();
    if (warp == 2) {
        constexpr uint32_t cols = S * kOzBN <= 32 ? 32 : S * kOzBN <= 64 ? 64 : S * kOzBN <= 128 ? 128
                                : S * kOzBN <= 256 ? 256 : 512;
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;\n" ::"r"(tbase), "n"(cols) : "memory");
    }
}


// ------------------------------------------------------------------ 128 x 128 tiles, two passes
// Measured (tools/ubench/ozaki_gemm.cu, 8192^2 x 4096 SYRK): S = 4 in one pass 2.30 ms
// vs 3.16 ms with 128 x 64 tiles; S = 8 in two passes 5.56 vs 5.45 ms -- per output
// element both move the same slice bytes from L2 (12 slice loads over 256 rows vs 8
// over 192), which bounds them at ~5 TB/s of L2 -> shared-memory traffic.
// k_oz_gemm2: the same product on 128 x 128 output tiles.  N = 128 halves the
// shared-memory operand traffic per MMA (A 4 KB + B 4 KB per 64 cycles = 128 B/clk,
// vs 192 B/clk for N = 64), but S accumulators of 128 columns do not fit TMEM, so
// the diagonals are taken in two passes of at most four (pass 0: d = s + t <= 3,
// slices 0..3, 64-byte k stages; pass 1: 4 <= d <= S - 1, all slices, 32-byte k
// stages -- both 64 KB per stage).  Roles: warps 0-3 = epilogue (TMEM lane quarters),
// warp 4 = producer (cp.async.bulk, runs ahead into pass 1 while pass 0 drains), warp
// 5 = MMA issuer (waits for the epilogue to release TMEM before pass 1).  Pass 0's
// epilogue writes C = (C or the gathered sum of the children's U^c) - P_0, pass 1's
// C -= P_1 (each element by one thread: a fixed order).
constexpr int kOz2BN = 128, kOz2Threads = 192, kOz2Stage = 64 * 1024, kOz2Stages = 3;
constexpr uint32_t kOz2Idesc = (2u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(kOz2BN >> 3) << 17) |
                               ((uint32_t)(kOzBM >> 4) << 24);
constexpr size_t kOz2Smem = (size_t)kOz2Stages * kOz2Stage + 2048;

__device__ __forceinline__ void oz2_bar_epi() { asm volatile("bar.sync 1, 128;\n" ::: "memory"); }

template <int S>
__global__ void __launch_bounds__(kOz2Threads, 1)
    k_oz_gemm2(double *__restrict__ Larena, double *__restrict__ Uarena, const GemmProb *__restrict__ probs,
               const OzProb *__restrict__ oprobs, const OzTile *__restrict__ tiles, const int8_t *__restrict__ slices,
               const int32_t *__restrict__ expo, const UpdGather gv) {
    constexpr int DA = S < 4 ? S : 4;                 // diagonals of pass 0
    constexpr int NP = S > 4 ? 2 : 1;                 // passes
    extern __shared__ __align__(1024) uint8_t osm[];
    uint64_t *full = reinterpret_cast<uint64_t *>(osm + kOz2Stages * kOz2Stage);
    uint64_t *empty = full + kOz2Stages;
    uint64_t *tfull = empty + kOz2Stages;             // MMA -> epilogue, one phase per pass
    uint64_t *tempty = tfull + 1;                     // epilogue -> MMA (TMEM released after pass 0)
    uint32_t *tbase_sh = reinterpret_cast<uint32_t *>(tempty + 1);
    int32_t *ej = reinterpret_cast<int32_t *>(tbase_sh + 1);   // E of the tile's 128 columns
    int *rq = ej + kOz2BN, *cq = rq + kOzBM;          // gather maps
    const OzTile t = tiles[blockIdx.x];
    const OzProb o = oprobs[t.oprob];
    const GemmProb g = probs[o.prob];
    const int ti = t.tij >> 16, tj = t.tij & 0xffff;
    const int i0 = ti * kOzBM, j0 = tj * kOz2BN;
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int KC = o.Kpad / 16;

    if (tid == 0) {
        for (int st = 0; st < kOz2Stages; st++) {
            mbar_init(full + st, 1);
            mbar_init(empty + st, 1);
        }
        mbar_init(tfull, 1);
        mbar_init(tempty, 4);
        asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
    }
    if (warp == 2) {
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;\n" ::"r"(smem_u32(tbase_sh))
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;\n" ::: "memory");
    }
    if (tid < kOz2BN) ej[tid] = expo[o.ex_off + j0 + tid];
    asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
    const uint32_t tbase = *tbase_sh;
    const int8_t *__restrict__ sl = slices + o.sl_off;
    const int64_t kstride = (int64_t)o.Mpad * 16, sstride = (int64_t)KC * kstride;

    if (warp == 4) {
        // ---- producer: pass p stage = ns slices x nkc k-cores x (128 A rows + 128 B rows)
        int gs = 0;
        for (int p = 0; p < NP; p++) {
            const int ns = p == 0 ? DA : S, nkc = ns <= 4 ? 4 : 2, KB = KC / nkc;
            for (int kb = 0; kb < KB; kb++, gs++) {
                const int st = gs % kOz2Stages;
                if (gs >= kOz2Stages) mbar_wait(empty + st, ((gs / kOz2Stages) - 1) & 1);
                if (lane == 0) mbar_arrive_tx(full + st, (unsigned)(2 * ns * nkc * kOzBM * 16));
                __syncwarp();
                uint8_t *As = osm + st * kOz2Stage, *Bs = As + ns * nkc * kOzBM * 16;
                for (int c = lane; c < 2 * ns * nkc; c += 32) {
                    const int isB = c >= ns * nkc, sc = isB ? c - ns * nkc : c, s = sc / nkc, kc = sc % nkc;
                    const int8_t *src = sl + s * sstride + (int64_t)(kb * nkc + kc) * kstride +
                                        (int64_t)(isB ? j0 : i0) * 16;
                    bulk_g2s((isB ? Bs : As) + (s * nkc + kc) * (kOzBM * 16), src, kOzBM * 16, full + st);
                }
            }
        }
    } else if (warp == 5) {
        // ---- MMA issuer
        int gs = 0;
        for (int p = 0; p < NP; p++) {
            const int ns = p == 0 ? DA : S, nkc = ns <= 4 ? 4 : 2, KB = KC / nkc;
            const int dlo = p == 0 ? 0 : DA, dhi = p == 0 ? DA : S;
            if (p == 1) {   // TMEM is free once pass 0's epilogue has read it
                mbar_wait(tempty, 0);
                asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
            }
            for (int kb = 0; kb < KB; kb++, gs++) {
                const int st = gs % kOz2Stages;
                mbar_wait(full + st, (gs / kOz2Stages) & 1);
                asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
                if (lane == 0) {
                    const uint32_t a0 = smem_u32(osm + st * kOz2Stage), b0 = a0 + ns * nkc * kOzBM * 16;
                    for (int kk = 0; kk < nkc / 2; kk++)
                        for (int s = 0; s < ns; s++) {
                            const uint64_t ad = oz_desc(a0 + (s * nkc + 2 * kk) * (kOzBM * 16), kOzBM * 16, 128);
                            for (int u = max(0, dlo - s); u < dhi - s && u < ns; u++) {
                                const uint64_t bd = oz_desc(b0 + (u * nkc + 2 * kk) * (kOzBM * 16), kOzBM * 16, 128);
                                oz_mma(tbase + (uint32_t)((s + u - dlo) * kOz2BN), ad, bd, (kb | kk | s) != 0, kOz2Idesc);
                            }
                        }
                    oz_commit(empty + st);
                }
                __syncwarp();
            }
            if (lane == 0) oz_commit(tfull);
            __syncwarp();
        }
    } else {
        // ---- epilogue warps 0-3: thread = tile row (TMEM lane)
        const int il = tid, i = i0 + il;
        const int sh = (g.flags >> 1) & 1;
        double *__restrict__ C = ((g.flags & 1) ? Uarena : Larena) + g.c_off;
        const int64_t ldc = g.ldc;
        const bool packed = (g.flags & 1) != 0;   // U^s: packed lower (mf_plan.h upk); L: column-major
        auto cidx = [&](int64_t i, int64_t j) -> int64_t { return packed ? upk(i, j, ldc) : i + j * ldc; };
        const int Ei = expo[o.ex_off + i];
        const bool row_ok = i < g.M && i >= sh;
        const bool gather = (g.flags & 4) != 0;
        if (gather) {   // C = 0 (+) U^c1 (+) U^c2 ..., in ascending child order (reading C6)
            if (row_ok)
                for (int c = 0; c < kOz2BN; c++) {
                    const int j = j0 + c;
                    if (j < g.N && i >= j && j >= sh) C[cidx(i - sh, j - sh)] = 0.0;
                }
            const int q0 = gv.child_ptr[g.s], q1 = gv.child_ptr[g.s + 1], kp = gv.sn_k[g.s];
            const int ntr1 = (g.M + kTileM - 1) / kTileM + 1;   // ea_qs tables are per 64-row tile
            const int tr0 = i0 / kTileM, tr1 = min(tr0 + kOzBM / kTileM, ntr1 - 1);
            const int tc0 = j0 / kTileN, tc1 = min(tc0 + kOz2BN / kTileN, ntr1 - 1);
            for (int jc = 0; jc < q1 - q0; jc++) {
                const int32_t *__restrict__ qs = gv.qs + g.qs_off + (int64_t)jc * ntr1;
                const int ra = qs[tr0], rb = qs[tr1], ca = qs[tc0], cb = qs[tc1];
                if (ra == rb || ca == cb) continue;   // uniform over the epilogue warps
                const int ch = gv.child_list[q0 + jc];
                const int mc = gv.sn_f[ch] - gv.sn_k[ch];
                const int32_t *__restrict__ rel = gv.relmap + gv.relmap_ptr[ch];
                const double *__restrict__ Uc = Uarena + gv.U_off[ch];
                oz2_bar_epi();   // the previous child's maps are consumed
                for (int x = tid; x < kOzBM + kOz2BN; x += 128) rq[x] = -1;
                oz2_bar_epi();
                for (int q = ra + tid; q < rb; q += 128) rq[__ldg(rel + q) - kp + sh - i0] = q;
                for (int q = ca + tid; q < cb; q += 128) cq[__ldg(rel + q) - kp + sh - j0] = q;
                oz2_bar_epi();
                const int qi = rq[il];
                if (qi >= 0 && row_ok)
                    for (int c = 0; c < kOz2BN; c++) {
                        const int qj = cq[c], j = j0 + c;
                        if (qj >= 0 && qi >= qj && j < g.N && i >= j && j >= sh)
                            C[cidx(i - sh, j - sh)] += __ldg(Uc + upk(qi, qj, mc));
                    }
            }
        }
        for (int p = 0; p < NP; p++) {
            const int dlo = p == 0 ? 0 : DA, dhi = p == 0 ? DA : S;
            mbar_wait(tfull, p & 1);
            asm volatile("tcgen05.fence::after_thread_sync;\n" ::: "memory");
#pragma unroll 1
            for (int c0 = 0; c0 < kOz2BN; c0 += 32) {
                double v[32];
#pragma unroll
                for (int q = 0; q < 32; q++) v[q] = 0.0;
#pragma unroll 1
                for (int d = dhi - 1; d >= dlo; d--) {   // smallest weight first
                    uint32_t r[32];
                    OZ_LD32(tbase + ((uint32_t)(warp * 32) << 16) + (uint32_t)((d - dlo) * kOz2BN + c0), r);
                    asm volatile("tcgen05.wait::ld.sync.aligned;\n" ::: "memory");
                    const double w = ldexp(1.0, -7 * (d + 2));
#pragma unroll
                    for (int q = 0; q < 32; q++) v[q] = fma((double)(int32_t)r[q], w, v[q]);
                }
                if (row_ok) {
#pragma unroll
                    for (int q = 0; q < 32; q++) {
                        const int j = j0 + c0 + q;
                        if (j < g.N && i >= j && j >= sh) {
                            double *cp = C + cidx(i - sh, j - sh);
                            *cp -= ldexp(v[q], Ei + ej[c0 + q]);
                        }
                    }
                }
            }
            if (p + 1 < NP) {   // TMEM read: the MMA warp may overwrite it with pass 1
                asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
                __syncwarp();
                if (lane == 0) mbar_arrive(tempty);
            }
        }
    }
    asm volatile("tcgen05.fence::before_thread_sync;\n" ::: "memory");
    __syncthreads();
    if (warp == 2)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;\n" ::"r"(tbase) : "memory");
}

// expo_words: the exponent words of this launch's problems (reset before the max).
template <int S>
inline cudaError_t oz_set_attr() {
    cudaError_t e = cudaFuncSetAttribute(k_oz_gemm<S>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)OzCfg<S>::SMEM);
    if (e == cudaSuccess)
        e = cudaFuncSetAttribute(k_oz_gemm2<S>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kOz2Smem);
    return e;
}

template <int S>
inline void launch_oz(double *L, double *U, const GemmProb *probs, const OzProb *oprobs, const int32_t *split_tasks,
                      int64_t nsplit, const OzTile *tiles, int64_t ntiles, int8_t *slices, int32_t *expo,
                      int64_t expo_words, cudaStream_t st, const UpdGather gv = UpdGather{}, int wide = 0) {
    if (nsplit > 0) {
        cudaMemsetAsync(expo, 0x80, (size_t)expo_words * sizeof(int32_t), st);   // 0x80808080 < any exponent
        k_oz_rowexp<S><<<(unsigned)nsplit, kOzBM, 0, st>>>(L, probs, oprobs, split_tasks, expo);
        k_oz_split<S><<<(unsigned)nsplit, kOzBM, 0, st>>>(L, probs, oprobs, split_tasks, slices, expo);
    }
    if (ntiles > 0) {
        static bool attr = false;   // libmf sets it up front (kernels_init), before any graph capture
        if (!attr) {
            oz_set_attr<S>();
            attr = true;
        }
        if (wide)   // 128 x 128 tiles, two passes
            k_oz_gemm2<S><<<(unsigned)ntiles, kOz2Threads, kOz2Smem, st>>>(L, U, probs, oprobs, tiles, slices, expo, gv);
        else
            k_oz_gemm<S><<<(unsigned)ntiles, kOzThreads, OzCfg<S>::SMEM, st>>>(L, U, probs, oprobs, tiles, slices,
                                                                                 expo, gv);
    }
}

}  // namespace mf
