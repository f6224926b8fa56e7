// dmma_update.cuh -- the FP64 DMMA Schur-update kernel (the dense contraction of
// the factor-update step: the syrk U^n = U^n - L2 L2^T of PAPER.md L27 / Fig. 1,
// and the trailing syrk/gemm updates of the blocked potrf of PAPER.md L325 /
// Fig. 9), as a template over its tile / pipeline shape.
//
//   C[i][j] -= sum_p A[i][p] A[j][p],  0 <= j < N, j <= i < M   (lower trapezoid)
//
// A (M x K) and C are column-major with leading dimensions lda / ldc; A lives in
// the L arena, C in the L arena (panel update) or the U arena (syrk on U^n).
//
// sm_100a has no f64 kind of tcgen05.mma (probe 1), so the FP64
// tensor path is warp-level mma.sync.m8n8k4.f64 (SASS DMMA.8x8x4).  Operands are
// staged into a STAGES-deep shared-memory ring either by every thread's 16-byte
// cp.async (LDGSTS, zero-fill at the edges; CTA barrier per k-tile) or -- the
// BULK variant, for launches of many long-K waves -- by warp 0's cp.async.bulk
// per operand column with full / empty mbarriers (no CTA barrier in the loop).
// Each warp owns a TM x TN sub-tile whose accumulators start from C (loaded while
// the first stages are in flight; for the syrk on U^s with the fused extend-add,
// gathered from the children's U^c instead) and accumulate C - A B^T directly
// (A fragments negated), so the epilogue is a masked store.  Columns are 16-byte aligned (lda even) and every problem's
// first row is even: the planner shifts a problem whose first row is odd (the
// syrk on U^n of a supernode with odd k) one row up, computes the extra leading
// row / column of the shifted space and masks it out here (flag bit 1).
#pragma once
#include <cstdint>

#include "mf_plan.h"

namespace mf {

__device__ __forceinline__ void cp_async16(void *smem, const void *gmem, bool valid) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    const int n = valid ? 16 : 0;
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;\n" ::"r"(s), "l"(gmem), "r"(n));
}
__device__ __forceinline__ void cp_async8(void *smem, const void *gmem, bool valid) {
    const unsigned s = (unsigned)__cvta_generic_to_shared(smem);
    const int n = valid ? 8 : 0;
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8, %2;\n" ::"r"(s), "l"(gmem), "r"(n));
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N)); }

__device__ __forceinline__ void dmma(double &c0, double &c1, double a, double b) {
    asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};\n"
                 : "+d"(c0), "+d"(c1)
                 : "d"(a), "d"(b));
}

// mbarrier + bulk-copy pipeline (the BULK variant): warp 0 stages every operand
// column of a k-tile with one cp.async.bulk per lane (rows i0 .. i0+BM of an A
// column are contiguous: 512 bytes), completing on the stage's "full" mbarrier;
// each warp waits on it, computes, and arrives on the stage's "empty" mbarrier,
// so no CTA-wide barrier sits in the main loop and no thread issues per-16-byte
// copies.  Rows past M / N are staged as they are (they only feed masked
// outputs: a DMMA output row depends on its own A row); k columns past K are
// zero-filled by the producer lanes.
__device__ __forceinline__ unsigned smem_u32(const void *p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t *b, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;\n" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(uint64_t *b, unsigned tx) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;\n" ::"r"(smem_u32(b)), "r"(tx) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t *b) {
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];\n" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t *b, unsigned parity) {
    asm volatile(
        "{\n .reg .pred p;\n MBW_%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra MBW_%=;\n}\n" ::"r"(
            smem_u32(b)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void bulk_g2s(void *dst, const void *src, unsigned bytes, uint64_t *b) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];\n" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(b))
                 : "memory");
}

// Fused extend-add (GemmProb flags bit 2): the syrk on U^s
// starts from the children's contributions gathered through their relative maps
// (F^s = A-part (+) U^c1 (+) U^c2 ...; the U^s part of F^s has no A
// entries), summed per element in ascending child order from 0 -- the order of
// the assembly kernel (reading C6), so U^s is bit-identical to the unfused path.
struct UpdGather {
    const int32_t *child_ptr, *child_list, *sn_k, *sn_f;
    const int64_t *U_off, *relmap_ptr;
    const int32_t *relmap, *qs;
};

template <int BM_, int BN_, int BK_, int STAGES_, int WARPS_M_, int WARPS_N_, int MINB_>
struct UpdCfg {
    static constexpr int BM = BM_, BN = BN_, BK = BK_, STAGES = STAGES_;
    static constexpr int WARPS_M = WARPS_M_, WARPS_N = WARPS_N_, MINB = MINB_;
    static constexpr int NT = 32 * WARPS_M * WARPS_N;
    static constexpr int TM = BM / WARPS_M, TN = BN / WARPS_N;   // warp tile
    static constexpr int MB = TM / 8, NB = TN / 8;                // DMMA blocks per warp
    static constexpr int SA = BM + 4, SB = BN + 4;                // pad: stride % 16 == 4 (conflict-free fragments)
    // operand staging: 16-byte chunks (2 rows); every thread keeps a fixed row
    // slot and walks the k dimension with a fixed stride, so there is no index
    // math in the main loop.
    static constexpr int CPA = BM / 2, CPB = BN / 2;              // 16-byte chunks per column
    static_assert(NT % CPA == 0 && NT % CPB == 0, "staging map");
    static constexpr int PSA16 = NT / CPA, PSB16 = NT / CPB;      // k stride of a thread
    static_assert(BK % PSA16 == 0 && BK % PSB16 == 0, "staging map");
    static constexpr int STAGE_WORDS = BK * (SA + SB);
    static constexpr size_t SMEM =
        (size_t)STAGES * STAGE_WORDS * sizeof(double) + 2 * STAGES * sizeof(uint64_t) + (BM + BN) * sizeof(int) +
        BN * sizeof(int64_t);
    static_assert(SA % 16 == 4 && SB % 16 == 4, "bank-conflict-free fragment loads");
    static_assert(TM % 8 == 0 && TN % 8 == 0 && BK % 4 == 0, "tile shape");
};

template <class Cfg, bool BULK = false>
__global__ void __launch_bounds__(Cfg::NT, Cfg::MINB)
    k_update_t(double *__restrict__ Larena, double *__restrict__ Uarena, const GemmProb *__restrict__ probs,
               const TileTask *__restrict__ tiles, const UpdGather gv) {
    constexpr int BM = Cfg::BM, BN = Cfg::BN, BK = Cfg::BK, STAGES = Cfg::STAGES, NT = Cfg::NT;
    constexpr int SA = Cfg::SA, SB = Cfg::SB, STAGE_WORDS = Cfg::STAGE_WORDS;
    constexpr int MB = Cfg::MB, NB = Cfg::NB, TM = Cfg::TM, TN = Cfg::TN;
    extern __shared__ __align__(16) double sm[];
    const TileTask t = tiles[blockIdx.x];
    const GemmProb g = probs[t.prob];
    const int ti = t.tij >> 16, tj = t.tij & 0xffff;
    const int i0 = ti * BM, j0 = tj * BN;
    const double *__restrict__ A = Larena + g.a_off;   // a_off even: 16-byte aligned rows pairs
    const int lda = g.lda, K = g.K;
    const int sh = (g.flags >> 1) & 1;                   // shifted problem: row / column 0 are padding
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const int wm = warp % Cfg::WARPS_M, wn = warp / Cfg::WARPS_M;
    const int gq = lane >> 2, tq = lane & 3;
    // fixed staging slots of this thread
    const int ra16 = 2 * (tid % Cfg::CPA), pa16 = tid / Cfg::CPA;
    const int rb16 = 2 * (tid % Cfg::CPB), pb16 = tid / Cfg::CPB;
    const bool oka16 = i0 + ra16 < g.M, okb16 = j0 + rb16 < g.N;   // pair (r, r+1): r+1 may run past M: harmless

    auto load_stage = [&](int stage, int kt) {
        double *As = sm + stage * STAGE_WORDS;
        double *Bs = As + BK * SA;
        const int p0 = kt * BK;
        const double *__restrict__ Ak = A + (int64_t)p0 * lda;
#pragma unroll
        for (int p = pa16; p < BK; p += Cfg::PSA16) {
            const bool ok = oka16 && (p0 + p < K);
            cp_async16(As + p * SA + ra16, ok ? Ak + i0 + ra16 + (int64_t)p * lda : A, ok);
        }
#pragma unroll
        for (int p = pb16; p < BK; p += Cfg::PSB16) {
            const bool ok = okb16 && (p0 + p < K);
            cp_async16(Bs + p * SB + rb16, ok ? Ak + j0 + rb16 + (int64_t)p * lda : A, ok);
        }
    };

    const int KT = (K + BK - 1) / BK;
    uint64_t *full = reinterpret_cast<uint64_t *>(sm + STAGES * STAGE_WORDS), *empty = full + STAGES;
    // BULK: warp 0 stages k-tile kt into ring slot `stage` (lane c: A column c, B column c - BK)
    auto issue_bulk = [&](int stage, int kt) {
        double *As = sm + stage * STAGE_WORDS;
        double *Bs = As + BK * SA;
        const int p0 = kt * BK, nv = min(BK, K - p0);
        if (nv < BK) {   // k columns past K: zeros (generic stores, published by the arrive below)
            for (int c = lane; c < 2 * BK; c += 32) {
                const int p = c < BK ? c : c - BK;
                if (p >= nv) {
                    double *dst = c < BK ? As + p * SA : Bs + p * SB;
                    for (int r = 0; r < (c < BK ? BM : BN); r++) dst[r] = 0.0;
                }
            }
        }
        __syncwarp();
        constexpr int ra = BM, rb = BN;
        if (lane == 0) mbar_arrive_tx(full + stage, (unsigned)(nv * (ra + rb) * sizeof(double)));
        __syncwarp();
        const double *__restrict__ Ak = A + (int64_t)p0 * lda;
        for (int c = lane; c < 2 * BK; c += 32) {
            const int p = c < BK ? c : c - BK;
            if (p < nv) {
                if (c < BK) bulk_g2s(As + p * SA, Ak + (int64_t)p * lda + i0, ra * sizeof(double), full + stage);
                else bulk_g2s(Bs + p * SB, Ak + (int64_t)p * lda + j0, rb * sizeof(double), full + stage);
            }
        }
    };
    if constexpr (BULK) {
        static_assert(Cfg::SA * sizeof(double) % 16 == 0 && Cfg::SB * sizeof(double) % 16 == 0, "bulk dst alignment");
        if (tid == 0) {
            for (int st = 0; st < STAGES; st++) {
                mbar_init(full + st, 1);
                mbar_init(empty + st, NT / 32);
            }
            asm volatile("fence.mbarrier_init.release.cluster;\n" ::: "memory");
        }
        __syncthreads();
        if (warp == 0)
            for (int st = 0; st < STAGES && st < KT; st++) issue_bulk(st, st);
    } else {
#pragma unroll
        for (int st = 0; st < STAGES - 1; st++) {
            if (st < KT) load_stage(st, st);
            cp_async_commit();
        }
    }
    // C(i - sh, j - sh) for the (shifted) tile coordinates (i, j)
    double *__restrict__ C = ((g.flags & 1) ? Uarena : Larena) + g.c_off;
    const int ldc = g.ldc;
    const bool packed = (g.flags & 1) != 0;   // U^s: packed lower (mf_plan.h upk); L: column-major
    auto cidx = [&](int i, int j) -> int64_t { return packed ? upk(i, j, ldc) : i + (int64_t)j * ldc; };
    double acc[MB][NB][2];
    if (!(g.flags & 4)) {
#pragma unroll
        for (int mb = 0; mb < MB; mb++) {
            const int i = i0 + wm * TM + mb * 8 + gq;
#pragma unroll
            for (int nb = 0; nb < NB; nb++)
#pragma unroll
                for (int e = 0; e < 2; e++) {
                    const int j = j0 + wn * TN + nb * 8 + 2 * tq + e;
                    acc[mb][nb][e] =
                        (i < g.M && j < g.N && i >= sh && j >= sh && i >= j) ? C[cidx(i - sh, j - sh)] : 0.0;
                }
        }
    } else {
        // C = 0 (+) U^c1 (+) U^c2 ... over this tile: per child, the rows landing in
        // tile row ti / tile column tj are the contiguous ranges qs[ti..ti+1) /
        // qs[tj..tj+1) of its U^c (precomputed); their positions in the tile go
        // to shared maps, then every accumulator adds its element if both its row
        // and its column come from the child (lower part only: rel is increasing).
#pragma unroll
        for (int mb = 0; mb < MB; mb++)
#pragma unroll
            for (int nb = 0; nb < NB; nb++) acc[mb][nb][0] = acc[mb][nb][1] = 0.0;
        int64_t *cqb = reinterpret_cast<int64_t *>(empty + STAGES);   // packed column bases of cq
        int *rq = reinterpret_cast<int *>(cqb + BN), *cq = rq + BM;
        const int q0 = gv.child_ptr[g.s], q1 = gv.child_ptr[g.s + 1], kp = gv.sn_k[g.s];
        const int ntr1 = (g.M + BM - 1) / BM + 1;
        for (int jc = 0; jc < q1 - q0; jc++) {
            const int32_t *__restrict__ qs = gv.qs + g.qs_off + (int64_t)jc * ntr1;
            const int ra = qs[ti], rb = qs[ti + 1], ca = qs[tj], cb = qs[tj + 1];
            if (ra == rb || ca == cb) continue;   // uniform over the CTA
            const int ch = gv.child_list[q0 + jc];
            const int mc = gv.sn_f[ch] - gv.sn_k[ch];
            const int32_t *__restrict__ rel = gv.relmap + gv.relmap_ptr[ch];
            const double *__restrict__ Uc = Uarena + gv.U_off[ch];
            __syncthreads();   // the previous child's maps are consumed
            for (int x = tid; x < BM + BN; x += NT) rq[x] = -1;
            __syncthreads();
            // front row r >= kp sits at shifted U row r - kp + sh
            for (int q = ra + tid; q < rb; q += NT) rq[__ldg(rel + q) - kp + sh - i0] = q;
            for (int q = ca + tid; q < cb; q += NT) {
                const int x = __ldg(rel + q) - kp + sh - j0;
                cq[x] = q;
                cqb[x] = upk_col(q, mc) - q;   // child column q of the packed U^c, indexed by row
            }
            __syncthreads();
#pragma unroll
            for (int mb = 0; mb < MB; mb++) {
                const int qi = rq[wm * TM + mb * 8 + gq];
                if (qi < 0) continue;
#pragma unroll
                for (int nb = 0; nb < NB; nb++)
#pragma unroll
                    for (int e = 0; e < 2; e++) {
                        const int x = wn * TN + nb * 8 + 2 * tq + e, qj = cq[x];
                        if (qj >= 0 && qi >= qj) acc[mb][nb][e] += __ldg(Uc + cqb[x] + qi);
                    }
            }
        }
    }
    for (int kt = 0; kt < KT; kt++) {
        if constexpr (BULK) {
            mbar_wait(full + kt % STAGES, (kt / STAGES) & 1);
            // release the PREVIOUS slot: its LDS reads were consumed by the DMMAs of
            // iteration kt-1, all issued before the wait loop above (a basic-block
            // boundary ptxas does not schedule across).  Releasing right after the
            // DMMAs instead lets ptxas hoist the arrive above them while their LDS are
            // still in flight, and the bulk refill (async proxy) then races those
            // reads (seen as stale A rows in ~10% of runs); a proxy fence there
            // costs a MEMBAR per k-tile.
            if (kt > 0) {
                const int ps = (kt - 1) % STAGES;
                __syncwarp();
                if (lane == 0) mbar_arrive(empty + ps);
                if (warp == 0 && kt - 1 + STAGES < KT) {
                    mbar_wait(empty + ps, ((kt - 1) / STAGES) & 1);
                    issue_bulk(ps, kt - 1 + STAGES);
                }
            }
        } else {
            cp_async_wait<STAGES - 2>();
            __syncthreads();
            const int nk = kt + STAGES - 1;
            if (nk < KT) load_stage(nk % STAGES, nk);
            cp_async_commit();
        }
        const double *As = sm + (kt % STAGES) * STAGE_WORDS + wm * TM + gq;
        const double *Bs = sm + (kt % STAGES) * STAGE_WORDS + BK * SA + wn * TN + gq;
#pragma unroll
        for (int kk = 0; kk < BK / 4; kk++) {
            double a[MB], b[NB];
#pragma unroll
            for (int mb = 0; mb < MB; mb++) a[mb] = -As[(kk * 4 + tq) * SA + mb * 8];
#pragma unroll
            for (int nb = 0; nb < NB; nb++) b[nb] = Bs[(kk * 4 + tq) * SB + nb * 8];
#pragma unroll
            for (int mb = 0; mb < MB; mb++)
#pragma unroll
                for (int nb = 0; nb < NB; nb++) dmma(acc[mb][nb][0], acc[mb][nb][1], a[mb], b[nb]);
        }
    }
    if constexpr (!BULK) cp_async_wait<0>();
#pragma unroll
    for (int mb = 0; mb < MB; mb++) {
        const int i = i0 + wm * TM + mb * 8 + gq;
        if (i >= g.M) continue;
#pragma unroll
        for (int nb = 0; nb < NB; nb++)
#pragma unroll
            for (int e = 0; e < 2; e++) {
                const int j = j0 + wn * TN + nb * 8 + 2 * tq + e;
                if (j < g.N && i >= j && j >= sh) C[cidx(i - sh, j - sh)] = acc[mb][nb][e];
            }
    }
}

template <class Cfg, bool BULK = false>
inline void launch_update_t(double *L, double *U, const GemmProb *probs, const TileTask *tiles, int64_t ntiles,
                            cudaStream_t st, const UpdGather gv = UpdGather{}) {
    if (ntiles <= 0) return;
    if (Cfg::SMEM > 48 * 1024) {   // idempotent; libmf also sets it up front (kernels_init) before graph capture
        static bool attr = false;
        if (!attr) {
            cudaFuncSetAttribute(k_update_t<Cfg, BULK>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)Cfg::SMEM);
            attr = true;
        }
    }
    k_update_t<Cfg, BULK><<<(unsigned)ntiles, Cfg::NT, Cfg::SMEM, st>>>(L, U, probs, tiles, gv);
}

}  // namespace mf
