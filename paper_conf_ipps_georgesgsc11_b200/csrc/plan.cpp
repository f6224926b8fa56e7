// plan.cpp -- device memory planner and static launch schedule (SURVEY.md
// Sec. 8(a) rows a7 "Schedule + variant choice" and B3 "device memory planner").
//
// The paper picks a CPU/GPU policy per F-U call by operation count (P_BH,
// PAPER.md L401) or by a learned classifier.  Here the
// choice is GPU-only and static, made once per sparsity pattern: fronts of
// order f <= small_front_max run in the batched shared-memory kernel, larger
// ones in the tiled path (Fig. 9: blocked potrf with width w,
// trsm on the panel, syrk/gemm trailing update, then the syrk on U^n).
//
// Memory (the paper's grow-only pinned/GPU buffers, become one
// planned HBM arena): every supernode s owns
//   * its L panel: ld_s x k_s column-major, ld_s = f_s rounded up to even
//     (16-byte aligned columns for the 16-byte cp.async staging), in the L arena;
//   * its update matrix U^s: m_s x m_s column-major (lower triangle used) in the
//     U arena, written by the F-U of s and read by the extend-add of its parent.
#include <algorithm>
#include <numeric>

#include "mf.h"
#include "mf_plan.h"

namespace mf {

static void add_tiles(Plan &P, int32_t prob, int32_t M, int32_t N) {
    const int32_t tm = (M + kTileM - 1) / kTileM, tn = (N + kTileN - 1) / kTileN;
    for (int32_t tj = 0; tj < tn; tj++)
        for (int32_t ti = 0; ti < tm; ti++) {
            // lower-trapezoid: skip tiles entirely above the diagonal (i < j everywhere)
            if ((int64_t)(ti + 1) * kTileM - 1 < (int64_t)tj * kTileN) continue;
            P.tiles.push_back({prob, (ti << 16) | tj});
        }
}

int build_plan(const Symbolic &S, const Options &opt, Plan &P) {
    P = Plan();
    const int32_t ns = (int32_t)S.sn_parent.size();
    P.nsuper = ns;
    P.w = opt.panel_w;
    P.small_max = opt.small_front_max;
    P.sn_k.resize(ns);
    P.sn_f.resize(ns);
    P.sn_ld.resize(ns);
    P.sn_level.resize(ns);
    P.L_off.resize(ns);
    P.U_off.resize(ns);
    P.fv_off.resize(ns);
    int64_t loff = 0, uoff = 0, fvoff = 0;
    for (int32_t s = 0; s < ns; s++) {
        int32_t k = S.sn_first[s + 1] - S.sn_first[s];
        int32_t f = (int32_t)(S.sn_rowptr[s + 1] - S.sn_rowptr[s]);
        int32_t m = f - k;
        P.sn_k[s] = k;
        P.sn_f[s] = f;
        P.sn_ld[s] = f + (f & 1);
        P.L_off[s] = loff;
        loff += (int64_t)P.sn_ld[s] * k;
        P.U_off[s] = uoff;
        int64_t uw = (int64_t)m * m;
        uoff += uw + (uw & 1);
        P.fv_off[s] = fvoff;
        fvoff += f + (f & 1);
        P.max_front = std::max(P.max_front, f);
    }
    P.L_words = loff + 2;   // +16 B slack: 16-byte chunk reads may touch one row past a column end
    P.U_words = uoff + 2;
    P.fv_words = fvoff + 2;
    P.rows_total = S.sn_rowptr[ns];

    // children (ascending) and levels (height: leaves = 0)
    P.child_ptr.assign(ns + 1, 0);
    for (int32_t s = 0; s < ns; s++)
        if (S.sn_parent[s] >= 0) P.child_ptr[S.sn_parent[s] + 1]++;
    for (int32_t s = 0; s < ns; s++) P.child_ptr[s + 1] += P.child_ptr[s];
    P.child_list.resize(P.child_ptr[ns]);
    {
        std::vector<int32_t> fill(P.child_ptr.begin(), P.child_ptr.end() - 1);
        for (int32_t s = 0; s < ns; s++)
            if (S.sn_parent[s] >= 0) P.child_list[fill[S.sn_parent[s]]++] = s;
    }
    int32_t nlev = 0;
    for (int32_t s = 0; s < ns; s++) {
        int32_t lv = 0;
        for (int32_t q = P.child_ptr[s]; q < P.child_ptr[s + 1]; q++)
            lv = std::max(lv, P.sn_level[P.child_list[q]] + 1);
        P.sn_level[s] = lv;
        nlev = std::max(nlev, lv + 1);
    }
    P.nlevels = nlev;

    // relative index maps: position of R_c[k_c + q] inside R_parent(c)
    std::vector<int32_t> pos(S.n, -1);
    P.relmap_ptr.assign(ns + 1, 0);
    for (int32_t c = 0; c < ns; c++)
        P.relmap_ptr[c + 1] = P.relmap_ptr[c] + (S.sn_parent[c] >= 0 ? P.sn_f[c] - P.sn_k[c] : 0);
    P.relmap.resize(P.relmap_ptr[ns]);
    P.relmap_total = P.relmap_ptr[ns];
    P.blrow.resize(S.brow.size());
    for (int32_t s = 0; s < ns; s++) {
        const int32_t *R = S.sn_rows.data() + S.sn_rowptr[s];
        for (int32_t i = 0; i < P.sn_f[s]; i++) pos[R[i]] = i;
        for (int32_t q = P.child_ptr[s]; q < P.child_ptr[s + 1]; q++) {
            int32_t c = P.child_list[q];
            const int32_t *Rc = S.sn_rows.data() + S.sn_rowptr[c];
            for (int32_t i = P.sn_k[c]; i < P.sn_f[c]; i++) {
                int32_t ps = pos[Rc[i]];
                if (ps < 0) return MF_ERR_ARG;  // would mean an inconsistent row structure
                P.relmap[P.relmap_ptr[c] + i - P.sn_k[c]] = ps;
            }
        }
        for (int32_t j = S.sn_first[s]; j < S.sn_first[s + 1]; j++)
            for (int64_t e = S.bcolptr[j]; e < S.bcolptr[j + 1]; e++) P.blrow[e] = pos[S.brow[e]];
        for (int32_t i = 0; i < P.sn_f[s]; i++) pos[R[i]] = -1;
    }

    // ---------------- schedule by level
    P.level_ptr.assign(nlev + 1, 0);
    for (int32_t s = 0; s < ns; s++) P.level_ptr[P.sn_level[s] + 1]++;
    for (int32_t l = 0; l < nlev; l++) P.level_ptr[l + 1] += P.level_ptr[l];
    P.level_list.resize(ns);
    {
        std::vector<int32_t> fill(P.level_ptr.begin(), P.level_ptr.end() - 1);
        for (int32_t s = 0; s < ns; s++) P.level_list[fill[P.sn_level[s]]++] = s;
    }
    // small-front classes: f <= small_max/4, <= small_max/2, <= small_max
    P.small_class_fmax = {std::max(8, P.small_max / 4), std::max(16, P.small_max / 2), P.small_max};
    const int w = P.w;
    P.levels.resize(nlev);
    for (int32_t l = 0; l < nlev; l++) {
        LevelPlan &LP = P.levels[l];
        std::vector<int32_t> fronts(P.level_list.begin() + P.level_ptr[l], P.level_list.begin() + P.level_ptr[l + 1]);
        LP.small_class_off.assign(kSmallClasses + 1, 0);
        LP.small_class_off[0] = (int32_t)P.small_list.size();
        for (int cls = 0; cls < kSmallClasses; cls++) {
            int lo = cls == 0 ? 0 : P.small_class_fmax[cls - 1];
            for (int32_t s : fronts)
                if (P.sn_f[s] > lo && P.sn_f[s] <= P.small_class_fmax[cls]) P.small_list.push_back(s);
            LP.small_class_off[cls + 1] = (int32_t)P.small_list.size();
        }
        std::vector<int32_t> large;
        for (int32_t s : fronts)
            if (P.sn_f[s] > P.small_max) large.push_back(s);
        std::stable_sort(large.begin(), large.end(), [&](int32_t a, int32_t b) { return P.sn_k[a] > P.sn_k[b]; });
        LP.large_off = (int64_t)P.large_list.size();
        LP.nlarge = (int64_t)large.size();
        P.large_list.insert(P.large_list.end(), large.begin(), large.end());
        // assembly tasks
        LP.asm_off = (int64_t)P.asm_tasks.size() / 2;
        for (int32_t s : large)
            for (int32_t c0 = 0; c0 < P.sn_f[s]; c0 += kAsmCols) {
                P.asm_tasks.push_back(s);
                P.asm_tasks.push_back(c0);
            }
        LP.nasm = (int64_t)P.asm_tasks.size() / 2 - LP.asm_off;
        // waves over diagonal blocks of width w
        int32_t kmax = large.empty() ? 0 : P.sn_k[large[0]];
        for (int32_t j0 = 0; j0 < kmax; j0 += w) {
            LevelPlan::Wave W;
            W.j0 = j0;
            W.nactive = 0;
            while (W.nactive < (int32_t)large.size() && P.sn_k[large[W.nactive]] > j0) W.nactive++;
            W.trsm_off = (int64_t)P.trsm_tasks.size() / 2;
            W.prob_off = (int64_t)P.probs.size();
            W.tile_off = (int64_t)P.tiles.size();
            for (int32_t a = 0; a < W.nactive; a++) {
                int32_t s = large[a];
                int32_t k = P.sn_k[s], f = P.sn_f[s], ld = P.sn_ld[s];
                int32_t we = std::min(w, k - j0);
                for (int32_t r0 = j0 + we; r0 < f; r0 += kTrsmRows) {
                    P.trsm_tasks.push_back(s);
                    P.trsm_tasks.push_back(r0);
                }
                int32_t M = f - j0 - we, N = k - j0 - we;
                if (N > 0 && M > 0) {
                    GemmProb g;
                    g.a_off = P.L_off[s] + (int64_t)j0 * ld + (j0 + we);
                    g.c_off = P.L_off[s] + (int64_t)(j0 + we) * ld + (j0 + we);
                    g.lda = ld;
                    g.ldc = ld;
                    g.M = M;
                    g.N = N;
                    g.K = we;
                    g.c_in_U = 0;
                    int32_t pid = (int32_t)P.probs.size();
                    P.probs.push_back(g);
                    add_tiles(P, pid, M, N);
                }
            }
            W.ntrsm = (int64_t)P.trsm_tasks.size() / 2 - W.trsm_off;
            W.nprob = (int64_t)P.probs.size() - W.prob_off;
            W.ntile = (int64_t)P.tiles.size() - W.tile_off;
            LP.waves.push_back(W);
        }
        // final syrk on U^n with inner dimension k
        LP.syrk_prob_off = (int64_t)P.probs.size();
        LP.syrk_tile_off = (int64_t)P.tiles.size();
        for (int32_t s : large) {
            int32_t k = P.sn_k[s], f = P.sn_f[s], ld = P.sn_ld[s], m = f - k;
            if (m <= 0) continue;
            GemmProb g;
            g.a_off = P.L_off[s] + k;
            g.c_off = P.U_off[s];
            g.lda = ld;
            g.ldc = m;
            g.M = m;
            g.N = m;
            g.K = k;
            g.c_in_U = 1;
            int32_t pid = (int32_t)P.probs.size();
            P.probs.push_back(g);
            add_tiles(P, pid, m, m);
        }
        LP.syrk_nprob = (int64_t)P.probs.size() - LP.syrk_prob_off;
        LP.syrk_ntile = (int64_t)P.tiles.size() - LP.syrk_tile_off;
    }
    return MF_OK;
}

}  // namespace mf
