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
#include <cstdlib>
#include <map>
#include <set>
#include <cmath>
#include <functional>
#include <numeric>

#include "mf.h"
#include "mf_plan.h"

namespace mf {

// Tiles are emitted in bands of kTileBand tile columns, row-major inside a band,
// so the CTAs resident at one time cover a squarish block of the output and
// share both operand row panels in L2.
constexpr int32_t kTileBand = 16;
template <class Keep>
static void add_tiles(Plan &P, int32_t prob, int32_t M, int32_t N, Keep keep_col) {
    const int32_t tm = (M + kTileM - 1) / kTileM, tn = (N + kTileN - 1) / kTileN;
    for (int32_t tj0 = 0; tj0 < tn; tj0 += kTileBand)
        for (int32_t ti = 0; ti < tm; ti++)
            for (int32_t tj = tj0; tj < std::min(tn, tj0 + kTileBand); tj++) {
                // lower-trapezoid: skip tiles entirely above the diagonal (i < j everywhere)
                if ((int64_t)(ti + 1) * kTileM - 1 < (int64_t)tj * kTileN) continue;
                if (!keep_col(tj)) continue;
                P.tiles.push_back({prob, (ti << 16) | tj});
            }
}
static int64_t count_tiles(int32_t M, int32_t N) {
    const int32_t tm = (M + kTileM - 1) / kTileM, tn = (N + kTileN - 1) / kTileN;
    int64_t c = 0;
    for (int32_t tj = 0; tj < tn; tj++) c += std::max<int64_t>(0, tm - ((int64_t)tj * kTileN) / kTileM);
    return std::max<int64_t>(c, 1);
}
// Tile columns [tb[r], tb[r+1]) of an m x m lower syrk for rank r: contiguous
// ranges with (nearly) equal numbers of tiles.
static std::vector<int32_t> split_tile_columns(int32_t m, int R) {
    const int32_t tn = (m + kTileN - 1) / kTileN;
    std::vector<int64_t> w(tn);
    int64_t tot = 0;
    for (int32_t tj = 0; tj < tn; tj++) tot += (w[tj] = tn - tj);
    std::vector<int32_t> tb(R + 1, tn);
    tb[0] = 0;
    int64_t acc = 0;
    int r = 1;
    for (int32_t tj = 0; tj < tn && r < R; tj++) {
        acc += w[tj];
        while (r < R && acc * R >= tot * r) tb[r++] = tj + 1;
    }
    return tb;
}
// A top front is distributed over the ranks when it takes the tiled path and has
// at least two distribution blocks of pivot columns.
static bool dist_eligible(const Plan &P, int32_t s) {
    return P.sn_f[s] > P.small_max && P.sn_k[s] >= 2 * kDistLeaves * P.w;
}

// Solve program: per level, small supernodes in one batched launch; large ones
// (f > small_max) blocked by w columns so that no supernode is handled by a
// single CTA (the root of c5 has k = 14,900).
static void build_solve_plan(const Symbolic &S, Plan &P, const std::vector<char> &include,
                             std::vector<SolveLaunch> &fsolve, std::vector<SolveLaunch> &bsolve) {
    (void)S;
    const int w = P.w;
    std::vector<std::vector<int32_t>> large(P.nlevels), small(P.nlevels);
    static const int solve_small = [] {   // MF_SOLVE_SMALL: tuning override (<= kSolveSmallMax)
        const char *e = getenv("MF_SOLVE_SMALL");
        return e ? std::max(1, std::min(kSolveSmallMax, atoi(e))) : kSolveSmallMax;
    }();
    static const int solve_small_k = [] {   // MF_SOLVE_SMALL_K: above order 128, only fronts of k <= this
        const char *e = getenv("MF_SOLVE_SMALL_K");
        return e ? atoi(e) : kSolveSmallK;
    }();
    for (int32_t l = 0; l < P.nlevels; l++) {
        for (int32_t q = P.level_ptr[l]; q < P.level_ptr[l + 1]; q++) {
            const int32_t s = P.level_list[q];
            if (!include[s]) continue;
            const bool sm = P.sn_f[s] <= 128 || (P.sn_f[s] <= solve_small && P.sn_k[s] <= solve_small_k);
            (sm ? small[l] : large[l]).push_back(s);
        }
        std::stable_sort(large[l].begin(), large[l].end(),
                         [&](int32_t a, int32_t b) { return P.sn_k[a] > P.sn_k[b]; });
    }
    auto push_list = [&](const std::vector<int32_t> &v) {
        const int64_t off = (int64_t)P.solve_list.size();
        P.solve_list.insert(P.solve_list.end(), v.begin(), v.end());
        return off;
    };
    // dataflow solve of the large supernodes (kernels.cu): forward tasks = 64-row
    // blocks, backward tasks = w-column blocks; x slots of the backward sweep (one per
    // pivot column) and the inverses of the diagonal blocks
    auto bs_nseg = [&](int32_t s) {   // backward tail segments per column block (kernels.cu bsolve_cols_task)
        const int32_t ktop = (P.sn_k[s] - 1) / kSolveRowBlock, nsl = (P.sn_f[s] + kSolveRowBlock - 1) / kSolveRowBlock;
        const int32_t ntail = std::max(0, nsl - ktop - 1);
        return ntail > kSolveSegSlabs ? (ntail + kSolveSegSlabs - 1) / kSolveSegSlabs : 0;
    };
    auto ensure_df = [&](int32_t s) {
        if (P.df_part_off[s] >= 0) return;
        const int64_t nb = (P.sn_k[s] + w - 1) / w;
        P.dinv_off[s] = P.dinv_words;
        P.dinv_words += nb * 64 * 64;   // one 64 x 64 slot per block (w <= 64; identity-extended)
        for (int32_t b = 0; b < nb; b++) P.dinv_tasks.insert(P.dinv_tasks.end(), {s, b});
        P.df_part_off[s] = P.df_nparts;
        P.df_nparts += P.sn_k[s];
        if (const int32_t ns = bs_nseg(s)) {
            P.df_seg_off[s] = P.df_nseg_words;
            P.df_nseg_words += nb * ns * 64;
        }
    };
    // the deep register ring (1 CTA / SM) for levels whose largest front has several
    // blocks; the shallow one (3 CTAs / SM) for levels of small fronts
    auto deep_level = [&](const std::vector<int32_t> &v) {
        int32_t kmax = 0;
        for (int32_t s : v) kmax = std::max(kmax, P.sn_k[s]);
        return (int32_t)(kmax >= kSolveDeepK);
    };
    auto push_task = [&](int32_t s, int32_t t) {
        P.df_tasks.push_back(s);
        P.df_tasks.push_back(t);
    };
    auto push_init = [&](const std::vector<int32_t> &v) {   // (supernode, 2048-row part)
        const int64_t off = (int64_t)P.df_tasks.size() / 2;
        for (int32_t s : v)
            for (int32_t q = 0; q * kSolveInitRows < P.sn_f[s]; q++) push_task(s, q);
        return off;
    };
    static const int64_t fuse_init_max = [] {   // MF_SOLVE_FUSE_INIT: tuning override (0 = never fuse)
        const char *e = getenv("MF_SOLVE_FUSE_INIT");
        return e ? (int64_t)atoll(e) : (int64_t)kSolveFuseInitMax;
    }();
    for (int32_t l = 0; l < P.nlevels; l++) {
        if (!small[l].empty()) fsolve.push_back({SK_SMALL_F, 0, push_list(small[l]), (int64_t)small[l].size()});
        if (large[l].empty()) continue;
        int64_t ioff = push_init(large[l]), icnt = (int64_t)P.df_tasks.size() / 2 - ioff;
        if (icnt > fuse_init_max) {
            fsolve.push_back({SK_INIT_F, 0, ioff, icnt});
            ioff = icnt = 0;
        }
        // the pivot-row tasks of every front first, round robin (every chain starts at
        // once), then the rows below k; a task waits only on lower tickets of its front
        const int64_t off = (int64_t)P.df_tasks.size() / 2;
        int32_t maxrb = 0;
        for (int32_t s : large[l]) {
            ensure_df(s);
            maxrb = std::max(maxrb, (P.sn_k[s] + kSolveRowBlock - 1) / kSolveRowBlock);
        }
        for (int32_t rb = 0; rb < maxrb; rb++)
            for (int32_t s : large[l])
                if (rb * kSolveRowBlock < P.sn_k[s]) push_task(s, rb);
        for (int32_t s : large[l])
            for (int32_t rb = (P.sn_k[s] + kSolveRowBlock - 1) / kSolveRowBlock; rb * kSolveRowBlock < P.sn_f[s]; rb++)
                push_task(s, rb);
        fsolve.push_back({SK_DF_F, deep_level(large[l]), off, (int64_t)P.df_tasks.size() / 2 - off, ioff, icnt});
    }
    for (int32_t l = P.nlevels - 1; l >= 0; l--) {
        if (!large[l].empty()) {
            int64_t ioff = push_init(large[l]), icnt = (int64_t)P.df_tasks.size() / 2 - ioff;
            if (icnt > fuse_init_max) {
                bsolve.push_back({SK_INIT_B, 0, ioff, icnt});
                ioff = icnt = 0;
            }
            // the tail segments first (they wait for nothing), then the column blocks from
            // the last one down, round robin over the fronts
            const int64_t off = (int64_t)P.df_tasks.size() / 2;
            int32_t maxnb = 0;
            for (int32_t s : large[l]) {
                ensure_df(s);
                maxnb = std::max(maxnb, (P.sn_k[s] + w - 1) / w);
            }
            for (int32_t t = 0; t < maxnb; t++)
                for (int32_t s : large[l]) {
                    const int32_t nb = (P.sn_k[s] + w - 1) / w, ns = bs_nseg(s);
                    if (t < nb)
                        for (int32_t q = 1; q <= ns; q++) push_task(s, (nb - 1 - t) | (q << 16));
                }
            for (int32_t t = 0; t < maxnb; t++)
                for (int32_t s : large[l]) {
                    const int32_t nb = (P.sn_k[s] + w - 1) / w;
                    if (t < nb) push_task(s, nb - 1 - t);
                }
            bsolve.push_back({SK_DF_B, deep_level(large[l]), off, (int64_t)P.df_tasks.size() / 2 - off, ioff, icnt});
        }
        if (!small[l].empty()) bsolve.push_back({SK_SMALL_B, 0, push_list(small[l]), (int64_t)small[l].size()});
    }
}


// Subtree-to-GPU mapping (proportional/LPT): start from the
// tree roots as the frontier; repeatedly move the heaviest expandable frontier
// subtree's root into the "top" (its children join the frontier), assign the
// frontier subtrees to ranks by LPT on executed flops, and keep the frontier
// with the smallest makespan = max rank load + top load (the top starts after
// every frontier root's update matrix has arrived; its large fronts are shared by
// all ranks, the rest is replicated).
// Cost model of a top front, in flop-equivalents at ~30 TF/s: replicated = its
// flops; cooperative = flops / R + one exchange latency (~30 us) per distribution
// block + its broadcast bytes (L panel and U^n, ~400 GB/s effective).
constexpr double kXchgLatency = 9e8, kXchgPerByte = 75.0;
static double coop_cost(const Plan &P, int32_t s, double load) {
    if (!dist_eligible(P, s)) return 1e300;
    if (P.split_all) return load / P.nranks;   // no exchange cost: every eligible top front is shared
    const double k = P.sn_k[s], f = P.sn_f[s], m = f - k;
    const double nb = std::ceil(k / (kDistLeaves * P.w));
    return load / P.nranks + kXchgLatency * nb + kXchgPerByte * 8.0 * (f * k + m * m / 2);
}

static void map_subtrees(Plan &P, const std::vector<double> &front_load) {
    const int32_t ns = P.nsuper, R = P.nranks;
    P.owner.assign(ns, 0);
    P.top.assign(ns, 0);
    P.dist.assign(ns, 0);
    P.frontier_roots.clear();
    P.rank_load.assign(R, 0.0);
    P.top_load = 0;
    std::vector<double> sub(front_load);
    for (int32_t s = 0; s < ns; s++)
        for (int32_t q = P.child_ptr[s]; q < P.child_ptr[s + 1]; q++) sub[s] += sub[P.child_list[q]];
    std::vector<int32_t> roots;
    std::vector<int32_t> parent(ns, -1);
    for (int32_t s = 0; s < ns; s++)
        for (int32_t q = P.child_ptr[s]; q < P.child_ptr[s + 1]; q++) parent[P.child_list[q]] = s;
    for (int32_t s = 0; s < ns; s++)
        if (parent[s] < 0) roots.push_back(s);
    if (R <= 1) {
        P.rank_load[0] = 0;
        for (int32_t r : roots) P.rank_load[0] += sub[r];
        return;
    }
    auto lpt = [&](const std::vector<int32_t> &fr, std::vector<int32_t> &assign, std::vector<double> &load) {
        std::vector<int32_t> ord(fr.size());
        std::iota(ord.begin(), ord.end(), 0);
        std::stable_sort(ord.begin(), ord.end(), [&](int32_t a, int32_t b) { return sub[fr[a]] > sub[fr[b]]; });
        load.assign(R, 0.0);
        assign.assign(fr.size(), 0);
        for (int32_t i : ord) {
            int32_t best = 0;
            for (int32_t r = 1; r < R; r++)
                if (load[r] < load[best]) best = r;
            assign[i] = best;
            load[best] += sub[fr[i]];
        }
        return *std::max_element(load.begin(), load.end());
    };
    std::vector<int32_t> fr = roots, best_fr = roots, assign, best_assign;
    std::vector<double> load, best_load;
    std::vector<char> is_top(ns, 0), best_top(ns, 0);
    double topl = 0, best_make = lpt(fr, best_assign, best_load);
    for (int iter = 0; iter < 64 * R && (int)fr.size() < 64 * R; iter++) {
        int32_t pick = -1;
        for (size_t i = 0; i < fr.size(); i++)
            if (P.child_ptr[fr[i] + 1] > P.child_ptr[fr[i]] && (pick < 0 || sub[fr[i]] > sub[fr[pick]])) pick = (int32_t)i;
        if (pick < 0) break;
        const int32_t v = fr[pick];
        fr.erase(fr.begin() + pick);
        is_top[v] = 1;
        topl += std::min(front_load[v], coop_cost(P, v, front_load[v]));   // cooperative or replicated
        for (int32_t q = P.child_ptr[v]; q < P.child_ptr[v + 1]; q++) fr.push_back(P.child_list[q]);
        double bc = 0;   // broadcast of the frontier roots' update matrices
        for (int32_t r : fr) {
            const double m = P.sn_f[r] - P.sn_k[r];
            bc += kXchgLatency / 8 + kXchgPerByte * 8.0 * m * (m + 1) / 2;   // packed lower U^c
        }
        const double make = lpt(fr, assign, load) + topl + bc;
        // split_all: the first frontier with >= R subtrees wins, whatever the model says
        const bool forced = P.split_all && (int)best_fr.size() < R && (int)fr.size() >= R;
        if (forced || (make < best_make && !(P.split_all && (int)fr.size() < R && (int)best_fr.size() >= R))) {
            best_make = make;
            best_fr = fr;
            best_assign = assign;
            best_load = load;
            best_top = is_top;
        }
    }
    P.top = best_top;
    P.rank_load = best_load;
    for (int32_t s = 0; s < ns; s++)
        if (P.top[s]) {
            P.top_load += front_load[s];
            P.dist[s] = coop_cost(P, s, front_load[s]) < front_load[s];
        }
    // owner of every supernode below the frontier = owner of its frontier root
    for (size_t i = 0; i < best_fr.size(); i++) {
        const int32_t rt = best_fr[i];
        P.frontier_roots.push_back(rt);
        std::vector<int32_t> stack{rt};
        while (!stack.empty()) {
            const int32_t v = stack.back();
            stack.pop_back();
            P.owner[v] = best_assign[i];
            for (int32_t q = P.child_ptr[v]; q < P.child_ptr[v + 1]; q++) stack.push_back(P.child_list[q]);
        }
    }
    std::sort(P.frontier_roots.begin(), P.frontier_roots.end());
}

// Single GPU: split the elimination tree into concurrent branches (the paper's
// task parallelism over independent subtrees [PAPER.md L443, L797], here as CUDA-
// graph branches on their own streams of ONE GPU).  The heaviest expandable
// frontier subtree is moved into the "top" until the frontier holds >= B
// subtrees; those are assigned to B branches by LPT on executed flops.  The top
// fronts run on the main stream after every branch has finished.  While one
// branch runs latency-bound work (pivot chains, small fronts, narrow updates,
// assembly), the others keep the DMMA pipes busy.
static void assign_branches(Plan &P, const std::vector<double> &front_load, int B) {
    const int32_t ns = P.nsuper;
    P.branch.assign(ns, -1);
    P.nbranch = 1;
    if (B <= 1 || ns == 0) return;
    std::vector<double> sub(front_load);
    std::vector<int32_t> parent(ns, -1);
    for (int32_t s = 0; s < ns; s++)
        for (int32_t q = P.child_ptr[s]; q < P.child_ptr[s + 1]; q++) {
            sub[s] += sub[P.child_list[q]];
            parent[P.child_list[q]] = s;
        }
    std::vector<int32_t> fr;
    for (int32_t s = 0; s < ns; s++)
        if (parent[s] < 0) fr.push_back(s);
    while ((int)fr.size() < B) {
        int32_t pick = -1;
        for (size_t i = 0; i < fr.size(); i++)
            if (P.child_ptr[fr[i] + 1] > P.child_ptr[fr[i]] && (pick < 0 || sub[fr[i]] > sub[fr[pick]]))
                pick = (int32_t)i;
        if (pick < 0) break;
        const int32_t v = fr[pick];
        fr.erase(fr.begin() + pick);
        for (int32_t q = P.child_ptr[v]; q < P.child_ptr[v + 1]; q++) fr.push_back(P.child_list[q]);
    }
    if (fr.size() < 2) return;   // nothing to run concurrently: one stream
    const int nb = std::min<int>(B, (int)fr.size());
    std::stable_sort(fr.begin(), fr.end(), [&](int32_t a, int32_t b) { return sub[a] > sub[b]; });
    std::vector<double> load(nb, 0.0);
    for (int32_t rt : fr) {
        const int b = (int)(std::min_element(load.begin(), load.end()) - load.begin());
        load[b] += sub[rt];
        std::vector<int32_t> stack{rt};
        while (!stack.empty()) {
            const int32_t v = stack.back();
            stack.pop_back();
            P.branch[v] = b;
            for (int32_t q = P.child_ptr[v]; q < P.child_ptr[v + 1]; q++) stack.push_back(P.child_list[q]);
        }
    }
    P.nbranch = nb;
}

// U-arena liveness (single GPU): U^s is written at front s's level and read only
// by its parent (assembly of the panel columns and the syrk prologue's gather, or
// the parent's small-front kernel) at the parent's level, in the same stream or,
// for a branch root, in the top pass after the branches joined.  Slots are
// therefore recycled level by level with a first-fit allocator: each concurrent
// branch in its own region (branches run concurrently), the top pass over the
// whole arena minus the frontier roots' still-live slots.  Only offsets change.
static void plan_u_reuse(Plan &P) {
    const int32_t ns = P.nsuper;
    auto words = [&](int32_t s) -> int64_t {   // packed lower U^s (mf_plan.h upk)
        const int64_t m = P.sn_f[s] - P.sn_k[s], w = m * (m + 1) / 2;
        return w + (w & 1);
    };
    std::vector<int64_t> off(ns, -1);
    // free list indexed both ways: by offset (coalescing neighbours on release) and
    // by length (best fit in O(log n) -- a first-fit scan over the offset map cost
    // ~10 s of analyze on c2's 255k supernodes)
    std::map<int64_t, int64_t> freel;                 // offset -> length
    std::multimap<int64_t, int64_t> bylen;            // length -> offset
    int64_t hw = 0;                                   // high-water mark of the current allocator
    auto drop_len = [&](int64_t o, int64_t len) {
        auto r = bylen.equal_range(len);
        for (auto it = r.first; it != r.second; ++it)
            if (it->second == o) {
                bylen.erase(it);
                return;
            }
    };
    auto put = [&](int64_t o, int64_t len) {
        freel[o] = len;
        bylen.emplace(len, o);
    };
    auto clear_free = [&]() {
        freel.clear();
        bylen.clear();
    };
    auto alloc = [&](int64_t len) -> int64_t {
        auto it = bylen.lower_bound(len);             // smallest free block that fits
        if (it != bylen.end()) {
            const int64_t o = it->second, rem = it->first - len;
            bylen.erase(it);
            freel.erase(o);
            if (rem) put(o + len, rem);
            return o;
        }
        const int64_t o = hw;
        hw += len;
        return o;
    };
    auto release = [&](int64_t o, int64_t len) {
        auto nx = freel.lower_bound(o);
        if (nx != freel.end() && o + len == nx->first) {   // merge with the next block
            len += nx->second;
            drop_len(nx->first, nx->second);
            freel.erase(nx);
        }
        auto it = freel.lower_bound(o);
        if (it != freel.begin()) {
            auto pv = std::prev(it);
            if (pv->first + pv->second == o) {              // merge into the previous block
                drop_len(pv->first, pv->second);
                o = pv->first;
                len += pv->second;
                freel.erase(pv);
            }
        }
        put(o, len);
    };
    auto run_group = [&](int32_t g) {
        for (int32_t l = 0; l < P.nlevels; l++) {
            for (int32_t q = P.level_ptr[l]; q < P.level_ptr[l + 1]; q++) {
                const int32_t s = P.level_list[q];
                if (P.branch[s] != g) continue;
                off[s] = words(s) > 0 ? alloc(words(s)) : 0;
            }
            for (int32_t q = P.level_ptr[l]; q < P.level_ptr[l + 1]; q++) {   // children consumed at level l
                const int32_t s = P.level_list[q];
                if (P.branch[s] != g) continue;
                for (int32_t c = P.child_ptr[s]; c < P.child_ptr[s + 1]; c++) {
                    const int32_t ch = P.child_list[c];
                    if (words(ch) > 0 && off[ch] >= 0) release(off[ch], words(ch));
                }
            }
        }
    };
    int64_t total = 0;
    std::vector<std::pair<int64_t, int64_t>> live;   // branch roots' slots, live into the top pass
    for (int32_t b = 0; b < (P.nbranch > 1 ? P.nbranch : 0); b++) {
        clear_free();
        hw = 0;
        run_group(b);
        for (int32_t s = 0; s < ns; s++)   // shift the branch's region behind the previous ones
            if (P.branch[s] == b && off[s] >= 0 && words(s) > 0) off[s] += total;
        total += hw;
    }
    // top pass (or everything, without branches): the whole arena is free except
    // the slots of branch fronts whose parent is a top front
    clear_free();
    for (int32_t s = 0; s < ns; s++)
        if (P.branch[s] < 0)
            for (int32_t c = P.child_ptr[s]; c < P.child_ptr[s + 1]; c++) {
                const int32_t ch = P.child_list[c];
                if (P.branch[ch] >= 0 && words(ch) > 0) live.emplace_back(off[ch], words(ch));
            }
    std::sort(live.begin(), live.end());
    int64_t cur = 0;
    for (auto &iv : live) {
        if (iv.first > cur) put(cur, iv.first - cur);
        cur = std::max(cur, iv.first + iv.second);
    }
    if (total > cur) put(cur, total - cur);
    hw = total;
    run_group(-1);
    for (int32_t s = 0; s < ns; s++) P.U_off[s] = off[s] >= 0 ? off[s] : 0;
    P.U_words = hw + 2;
}

// Ozaki-scheme Schur updates (csrc/ozaki_update.cuh): every
// KC_UPDATE launch whose average inner dimension is long enough for the int8
// tensor cores to beat FP64 DMMA (the split pass and the TMEM epilogue are paid
// per launch and per tile) is given an Ozaki form: its problems (rows padded to
// 128, K to 64), the (problem, 128-row block, k segment) split tasks and its
// 128 x 64 tiles -- the union of its 64 x 64 DMMA tiles, so partial tile sets
// (multi-GPU column ownership) carry over.  Slices live in a scratch region per
// stream (branches run concurrently), sized for the largest launch of the stream.
constexpr double kOzMinK = 2048;   // measured per launch on c5 (tools/oz_launches.py): DMMA wins below
static int plan_ozaki(Plan &P, int S) {
    P.oz_slices = S;
    if (S <= 0) return MF_OK;
    auto up = [](int64_t x, int64_t a) { return (x + a - 1) / a * a; };
    std::map<int32_t, std::pair<int64_t, int64_t>> region;   // stream -> (slice bytes, exponent words)
    std::vector<std::pair<std::vector<Launch> *, size_t>> conv;
    // reduced slices need fewer pair MMAs per tile: they beat DMMA from K ~ 1024 (c5, S = 3 / 4:
    // 153.6 / 160.9 ms at 1024 vs 167.7 / 172.7 ms at 2048 and 158.7 / 167.8 at 512)
    double min_k = S >= 7 ? kOzMinK : 1024;   // MF_OZ_MIN_K: tests drive small problems through the int8 path
    if (const char *e = getenv("MF_OZ_MIN_K")) min_k = atof(e);
    for (std::vector<Launch> *prog : {&P.program, &P.program_top}) {
        for (size_t li = 0; li < prog->size(); li++) {
            Launch &L = (*prog)[li];
            if (L.kind != KC_UPDATE || L.count == 0) continue;
            if (L.flops / (2.0 * kTileM * kTileN * L.count) < min_k) continue;
            std::vector<int32_t> probs;
            std::map<int32_t, int32_t> local;
            bool ok = true;
            for (int64_t t = L.off; t < L.off + L.count; t++) {
                const int32_t p = P.tiles[t].prob;
                if (local.emplace(p, (int32_t)probs.size()).second) probs.push_back(p);
            }
            for (int32_t p : probs)
                if (P.probs[p].K > kOzMaxK) ok = false;
            if (!ok) continue;
            L.oz = 1;
            L.oz_p = (int64_t)P.oz_probs.size();
            L.oz_np = (int64_t)probs.size();
            int64_t bytes = 0, words = 0;
            for (int32_t p : probs) {
                const GemmProb &g = P.probs[p];
                OzProb o{p, (int32_t)up(g.M, kOzBM), (int32_t)up(g.K, kOzBK), 0, bytes, words};
                bytes += (int64_t)S * o.Mpad * o.Kpad;
                words += o.Mpad;
                P.oz_probs.push_back(o);
            }
            L.oz_s = (int64_t)P.oz_split.size() / 3;
            for (int64_t q = 0; q < L.oz_np; q++) {
                const OzProb &o = P.oz_probs[L.oz_p + q];
                for (int32_t rb = 0; rb < o.Mpad / kOzBM; rb++)
                    for (int32_t sg = 0; sg < (o.Kpad + kOzSeg - 1) / kOzSeg; sg++)
                        P.oz_split.insert(P.oz_split.end(), {(int32_t)(L.oz_p + q), rb, sg});
            }
            L.oz_ns = (int64_t)P.oz_split.size() / 3 - L.oz_s;
            // 128 x 128 tiles (two-pass kernel) when every problem of the launch is
            // computed whole; a launch with a partial tile set (multi-GPU column
            // ownership) keeps the DMMA tile columns with 128 x 64 tiles
            std::map<int32_t, int64_t> have;
            for (int64_t t = L.off; t < L.off + L.count; t++) have[P.tiles[t].prob]++;
            bool whole = true;
            for (int32_t p : probs) whole = whole && have[p] == count_tiles(P.probs[p].M, P.probs[p].N);
            // (measured, tools/ubench/ozaki_gemm.cu: with S <= 4 the single-pass wide kernel is
            // 1.4x the 128 x 64 one; with S = 8 both move the same slice bytes per output
            // from L2 and run alike, so the narrow kernel stays)
            // (and only without the fused extend-add gather: its epilogue gathers the
            // children through global read-modify-writes, which ate the gain on c5)
            bool gath = false;
            for (int32_t p : probs) gath = gath || (P.probs[p].flags & kProbGather);
            L.oz_wide = (whole && S <= 4 && !gath) ? 1 : 0;
            const int32_t bn = L.oz_wide ? 128 : kOzBN;
            L.oz_t = (int64_t)P.oz_tiles.size();
            std::set<std::pair<int32_t, int32_t>> seen;
            for (int64_t t = L.off; t < L.off + L.count; t++) {
                const TileTask &tt = P.tiles[t];
                static_assert(kTileN == kOzBN, "Ozaki tiles keep the DMMA tile columns");
                const int32_t q = local[tt.prob];
                const int32_t tij = (((tt.tij >> 16) * kTileM / kOzBM) << 16) | ((tt.tij & 0xffff) * kTileN / bn);
                if (seen.emplace(q, tij).second) P.oz_tiles.push_back(OzTile{(int32_t)(L.oz_p + q), tij});
            }
            L.oz_nt = (int64_t)P.oz_tiles.size() - L.oz_t;
            for (int64_t t = L.oz_t; t < L.oz_t + L.oz_nt; t++)
                L.int8_ops += 2.0 * kOzBM * bn * (double)P.oz_probs[P.oz_tiles[t].oprob].Kpad * (S * (S + 1) / 2);
            L.oz_ne = words;
            auto &rg = region[L.stream];
            rg.first = std::max(rg.first, bytes);
            rg.second = std::max(rg.second, words);
            conv.emplace_back(prog, li);
        }
    }
    std::map<int32_t, std::pair<int64_t, int64_t>> base;
    int64_t tb = 0, tw = 0;
    for (auto &kv : region) {
        base[kv.first] = {tb, tw};
        tb += up(kv.second.first, 1024);
        tw += up(kv.second.second, 32);
    }
    for (auto &c : conv) {
        Launch &L = (*c.first)[c.second];
        const auto b = base[L.stream];
        for (int64_t q = L.oz_p; q < L.oz_p + L.oz_np; q++) P.oz_probs[q].sl_off += b.first;
        L.oz_e = b.second;   // ex_off stays relative to the launch's exponent region
    }
    P.oz_scratch_bytes = tb;
    P.oz_expo_words = tw;
    return MF_OK;
}

int build_plan(const Symbolic &S, const Options &opt, Plan &P) {
    P = Plan();
    const int32_t ns = (int32_t)S.sn_parent.size();
    P.nsuper = ns;
    P.nranks = std::max(1, opt.nranks);
    P.rank = opt.rank;
    P.w = opt.panel_w;
    P.small_max = opt.small_front_max;
    P.split_all = opt.split_all;
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
        int64_t uw = (int64_t)m * (m + 1) / 2;   // packed lower (mf_plan.h upk)
        uoff += uw + (uw & 1);
        P.fv_off[s] = fvoff;
        fvoff += f + (f & 1);
        P.max_front = std::max(P.max_front, f);
        // epoch-tagged leaf / panel flags hold the diagonal-block index in 16 bits
        if (k / std::max(1, opt.panel_w) >= 0xffff) return MF_ERR_ARG;
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
    // (<= 16 and <= 32: one warp per front; <= 64 and <= small_max: one CTA per front)
    // (+ <= 96 when small_max > 96: 74 KB of shared memory, 3 CTAs / SM instead of
    // the 1 that a 128-order front's 132 KB allows; c2 has ~4k such fronts per level)
    P.small_class_fmax = {std::min(16, P.small_max), std::min(32, P.small_max), std::min(64, P.small_max),
                          std::min(96, P.small_max), P.small_max};
    // kernel variant per front: the learned selector y(x) = argmax_j x . theta_j over
    // the feasible classes (Eq. 5), a forced class, or the default
    // front-order thresholds (the analogue of the paper's baseline P_BH, L401).
    // front_fmax = the order bound of the class's shared-memory / warp kernel, 0 = tiled.
    std::vector<int32_t> front_fmax(ns, 0);
    P.variant.assign(ns, kVariantTiled);
    for (int32_t s = 0; s < ns; s++) {
        const int32_t f = P.sn_f[s], k = P.sn_k[s];
        auto feasible = [&](int j) { return j == kVariantTiled || f <= kVariantFmax[j]; };
        int v = -1;
        if (opt.force_variant >= 0 && opt.force_variant < kVariants && feasible(opt.force_variant)) {
            v = opt.force_variant;
        } else if ((int)opt.variant_theta.size() == kVariantFeatures * kVariants) {
            double x[kVariantFeatures], best = -1e300;
            variant_features(f - k, k, x);
            for (int j = 0; j < kVariants; j++) {
                if (!feasible(j)) continue;
                double sc = 0;
                for (int q = 0; q < kVariantFeatures; q++) sc += x[q] * opt.variant_theta[q * kVariants + j];
                if (sc > best) {
                    best = sc;
                    v = j;
                }
            }
        }
        if (v >= 0) {
            P.variant[s] = v;
            front_fmax[s] = kVariantFmax[v];
        } else if (f <= P.small_max) {
            for (int cls = 0; cls < kSmallClasses; cls++)
                if (f <= P.small_class_fmax[cls]) {
                    front_fmax[s] = P.small_class_fmax[cls];
                    break;
                }
            P.variant[s] = kVariantTiled;
            for (int j = 0; j < kVariantTiled; j++)
                if (front_fmax[s] <= kVariantFmax[j]) {
                    P.variant[s] = j;
                    break;
                }
        }
    }
    std::vector<int32_t> fmax_classes;
    for (int32_t s = 0; s < ns; s++)
        if (front_fmax[s] > 0) fmax_classes.push_back(front_fmax[s]);
    std::sort(fmax_classes.begin(), fmax_classes.end());
    fmax_classes.erase(std::unique(fmax_classes.begin(), fmax_classes.end()), fmax_classes.end());
    const int w = P.w;
    // algorithmic bytes of assembling front s: its A entries (value + index), the
    // children's U^c lower triangles and relative maps (read once)
    auto asm_bytes = [&](int32_t s) {
        double b = 0;
        const int64_t e0 = S.bcolptr[S.sn_first[s]], e1 = S.bcolptr[S.sn_first[s + 1]];
        b += (double)(e1 - e0) * (8 + 4);
        for (int32_t q = P.child_ptr[s]; q < P.child_ptr[s + 1]; q++) {
            const double mc = P.sn_f[P.child_list[q]] - P.sn_k[P.child_list[q]];
            b += 8.0 * mc * (mc + 1) / 2 + 4.0 * mc;
        }
        return b;
    };
    // fused extend-add: child c's relative map positions below the parent's pivot
    // columns: np = #rows of U^c landing in panel columns (a prefix: rel is
    // increasing); its lower entries in panel columns = np mc - np (np - 1) / 2
    auto child_np = [&](int32_t c, int32_t kp) -> int64_t {
        const int32_t *rel = P.relmap.data() + P.relmap_ptr[c];
        const int32_t mc = P.sn_f[c] - P.sn_k[c];
        return std::lower_bound(rel, rel + mc, kp) - rel;
    };
    auto child_panel_entries = [&](int32_t c, int32_t kp) {
        const double np = (double)child_np(c, kp), mc = P.sn_f[c] - P.sn_k[c];
        return np * mc - np * (np - 1) / 2;
    };
    // assembly bytes of the panel columns only (the U^s part is gathered by the syrk)
    auto asm_bytes_panel = [&](int32_t s) {
        const int64_t e0 = S.bcolptr[S.sn_first[s]], e1 = S.bcolptr[S.sn_first[s + 1]];
        double b = (double)(e1 - e0) * (8 + 4);
        for (int32_t q = P.child_ptr[s]; q < P.child_ptr[s + 1]; q++) {
            const int32_t c = P.child_list[q];
            b += 8.0 * child_panel_entries(c, P.sn_k[s]) + 4.0 * (P.sn_f[c] - P.sn_k[c]);
        }
        return b;
    };
    P.fuse_ea = opt.fuse_ea ? 1 : 0;
    auto panel_words = [&](int32_t s) {
        const double k = P.sn_k[s], m = P.sn_f[s] - P.sn_k[s];
        return k * (k + 1) / 2 + k * m;
    };
    auto upd_flops = [](double M, double N, double K) { return 2.0 * K * (N * (N + 1) / 2 + (M - N) * N); };
    auto upd_bytes = [](double M, double N, double K) { return 8.0 * (M * K + 2 * (N * (N + 1) / 2 + (M - N) * N)); };
    // ---- subtree-to-GPU mapping and the per-rank inclusion masks
    {
        std::vector<double> front_load(ns);
        for (int32_t s = 0; s < ns; s++) {
            const double k = P.sn_k[s], m = P.sn_f[s] - P.sn_k[s];
            front_load[s] = k * m * m + m * k * (k + 1) + k * (k + 1) * (2 * k + 1) / 6;
        }
        map_subtrees(P, front_load);
        if (P.nranks == 1) assign_branches(P, front_load, opt.nbranch);
        else P.branch.assign(ns, -1);
    }
    // U-slot recycling (single GPU; multi-GPU exchanges address the U arena by
    // supernode and keep disjoint slots).  MF_U_REUSE=0 disables it (A/B checks).
    {
        const char *e = getenv("MF_U_REUSE");
        if (P.nranks == 1 && (!e || atoi(e) != 0)) plan_u_reuse(P);
    }
    // Inclusion masks.  Local program: the supernodes of this rank's subtrees.  Top
    // program (multi-GPU): EVERY rank holds a replica of every top front; the
    // pivot-column blocks of the large top fronts are owned block-cyclically (the
    // owner factors a block and broadcasts it), the trailing updates are split by
    // owned column, and the syrk on U^n by contiguous column ranges (all-gathered
    // by broadcasts), so the top's flops are divided over the ranks.
    const int R = P.nranks;
    const int32_t Wd = kDistLeaves * w;   // distribution block: kDistLeaves leaves of w columns
    std::vector<char> inc_local(ns), inc_top(ns), inc_top_solve(ns);
    for (int32_t s = 0; s < ns; s++) {
        inc_local[s] = !P.top[s] && P.owner[s] == P.rank;
        inc_top[s] = P.top[s] && R > 1;
        inc_top_solve[s] = P.top[s] && P.rank == 0;   // the top solve stays on rank 0
        if (P.top[s]) P.top_list.push_back(s);                            // every rank: y columns broadcast by rank 0
        if (inc_local[s] || inc_top_solve[s]) P.own_list.push_back(s);   // columns this rank finalises in the solve
    }
    auto blk_owner = [&](int32_t s, int32_t t) -> int32_t { return P.dist[s] ? (t + s) % R : -1; };
    auto blk_mine = [&](int32_t s, int32_t t) { const int32_t o = blk_owner(s, t); return o < 0 || o == P.rank; };
    std::vector<Launch> *cur = &P.program;
    // the update of the pivot-column leaves [mid, b) by the factored leaves [a, mid)
    // (units of w) for the fronts fl (sorted by k descending): one DMMA launch with
    // inner dimension (mid - a) w; tiles of global column col only if keep(s, col)
    // look-ahead bookkeeping: the next main-stream launch after a panel that ran
    // beside a side-stream update must join the side stream
    bool need_join = false, join_armed = false;
    auto push = [&](Launch L) {
        if (join_armed && !L.side) {
            L.join = 1;
            join_armed = need_join = false;
        }
        cur->push_back(L);
    };
    // the update of the pivot-column leaves [jlo, b) (default jlo = mid) by the
    // factored leaves [a, mid) (units of w)
    auto rec_update_cols = [&](const std::vector<int32_t> &fl, int32_t a, int32_t mid, int32_t jlo, int32_t b,
                               int32_t l, const std::function<bool(int32_t, int32_t)> &keep, int32_t side) {
        const int32_t c0 = jlo * w, c_lo = a * w;
        Launch Lu{KC_UPDATE, 0, (int64_t)P.tiles.size(), 0, 0.0, 0.0, l};
        Lu.side = side;
        for (int32_t s : fl) {
            const int32_t k = P.sn_k[s], f = P.sn_f[s], ld = P.sn_ld[s];
            if (k <= c0) continue;
            const int32_t M = f - c0, N = std::min(b * w, k) - c0, K = mid * w - c_lo;
            if (M <= 0 || N <= 0) continue;
            GemmProb g;
            g.a_off = P.L_off[s] + (int64_t)c_lo * ld + c0;
            g.c_off = P.L_off[s] + (int64_t)c0 * ld + c0;
            g.lda = ld;
            g.ldc = ld;
            g.M = M;
            g.N = N;
            g.K = K;
            g.flags = 0;
            const int32_t pid = (int32_t)P.probs.size();
            P.probs.push_back(g);
            const int64_t t0 = (int64_t)P.tiles.size();
            add_tiles(P, pid, M, N, [&](int32_t tj) { return keep(s, c0 + tj * kTileN); });
            const int64_t nt = (int64_t)P.tiles.size() - t0;
            if (nt == 0) {
                P.probs.pop_back();
                continue;
            }
            const double frac = (double)nt / (double)count_tiles(M, N);
            Lu.flops += frac * upd_flops(M, N, K);
            Lu.bytes += frac * upd_bytes(M, N, K);
        }
        Lu.count = (int64_t)P.tiles.size() - Lu.off;
        if (Lu.count) push(Lu);
        return Lu.count > 0;
    };
    auto rec_update = [&](const std::vector<int32_t> &fl, int32_t a, int32_t mid, int32_t b, int32_t l,
                          const std::function<bool(int32_t, int32_t)> &keep) {
        rec_update_cols(fl, a, mid, mid, b, l, keep, 0);
    };
    bool lookahead_pass = false;
    auto keep_all = [](int32_t, int32_t) { return true; };
    // the blocked factorization of the pivot-column leaves [a, b) (units of w) of the
    // fronts fl (sorted by k descending, stored at P.large_list[loff..])
    // the dataflow panel of the leaves [a, b) (b - a <= kPanelMaxBlocks, w = 64):
    // tasks = 64-row tile rows from j0 down, row-major over the active fronts
    auto emit_panel = [&](const std::vector<int32_t> &fl, int32_t a, int32_t b, int32_t l) {
        const int32_t j0 = a * w, j1 = b * w;
        std::vector<int32_t> act;
        int32_t maxc = 0;
        for (int32_t s : fl)
            if (P.sn_k[s] > j0) {
                act.push_back(s);
                maxc = std::max(maxc, (P.sn_f[s] - j0 + 63) / 64);
            }
        if (act.empty()) return;
        Launch Lp{KC_PANEL, j0, (int64_t)P.panel_tasks.size() / 2, 0, 0.0, 0.0, l};
        Lp.count2 = b - a;
        for (int32_t c = 0; c < maxc; c++)
            for (int32_t s : act)
                if (j0 + 64 * c < P.sn_f[s]) {
                    P.panel_tasks.push_back(s);
                    P.panel_tasks.push_back(c);
                }
        for (int32_t s : act) {
            const double f = P.sn_f[s];
            const int32_t je = std::min(P.sn_k[s], j1);
            for (int32_t j = j0; j < je; j++) {   // column j: scale (f - j) entries, update columns j+1 .. je-1
                Lp.flops += f - j;
                for (int32_t cc = j + 1; cc < je; cc++) Lp.flops += 2.0 * (f - cc);
            }
            Lp.bytes += 16.0 * (f - j0) * (je - j0);
        }
        Lp.count = (int64_t)P.panel_tasks.size() / 2 - Lp.off;
        push(Lp);
        if (need_join) join_armed = true;   // the side update must finish before the next main launch
    };
    std::function<void(const std::vector<int32_t> &, int64_t, int32_t, int32_t, int32_t)> rec =
        [&](const std::vector<int32_t> &fl, int64_t loff, int32_t a, int32_t b, int32_t l) {
        if (w == 64 && b - a <= kPanelMaxBlocks) {
            emit_panel(fl, a, b, l);
            return;
        }
        if (b - a == 1) {
            const int32_t j0 = a * w;
            int32_t na = 0;   // fronts (prefix of fl) with k > j0
            while (na < (int32_t)fl.size() && P.sn_k[fl[na]] > j0) na++;
            if (na == 0) return;
            Launch Lp{KC_POTRF, j0, loff, na, 0.0, 0.0, l};
            Launch Lt{KC_TRSM, j0, (int64_t)P.trsm_tasks.size() / 2, 0, 0.0, 0.0, l};
            for (int32_t q = 0; q < na; q++) {
                const int32_t s = fl[q];
                const int32_t k = P.sn_k[s], f = P.sn_f[s];
                const int32_t we = std::min(w, k - j0);
                Lp.flops += (double)we * (we + 1) * (2.0 * we + 1) / 6;
                Lp.bytes += 8.0 * we * (we + 1);
                for (int32_t r0 = j0 + we; r0 < f; r0 += kTrsmRows) {
                    P.trsm_tasks.push_back(s);
                    P.trsm_tasks.push_back(r0);
                }
                const double rows = f - j0 - we;
                Lt.flops += rows * we * we;
                Lt.bytes += 8.0 * (2 * rows * we + (double)we * (we + 1) / 2);
            }
            Lt.count = (int64_t)P.trsm_tasks.size() / 2 - Lt.off;
            if (na <= kFuseLeafMaxFronts && Lt.count) {   // one launch: potrf CTAs + flag-waiting trsm CTAs
                Launch Lf{KC_LEAF, j0, Lp.off, Lp.count, Lp.flops + Lt.flops, Lp.bytes + Lt.bytes, l};
                Lf.off2 = Lt.off;
                Lf.count2 = Lt.count;
                push(Lf);
                return;
            }
            push(Lp);
            if (Lt.count) push(Lt);
            return;
        }
        const int32_t mid = a + (b - a + 1) / 2;
        rec(fl, loff, a, mid, l);
        // look-ahead: the first panel of rec(mid, b) covers the leaves [mid, f1); only
        // those columns of the update are on its critical path.  The rest [f1, b) runs
        // on the side stream, beside that panel, and is joined before the next launch.
        int32_t f1 = b;
        if (lookahead_pass && w == 64 && !need_join) {
            f1 = mid;
            int32_t bb = b;
            while (bb - f1 > kPanelMaxBlocks) bb = f1 + (bb - f1 + 1) / 2;
            f1 = bb;
        }
        if (f1 < b) {
            // the side part is forked AFTER the critical part: when that finishes, the
            // panel (high priority) and the side update become ready together, and the
            // panel's CTAs are placed first (the side's long-K tiles would otherwise
            // hold every SM slot for up to a millisecond)
            rec_update_cols(fl, a, mid, mid, f1, l, keep_all, 0);
            if (rec_update_cols(fl, a, mid, f1, b, l, keep_all, 1)) {
                need_join = true;
                P.nside++;
            }
        } else {
            rec_update(fl, a, mid, b, l, keep_all);
        }
        rec(fl, loff, mid, b, l);
    };
    auto push_large = [&](const std::vector<int32_t> &fl) {
        const int64_t off = (int64_t)P.large_list.size();
        P.large_list.insert(P.large_list.end(), fl.begin(), fl.end());
        return off;
    };
    auto push_xfers = [&](std::vector<XferSpec> &&x, int32_t l) {
        push(Launch{KC_EXCHANGE, (int32_t)P.xfers.size(), 0, 0, 0.0, 0.0, l});
        P.xfers.push_back(std::move(x));
    };
    // passes over the levels: single GPU = one per branch (stream b), then the top
    // fronts (main stream); multi-GPU = this rank's subtrees, then the top program
    struct Pass { std::vector<char> inc; std::vector<Launch> *prog; int32_t stream; };
    std::vector<Pass> passes;
    if (R == 1 && P.nbranch > 1) {
        for (int32_t b = 0; b <= P.nbranch; b++) {
            const int32_t want = b < P.nbranch ? b : -1;
            std::vector<char> m(ns);
            for (int32_t s = 0; s < ns; s++) m[s] = P.branch[s] == want;
            passes.push_back({std::move(m), &P.program, want});
        }
    } else {
        passes.push_back({inc_local, &P.program, -1});
        passes.push_back({inc_top, &P.program_top, -1});
    }
    for (const Pass &pass : passes) {
    const std::vector<char> &inc = pass.inc;
    cur = pass.prog;
    lookahead_pass = opt.lookahead && opt.ozaki_slices == 0 && R == 1 && pass.stream < 0;
    const size_t pass_begin = cur->size();
    for (int32_t l = 0; l < nlev; l++) {
        std::vector<int32_t> fronts;
        for (int32_t q = P.level_ptr[l]; q < P.level_ptr[l + 1]; q++)
            if (inc[P.level_list[q]]) fronts.push_back(P.level_list[q]);
        for (int32_t fm : fmax_classes) {
            Launch L{KC_SMALL, fm, (int64_t)P.small_list.size(), 0, 0.0, 0.0, l};
            for (int32_t s : fronts)
                if (front_fmax[s] == fm) {
                    P.small_list.push_back(s);
                    const double k = P.sn_k[s], m = P.sn_f[s] - P.sn_k[s];
                    L.flops += k * m * m + m * k * (k + 1) + k * (k + 1) * (2 * k + 1) / 6;
                    L.bytes += asm_bytes(s) + 8.0 * (panel_words(s) + m * (m + 1) / 2);
                }
            L.count = (int64_t)P.small_list.size() - L.off;
            if (L.count) push(L);
        }
        std::vector<int32_t> large;
        for (int32_t s : fronts)
            if (front_fmax[s] == 0) large.push_back(s);
        if (large.empty()) continue;
        std::stable_sort(large.begin(), large.end(), [&](int32_t a, int32_t b) { return P.sn_k[a] > P.sn_k[b]; });
        // assembly (every rank assembles its replica of a top front)
        {
            Launch L{KC_ASSEMBLE, 0, (int64_t)P.asm_tasks.size() / 2, 0, 0.0, 0.0, l};
            for (int32_t s : large) {
                // fused extend-add: only the panel columns (the syrk gathers U^s)
                const int32_t cend = P.fuse_ea ? P.sn_k[s] : P.sn_f[s];
                const int32_t nrb = (P.sn_f[s] + kAsmRowBlock - 1) / kAsmRowBlock;
                if (nrb >= (1 << 11) || cend >= (1 << 20)) return MF_ERR_ARG;   // task encoding
                for (int32_t c0 = 0; c0 < cend; c0 += kAsmCols) {
                    // panel columns span every row; U columns start at their diagonal
                    const int32_t rb0 = c0 < P.sn_k[s] ? 0 : c0 / kAsmRowBlock;
                    for (int32_t rb = rb0; rb < nrb; rb++) {
                        P.asm_tasks.push_back(s);
                        P.asm_tasks.push_back(c0 | (rb << 20));
                    }
                }
                const double f = P.sn_f[s], k = P.sn_k[s], m = f - k;
                if (P.fuse_ea)
                    L.bytes += asm_bytes_panel(s) + 8.0 * f * k;                // write the panel
                else
                    L.bytes += asm_bytes(s) + 8.0 * (f * k + m * (m + 1) / 2);   // zero + write panel and U
            }
            L.count = (int64_t)P.asm_tasks.size() / 2 - L.off;
            push(L);
        }
        // Blocked factorization of the k pivot columns of every large front, in
        // lockstep over the level (Fig. 9: w x w potrf kernel, trsm
        // on the rows below it, trailing update).  The trailing updates follow a
        // recursive split of the block range (left half factored, then ONE update
        // of the right half with inner dimension = the left half's width, then the
        // right half), so most flops run with a long inner dimension instead of
        // w-wide right-looking steps.  A front whose k ends inside the range
        // simply drops out of the launches beyond its last block.
        const int32_t nbw = (P.sn_k[large[0]] + w - 1) / w;
        bool any_dist = false;
        for (int32_t s : large) any_dist = any_dist || P.dist[s];
        if (!any_dist) {
            rec(large, push_large(large), 0, nbw, l);
        } else {
            // distributed: the same recursion over blocks of Wd columns; a block (a
            // "super-leaf") is factored by its owner alone (inner recursion over its
            // leaves) and then broadcast; updates above the block level are split by
            // owned column
            const int32_t nbd = (P.sn_k[large[0]] + Wd - 1) / Wd;
            std::function<void(int32_t, int32_t)> rec_d = [&](int32_t A, int32_t B) {
                if (B - A == 1) {
                    const int32_t t = A;
                    std::vector<int32_t> fl;
                    std::vector<XferSpec> x;
                    for (int32_t s : large) {
                        if (P.sn_k[s] <= t * Wd) continue;
                        if (blk_mine(s, t)) fl.push_back(s);
                        const int32_t o = blk_owner(s, t);
                        if (o >= 0) {   // block columns [t Wd, min(k, (t+1) Wd)), rows t Wd .. f
                            const int32_t ld = P.sn_ld[s], j0 = t * Wd, nc = std::min(P.sn_k[s], j0 + Wd) - j0;
                            x.push_back(XferSpec{MF_XFER_BCAST, o, 0, P.L_off[s] + (int64_t)j0 * ld + j0,
                                                 (int64_t)(nc - 1) * ld + (P.sn_f[s] - j0)});
                        }
                    }
                    if (!fl.empty())
                        rec(fl, push_large(fl), t * kDistLeaves, std::min(nbw, (t + 1) * kDistLeaves), l);
                    if (!x.empty()) push_xfers(std::move(x), l);
                    return;
                }
                const int32_t mid = A + (B - A + 1) / 2;
                rec_d(A, mid);
                // the update of blocks [mid, B) by blocks [A, mid): the generic
                // recursion's update step at leaf granularity, tiles of owned columns
                std::vector<int32_t> fl;
                for (int32_t s : large)
                    if (P.sn_k[s] > mid * Wd) fl.push_back(s);
                if (!fl.empty())
                    rec_update(fl, A * kDistLeaves, mid * kDistLeaves, B * kDistLeaves, l,
                               [&](int32_t s, int32_t col) { return blk_mine(s, col / Wd); });
                rec_d(mid, B);
            };
            rec_d(0, nbd);
        }
        // the syrk on U^n with inner dimension k (one launch for the level); a
        // distributed front's tile columns are split into contiguous ranges balanced
        // by work, then every range is broadcast by the rank that computed it
        Launch Ls{KC_UPDATE, 1, (int64_t)P.tiles.size(), 0, 0.0, 0.0, l};
        std::vector<XferSpec> ux;
        for (int32_t s : large) {
            const int32_t k = P.sn_k[s], f = P.sn_f[s], ld = P.sn_ld[s], m = f - k;
            if (m <= 0) continue;
            GemmProb g;
            g.a_off = P.L_off[s] + k;
            g.c_off = P.U_off[s];
            g.lda = ld;
            g.ldc = m;
            g.M = m;
            g.N = m;
            g.K = k;
            g.flags = 1;
            // odd first row (odd k): shift the problem one row / column up-left
            const int32_t sh = (int32_t)(g.a_off & 1);
            g.a_off -= sh;
            g.M += sh;
            g.N += sh;
            g.flags |= sh << 1;
            // syrk bytes: read the k columns of L2, write the lower U^s; fused
            // extend-add: + the children's entries landing in U^s (and their maps)
            // instead of reading an assembled U^s
            double sbytes = upd_bytes(m, m, k);
            if (P.fuse_ea) {
                g.flags |= kProbGather;
                g.s = s;
                g.qs_off = (int32_t)P.ea_qs.size();
                const int32_t ntr = (g.M + kTileM - 1) / kTileM;
                sbytes = 8.0 * ((double)m * k + (double)m * (m + 1) / 2);
                for (int32_t q = P.child_ptr[s]; q < P.child_ptr[s + 1]; q++) {
                    const int32_t c = P.child_list[q], mc = P.sn_f[c] - P.sn_k[c];
                    const int32_t *rel = P.relmap.data() + P.relmap_ptr[c];
                    // first child row whose parent row is >= max(k, k - sh + 64 t)
                    for (int32_t t = 0; t <= ntr; t++) {
                        const int32_t key = std::max(k, k - sh + kTileM * t);
                        P.ea_qs.push_back((int32_t)(std::lower_bound(rel, rel + mc, key) - rel));
                    }
                    const double mcd = mc;
                    sbytes += 8.0 * (mcd * (mcd + 1) / 2 - child_panel_entries(c, k)) + 4.0 * mc;
                }
                if (P.ea_qs.size() > (size_t)INT32_MAX) return MF_ERR_NOMEM;
            }
            const int32_t pid = (int32_t)P.probs.size();
            P.probs.push_back(g);
            if (!P.dist[s]) {
                add_tiles(P, pid, g.M, g.N, [](int32_t) { return true; });
                Ls.flops += upd_flops(m, m, k);
                Ls.bytes += sbytes;
                continue;
            }
            const std::vector<int32_t> tb = split_tile_columns(g.N, R);
            const int64_t t0 = (int64_t)P.tiles.size();
            add_tiles(P, pid, g.M, g.N, [&](int32_t tj) { return tj >= tb[P.rank] && tj < tb[P.rank + 1]; });
            const double frac = (double)((int64_t)P.tiles.size() - t0) / (double)count_tiles(g.M, g.N);
            Ls.flops += frac * upd_flops(m, m, k);
            Ls.bytes += frac * sbytes;
            for (int r = 0; r < R; r++) {   // original columns of rank r's shifted tile columns
                const int32_t c0 = std::max(0, tb[r] * kTileN - sh), c1 = std::min(m, tb[r + 1] * kTileN - sh);
                if (c1 <= c0) continue;
                ux.push_back(XferSpec{MF_XFER_BCAST, r, 1, P.U_off[s] + upk_col(c0, m),   // packed columns [c0, c1)
                                      upk_col(c1, m) - upk_col(c0, m)});
            }
        }
        Ls.count = (int64_t)P.tiles.size() - Ls.off;
        if (Ls.count) push(Ls);
        if (!ux.empty()) push_xfers(std::move(ux), l);
    }
    if (join_armed || need_join) {   // (cannot happen: every fork is followed by its panel and a launch)
        return MF_ERR_STATE;
    }
    for (size_t i = pass_begin; i < cur->size(); i++) (*cur)[i].stream = pass.stream;
    }   // pass
    for (const GemmProb &g : P.probs)   // the DMMA kernel stages 16-byte row pairs
        if ((g.a_off & 1) || (g.lda & 1)) return MF_ERR_STATE;
    P.df_part_off.assign(ns, -1);
    P.df_seg_off.assign(ns, -1);
    P.dinv_off.assign(ns, -1);
    build_solve_plan(S, P, inc_local, P.fsolve, P.bsolve);
    build_solve_plan(S, P, inc_top_solve, P.fsolve_top, P.bsolve_top);
    return plan_ozaki(P, opt.ozaki_slices);
}

}  // namespace mf
